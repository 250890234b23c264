// Layout check for the tf32 UMMA operands of k_mlp_l1_tma: A = W tile
// [64 rows x 32 k] in the stored K-major core order (lo rows zero), B = p
// [32 k x 64 seeds] brought in by tensor TMA with the 128-byte swizzle and read
// MN-major.  D = A B on the tensor cores vs the host product of small integers
// (exact in tf32).  Descriptor fields are arguments so that their meaning can
// be established by measurement:
//   ./umma_layout a_lbo a_sbo b_lbo b_sbo b_swz b_major raw_lowbits
// nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o umma_layout umma_layout.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#define CK(x)                                                                         \
  do {                                                                                \
    cudaError_t e = (x);                                                              \
    if (e != cudaSuccess) {                                                           \
      printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e));                \
      return 1;                                                                       \
    }                                                                                 \
  } while (0)

constexpr int BC = 64, NM = 128, KB = 32;

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t a, uint32_t lbo, uint32_t sbo, uint32_t swz) {
  return (uint64_t)((a >> 4) & 0x3FFFu) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
         ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46) | ((uint64_t)swz << 61);
}

__global__ void k_umma(const float* wt, const float* bk, const __grid_constant__ CUtensorMap tm, float* d, uint32_t a_lbo,
                  uint32_t a_sbo, uint32_t b_lbo, uint32_t b_sbo, uint32_t b_swz, uint32_t b_major) {
  extern __shared__ __align__(1024) uint8_t raw[];
  uint8_t* sm = raw + ((1024u - (su32(raw) & 1023u)) & 1023u);
  uint8_t* sa = sm;               // 16 KB: hi 8 KB, lo 8 KB (zero)
  uint8_t* sb = sm + 16384;       // 16 KB: hi blocks 2 x 4 KB, lo (zero)
  __shared__ uint64_t bar, done;
  __shared__ uint32_t tmem_sh;
  const int tid = threadIdx.x;
  for (int i = tid; i < 32768 / 4; i += blockDim.x) reinterpret_cast<float*>(sm)[i] = 0.f;
  if (tid < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" ::"r"(su32(&tmem_sh)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&done)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_sh;
  if (tid == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar)), "r"(b_major ? 8192 + 8192 : 8192 + 16384));
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 8192, [%2];" ::"r"(
                     su32(sa)), "l"(wt), "r"(su32(&bar)) : "memory");
    if (!b_major)  // host-built K-major B (core (k/4, n/8) at (k/4) * 2048 + (n/8) * 128)
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 16384, [%2];" ::"r"(
                       su32(sb)), "l"(bk), "r"(su32(&bar)) : "memory");
    else
    for (int j = 0; j < 2; ++j)
      asm volatile(
          "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
          " [%0], [%1, {%2, %3}], [%4];" ::"r"(su32(sb + j * 4096)), "l"(&tm), "r"(32 * j), "r"(0),
          "r"(su32(&bar)) : "memory");
    asm volatile(
        "{\n\t.reg .pred P;\nW1:\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n\t@!P bra W1;\n}" ::"r"(
            su32(&bar)));
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | (b_major << 16) | ((uint32_t)(NM >> 3) << 17) |
                           ((uint32_t)(128 >> 4) << 24);
    for (int ks = 0; ks < KB / 8; ++ks) {
      const uint64_t da = desc(su32(sa) + ks * 2 * a_lbo, a_lbo, a_sbo, 0);
      const uint64_t db = desc(su32(sb) + ks * (b_major ? b_sbo : 2 * b_lbo), b_lbo, b_sbo, b_swz);
      const uint32_t acc = ks > 0;
      asm volatile(
          "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
          "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
          "l"(da), "l"(db), "r"(idesc), "r"(acc));
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&done)));
  }
  __syncwarp();
  asm volatile(
      "{\n\t.reg .pred P;\nW2:\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n\t@!P bra W2;\n}" ::"r"(
          su32(&done)));
  __syncwarp();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const int w = tid / 32, lane = tid % 32;
  for (int c = 0; c < NM; ++c) {
    uint32_t v;
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%1];" : "=r"(v) : "r"(tmem + ((uint32_t)(w * 32) << 16) + c));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    d[(w * 32 + lane) * NM + c] = __uint_as_float(v);
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (tid < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" ::"r"(tmem));
}

int main(int argc, char** argv) {
  const uint32_t a_lbo = argc > 1 ? atoi(argv[1]) : 128, a_sbo = argc > 2 ? atoi(argv[2]) : 1024;
  const uint32_t b_lbo = argc > 3 ? atoi(argv[3]) : 4096, b_sbo = argc > 4 ? atoi(argv[4]) : 1024;
  const uint32_t b_swz = argc > 5 ? atoi(argv[5]) : 2, b_major = argc > 6 ? atoi(argv[6]) : 1;
  const int lowbits = argc > 7 ? atoi(argv[7]) : 0;
  std::vector<float> W(64 * KB), P(KB * BC), wt(2048, 0.f);
  for (int h = 0; h < 64; ++h)
    for (int k = 0; k < KB; ++k) W[h * KB + k] = (float)((h * 7 + k * 3) % 11 - 5);
  for (int k = 0; k < KB; ++k)
    for (int s = 0; s < BC; ++s) P[k * BC + s] = (float)((k * 5 + s * 13) % 9 - 4);
  for (int h = 0; h < 64; ++h)
    for (int k = 0; k < KB; ++k) wt[((h / 8) * 1024 + (k / 4) * 128 + (h % 8) * 16 + (k % 4) * 4) / 4] = W[h * KB + k];
  std::vector<float> Praw = P;
  if (lowbits)  // set low mantissa bits: a truncating MMA ignores them
    for (auto* v : {&wt, &Praw})
      for (auto& x : *v) {
        uint32_t b;
        memcpy(&b, &x, 4);
        if (x != 0.f) b |= 0x1FFFu;
        memcpy(&x, &b, 4);
      }
  std::vector<float> bk(4096, 0.f);
  for (int k = 0; k < KB; ++k)
    for (int n = 0; n < BC; ++n) bk[((k / 4) * 2048 + (n / 8) * 128 + (n % 8) * 16 + (k % 4) * 4) / 4] = Praw[k * BC + n];
  float *dwt, *dp, *dd, *dbk;
  CK(cudaMalloc(&dbk, 16384));
  CK(cudaMemcpy(dbk, bk.data(), 16384, cudaMemcpyHostToDevice));
  CK(cudaMalloc(&dwt, 8192));
  CK(cudaMalloc(&dp, KB * BC * 4));
  CK(cudaMalloc(&dd, 128 * NM * 4));
  CK(cudaMemcpy(dwt, wt.data(), 8192, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dp, Praw.data(), KB * BC * 4, cudaMemcpyHostToDevice));
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
  typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                          const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                          CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
  CUtensorMap tm;
  const cuuint64_t dims[2] = {BC, KB}, strides[1] = {BC * 4};
  const cuuint32_t box[2] = {32, KB}, es[2] = {1, 1};
  if (((Enc)fn)(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, dp, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                b_swz == 2 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
    printf("encode failed\n");
    return 1;
  }
  CK(cudaFuncSetAttribute(k_umma, cudaFuncAttributeMaxDynamicSharedMemorySize, 32768 + 1024));
  k_umma<<<1, 128, 32768 + 1024>>>(dwt, dbk, tm, dd, a_lbo, a_sbo, b_lbo, b_sbo, b_swz, b_major);
  CK(cudaDeviceSynchronize());
  std::vector<float> D(128 * NM);
  CK(cudaMemcpy(D.data(), dd, D.size() * 4, cudaMemcpyDeviceToHost));
  int bad = 0, first = -1;
  for (int h = 0; h < 64; ++h)
    for (int s = 0; s < BC; ++s) {
      double ref = 0;
      for (int k = 0; k < KB; ++k) ref += (double)W[h * KB + k] * P[k * BC + s];
      if (D[h * NM + s] != (float)ref) {
        if (first < 0) first = h * NM + s;
        ++bad;
      }
    }
  printf("D[0][0..3] %g %g %g %g\n", D[0], D[1], D[2], D[3]);
  int nz = 0;
  for (int h = 0; h < 128; ++h)
    for (int s = 0; s < NM; ++s)
      if ((h >= 64 || s >= BC) && D[h * NM + s] != 0.f) ++nz;
  printf("a_lbo %u a_sbo %u b_lbo %u b_sbo %u swz %u bmajor %u lowbits %d: %d of 4096 wrong, %d nonzero outside",
         a_lbo, a_sbo, b_lbo, b_sbo, b_swz, b_major, lowbits, bad, nz);
  if (first >= 0) {
    const int h = first / NM, s = first % NM;
    double ref = 0;
    for (int k = 0; k < KB; ++k) ref += (double)W[h * KB + k] * P[k * BC + s];
    printf(" (first h %d s %d got %g want %g)", h, s, D[first], ref);
  }
  printf("\n");
  return 0;
}
