// Debug: one CTA, D[128 x NM] = A[128 x K] B[K x NM] with tcgen05 kind::tf32,
// A K-major and B MN-major in no-swizzle core-matrix layouts; tries the
// LBO / SBO assignments and reports the max error against a host product.
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <vector>
#include <cstdlib>
#include <cuda_runtime.h>

constexpr int M = 128, NM = 64, K = 32;

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t a, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((a >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
         ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46);
}

__global__ void kern(const float* A, const float* B, float* D, int variant) {
  __shared__ __align__(1024) float sa[M * K];
  __shared__ __align__(1024) float sb[K * NM];
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase;
  const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  // A element (r,k): core (k/4, r/8) at ((k/4)*16 + r/8)*128 B + (r%8)*16 + (k%4)*4
  for (int i = tid; i < M * K; i += blockDim.x) {
    const int r = i / K, k = i % K;
    sa[(((k / 4) * 16 + r / 8) * 128 + (r % 8) * 16 + (k % 4) * 4) / 4] = A[r * K + k];
  }
  // B element (k,n): core (n/4, k/8) at ((k/8)*(NM/4) + n/4)*128 + (k%8)*16 + (n%4)*4
  for (int i = tid; i < K * NM; i += blockDim.x) {
    const int k = i / NM, n = i % NM;
    if (variant < 8)
      sb[(((k / 8) * (NM / 4) + n / 4) * 128 + (k % 8) * 16 + (n % 4) * 4) / 4] = B[k * NM + n];
    else  // K-major B: core (n/8, k/4) at ((k/4)*(NM/8) + n/8)*128 + (n%8)*16 + (k%4)*4
      sb[(((k / 4) * (NM / 8) + n / 8) * 128 + (n % 8) * 16 + (k % 4) * 4) / 4] = B[k * NM + n];
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 64;" ::"r"(su32(&tbase)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tm = tbase;
  // pre-fill D with 1000 + row via tcgen05.st so we can tell "MMA did nothing" from "ld broken"
  for (int c = 0; c < NM; c += 16) {
    uint32_t v[16];
    for (int x = 0; x < 16; ++x) v[x] = __float_as_uint(1000.f + warp * 32 + lane);
    asm volatile("tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};"
                 :: "r"(tm + ((uint32_t)(warp * 32) << 16) + c), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]),
                    "r"(v[6]), "r"(v[7]), "r"(v[8]), "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15]));
  }
  asm volatile("tcgen05.wait::st.sync.aligned;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t A_LBO = 16 * 128, A_SBO = 128, B_LBO = (NM / 4) * 128, B_SBO = 128;
  const uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | (variant < 8 ? (1u << 16) : 0u) |
                         ((uint32_t)(NM >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
  if (tid == 0) {
    for (int ks = 0; ks < K / 8; ++ks) {
      uint64_t da, db;
      const uint32_t a0 = su32(sa) + ks * 2 * A_LBO, b0 = su32(sb) + ks * B_LBO;
      if (variant >= 8) { da = desc(a0, A_LBO, A_SBO); db = desc(su32(sb) + ks * 2 * (NM / 8) * 128, (NM / 8) * 128, 128); }
      else if (variant % 4 == 0) { da = desc(a0, A_LBO, A_SBO); db = desc(b0, B_LBO, B_SBO); }
      else if (variant % 4 == 1) { da = desc(a0, A_SBO, A_LBO); db = desc(b0, B_LBO, B_SBO); }
      else if (variant % 4 == 2) { da = desc(a0, A_LBO, A_SBO); db = desc(b0, B_SBO, B_LBO); }
      else { da = desc(a0, A_SBO, A_LBO); db = desc(b0, B_SBO, B_LBO); }
      const uint32_t acc = (variant >= 4) ? 1u : (ks > 0);
      asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                   "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tm),
                   "l"(da), "l"(db), "r"(IDESC), "r"(acc));
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)));
  }
  asm volatile("{\n\t.reg .pred P;\nW:\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n\t@!P bra W;\n}" ::"r"(su32(&bar)));
  asm volatile("tcgen05.fence::after_thread_sync;");
  for (int c = 0; c < NM; c += 16) {
    uint32_t v[16];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                   "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
                 : "r"(tm + ((uint32_t)(warp * 32) << 16) + c));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    for (int x = 0; x < 16; ++x) D[(warp * 32 + lane) * NM + c + x] = __uint_as_float(v[x]);
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 64;" ::"r"(tm));
}

int main() {
  std::vector<float> A(M * K), B(K * NM), D(M * NM), R(M * NM, 0.f);
  const bool ones = getenv("ONES") != nullptr;
  for (int i = 0; i < M * K; ++i) A[i] = ones ? 1.f : (float)((i * 7) % 13) - 6.f;   // small integers: exact in tf32
  for (int i = 0; i < K * NM; ++i) B[i] = ones ? 1.f : (float)((i * 5) % 11) - 5.f;
  for (int r = 0; r < M; ++r)
    for (int n = 0; n < NM; ++n) {
      double s = 0;
      for (int k = 0; k < K; ++k) s += (double)A[r * K + k] * B[k * NM + n];
      R[r * NM + n] = (float)s;
    }
  float *dA, *dB, *dD;
  cudaMalloc(&dA, A.size() * 4); cudaMalloc(&dB, B.size() * 4); cudaMalloc(&dD, D.size() * 4);
  cudaMemcpy(dA, A.data(), A.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, B.data(), B.size() * 4, cudaMemcpyHostToDevice);
  int vs[2] = {8, 0};
  for (int vi = 0; vi < 2; ++vi) { const int v = vs[vi];
    cudaMemset(dD, 0, D.size() * 4);
    kern<<<1, 128>>>(dA, dB, dD, v);
    cudaError_t e = cudaDeviceSynchronize();
    cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
    double err = 0;
    for (int i = 0; i < M * NM; ++i) err = fmax(err, fabs(D[i] - R[i]));
    printf("variant %d: %s max err %g  D[0]=%g R[0]=%g D[1]=%g R[1]=%g D[NM]=%g R[NM]=%g\n", v,
           cudaGetErrorString(e), err, D[0], R[0], D[1], R[1], D[NM], R[NM]);
  }
  return 0;
}
