// Row gathers: register loads (float4 per lane, double-buffered) vs 1D TMA
// bulk copies (cp.async.bulk -> shared ring, mbarrier) of 512-byte rows.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tma_gather tma_gather.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
#include <cuda.h>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); return 1; } } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// each warp: n_batches batches of 12 rows (idx[12*b + r]); sums rows into acc
__global__ void k_ldg(const float* __restrict__ rows, const int* __restrict__ idx, int n_batches,
                      float* out) {
  const int lane = threadIdx.x & 31;
  const int w = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32;
  const int nw = gridDim.x * (blockDim.x / 32);
  float4 acc = make_float4(0, 0, 0, 0);
  for (int b = w; b < n_batches; b += nw) {
    float4 v[12];
#pragma unroll
    for (int r = 0; r < 12; ++r) {
      const int j = __ldg(idx + 12 * b + r);
      v[r] = __ldg(reinterpret_cast<const float4*>(rows + (size_t)j * 128) + lane);
    }
#pragma unroll
    for (int r = 0; r < 12; ++r) { acc.x += v[r].x; acc.y += v[r].y; acc.z += v[r].z; acc.w += v[r].w; }
  }
  out[(size_t)w * 32 + lane] = acc.x + acc.y + acc.z + acc.w;
}

template <int S, int FENCE>
__global__ void k_tma(const float* __restrict__ rows, const int* __restrict__ idx, int n_batches,
                      float* out) {
  extern __shared__ __align__(128) unsigned char sm[];
  const int lane = threadIdx.x & 31, wi = threadIdx.x / 32;
  const int w = blockIdx.x * (blockDim.x / 32) + wi;
  const int nw = gridDim.x * (blockDim.x / 32);
  float* ring = reinterpret_cast<float*>(sm) + (size_t)wi * S * 12 * 128;
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + (size_t)(blockDim.x / 32) * S * 12 * 512) + wi * S;
  if (lane == 0)
    for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(bars + s)));
  asm volatile("fence.mbarrier_init.release.cluster;");
  __syncwarp();
  auto issue = [&](int j, int s) {  // lanes 0..11 copy one row each
    if (lane == 0)
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(bars + s)), "r"(12 * 512));
    __syncwarp();
    if (lane < 12) {
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 512, [%2];"
                   ::"r"(su32(ring + (size_t)(s * 12 + lane) * 128)), "l"(rows + (size_t)j * 128),
                   "r"(su32(bars + s)) : "memory");
    }
  };
  int n = 0;
  for (int b = w; b < n_batches && n < S - 1; b += nw, ++n) issue(lane < 12 ? __ldg(idx + 12 * b + lane) : 0, n);
  // indices of the batch to issue next, loaded one iteration ahead
  int jn = 0;
  {
    const int bn = w + (S - 1) * nw;
    if (bn < n_batches && lane < 12) jn = __ldg(idx + 12 * bn + lane);
  }
  float4 acc = make_float4(0, 0, 0, 0);
  int it = 0;
  for (int b = w; b < n_batches; b += nw, ++it) {
    const int s = it % S;
    const uint32_t ph = (it / S) & 1;
    // prefetch b + (S-1) batches ahead into the stage consumed last iteration
    const int bn = b + (S - 1) * nw;
    if (bn < n_batches) {
      if (FENCE) asm volatile("fence.proxy.async.shared::cta;");
      issue(jn, (it + S - 1) % S);
      const int bnn = bn + nw;
      if (bnn < n_batches && lane < 12) jn = __ldg(idx + 12 * bnn + lane);
    }
    asm volatile("{\n\t.reg .pred P;\n\tWAIT_%=:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
                 "@!P bra WAIT_%=;\n\t}" ::"r"(su32(bars + s)), "r"(ph) : "memory");
#pragma unroll
    for (int r = 0; r < 12; ++r) {
      const float4 v = reinterpret_cast<const float4*>(ring + (size_t)(s * 12 + r) * 128)[lane];
      acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
    __syncwarp();
  }
  out[(size_t)w * 32 + lane] = acc.x + acc.y + acc.z + acc.w;
}

// gather4: one tensor-TMA instruction brings 4 rows (box {128, 1} x 4 row coords)
template <int S, int MODE>
__global__ void k_g4(const __grid_constant__ CUtensorMap tmap, const int* __restrict__ idx,
                     int n_batches, float* out) {
  extern __shared__ __align__(128) unsigned char sm[];
  const int lane = threadIdx.x & 31, wi = threadIdx.x / 32;
  const int w = blockIdx.x * (blockDim.x / 32) + wi;
  const int nw = gridDim.x * (blockDim.x / 32);
  float* ring = reinterpret_cast<float*>(sm) + (size_t)wi * S * 12 * 128;
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + (size_t)(blockDim.x / 32) * S * 12 * 512) + wi * S;
  if (lane == 0)
    for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(bars + s)));
  asm volatile("fence.mbarrier_init.release.cluster;");
  __syncwarp();
  auto issue = [&](int j, int s) {  // lanes 0..11 hold the 12 row ids; lanes 0,4,8 issue a gather4
    const int j1 = __shfl_down_sync(0xffffffffu, j, 1), j2 = __shfl_down_sync(0xffffffffu, j, 2),
              j3 = __shfl_down_sync(0xffffffffu, j, 3);
    if (lane == 0)
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(bars + s)), "r"(12 * 512));
    __syncwarp();
    if (lane < 12 && (lane & 3) == 0) {
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
                   " [%0], [%1, {%3, %4, %5, %6, %7}], [%2];"
                   ::"r"(su32(ring + (size_t)(s * 12 + lane) * 128)), "l"(&tmap), "r"(su32(bars + s)),
                   "r"(0), "r"(j), "r"(j1), "r"(j2), "r"(j3) : "memory");
    }
  };
  int n = 0;
  for (int b = w; b < n_batches && n < S - 1; b += nw, ++n) issue(lane < 12 ? __ldg(idx + 12 * b + lane) : 0, n);
  int jn = 0;
  {
    const int bn = w + (S - 1) * nw;
    if (bn < n_batches && lane < 12) jn = __ldg(idx + 12 * bn + lane);
  }
  float4 acc = make_float4(0, 0, 0, 0);
  int it = 0;
  for (int b = w; b < n_batches; b += nw, ++it) {
    const int s = it % S;
    const uint32_t ph = (it / S) & 1;
    const int bn = b + (S - 1) * nw;
    if (bn < n_batches) {
      asm volatile("fence.proxy.async.shared::cta;");
      issue(jn, (it + S - 1) % S);
      const int bnn = bn + nw;
      if (bnn < n_batches && lane < 12) jn = __ldg(idx + 12 * bnn + lane);
    }
    if (MODE != 2)
    asm volatile("{\n\t.reg .pred P;\n\tWAIT_%=:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
                 "@!P bra WAIT_%=;\n\t}" ::"r"(su32(bars + s)), "r"(ph) : "memory");
    if (MODE != 1) {
#pragma unroll
    for (int r = 0; r < 12; ++r) {
      const float4 v = reinterpret_cast<const float4*>(ring + (size_t)(s * 12 + r) * 128)[lane];
      acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
    }
    __syncwarp();
  }
  out[(size_t)w * 32 + lane] = acc.x + acc.y + acc.z + acc.w;
}

int main() {
  const int R = 168160, NB = 5500000 / 4;  // rows; batches of 12 rows (4 slots x 3 arrays)
  // three arrays as one (g, pi, am): R*3 rows, locality: slot rows near each other
  std::vector<float> h((size_t)3 * R * 128, 1.f);
  std::vector<int> idx((size_t)12 * NB);
  std::mt19937 rng(1);
  for (int b = 0; b < NB; ++b) {
    const int base = (int)((double)b / NB * R);
    for (int u = 0; u < 4; ++u) {
      int j = base + (int)(rng() % 2000) - 1000;
      j = j < 0 ? 0 : (j >= R ? R - 1 : j);
      for (int a = 0; a < 3; ++a) idx[12 * b + 4 * a + u] = a * R + j;
    }
  }
  float *rows, *out;
  int* di;
  CK(cudaMalloc(&rows, h.size() * 4));
  CK(cudaMalloc(&di, idx.size() * 4));
  CK(cudaMalloc(&out, (size_t)1 << 28));
  CK(cudaMemcpy(rows, h.data(), h.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(di, idx.data(), idx.size() * 4, cudaMemcpyHostToDevice));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  const double bytes = (double)NB * 12 * 512;
  for (int blocks_per_sm : {4, 8, 12, 16}) {
    const int grid = 148 * blocks_per_sm;
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(e0);
      k_ldg<<<grid, 64>>>(rows, di, NB, out);
      cudaEventRecord(e1);
      CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      if (rep) printf("ldg  64thr x %2d/SM: %.3f ms  %.2f TB/s\n", blocks_per_sm, ms, bytes / ms / 1e9);
    }
  }
  auto run_tma = [&](auto kern, int S, int warps, int blocks_per_sm) -> int {
    const size_t smem = (size_t)warps * S * (12 * 512 + 8);
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(e0);
      kern<<<148 * blocks_per_sm, 32 * warps, smem>>>(rows, di, NB, out);
      cudaEventRecord(e1);
      CK(cudaEventSynchronize(e1));
      CK(cudaGetLastError());
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      if (rep) printf("tma S=%d warps=%d x %d/SM (smem %zu KB): %.3f ms  %.2f TB/s\n", S, warps, blocks_per_sm,
                      smem / 1024, ms, bytes / ms / 1e9);
    }
    return 0;
  };
  run_tma(k_tma<2, 1>, 2, 16, 1);
  // tensor map over the [3R][128] fp32 rows
  typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                               const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                               CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
  CUtensorMap tmap;
  cuuint64_t dims[2] = {128, (cuuint64_t)3 * R};
  cuuint64_t strides[1] = {128 * 4};
  cuuint32_t box[2] = {128, 1};
  cuuint32_t es[2] = {1, 1};
  CUresult cr = ((EncodeFn)fn)(&tmap, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, rows, dims, strides, box, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                               CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("encode: %d\n", (int)cr);
  auto run_g4 = [&](auto kern, int S, int warps, int blocks_per_sm) -> int {
    const size_t smem = (size_t)warps * S * (12 * 512 + 8) + 1024;
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(e0);
      kern<<<148 * blocks_per_sm, 32 * warps, smem>>>(tmap, di, NB, out);
      cudaEventRecord(e1);
      CK(cudaEventSynchronize(e1));
      CK(cudaGetLastError());
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      if (rep) printf("g4 S=%d warps=%d x %d/SM (smem %zu KB): %.3f ms  %.2f TB/s\n", S, warps, blocks_per_sm,
                      smem / 1024, ms, bytes / ms / 1e9);
    }
    return 0;
  };
  run_g4(k_g4<2, 0>, 2, 16, 1);
  run_g4(k_g4<4, 0>, 4, 8, 1);
  run_g4(k_g4<4, 1>, 4, 8, 1);   // wait, no smem reads
  run_g4(k_g4<2, 0>, 2, 32, 1);
  run_g4(k_g4<3, 0>, 3, 20, 1);
  return 0;
}
