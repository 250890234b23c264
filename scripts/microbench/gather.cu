// Row-gather throughput microbenchmark (B200): rows of ROWB bytes gathered by a
// warp (16 B per lane) at random row indices, U loads in flight per warp.
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#include <vector>
#include <random>

template <int U>
__global__ void gather(const float4* __restrict__ tab, const int* __restrict__ idx, int n, int rowv,
                       float4* out) {
  const int lane = threadIdx.x & 31;
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int nw = (gridDim.x * blockDim.x) >> 5;
  float4 acc = make_float4(0, 0, 0, 0);
  for (int i = warp * U; i < n; i += nw * U) {
    int r[U];
#pragma unroll
    for (int u = 0; u < U; ++u) r[u] = idx[i + u];
    float4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = tab[(size_t)r[u] * rowv + lane];
#pragma unroll
    for (int u = 0; u < U; ++u) { acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w; }
  }
  if (acc.x == 12345.f) out[0] = acc;
}

int main() {
  const int rowv = 32;  // float4 per row: 512 B
  for (size_t rows : {200000ull, 4000000ull}) {   // 100 MB (L2-ish) and 2 GB (HBM)
    float4* tab; cudaMalloc(&tab, rows * rowv * 16); cudaMemset(tab, 0, rows * rowv * 16);
    const int n = 1 << 24;
    std::vector<int> h(n + 64);
    std::mt19937 g(1); for (auto& x : h) x = g() % rows;
    int* idx; cudaMalloc(&idx, h.size() * 4); cudaMemcpy(idx, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
    float4* out; cudaMalloc(&out, 16);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    for (int blocks_per_sm : {4, 8, 16}) {
      for (int U : {1, 4, 8}) {
        auto run = [&]() {
          dim3 grid(148 * blocks_per_sm);
          if (U == 1) gather<1><<<grid, 128>>>(tab, idx, n, rowv, out);
          if (U == 4) gather<4><<<grid, 128>>>(tab, idx, n, rowv, out);
          if (U == 8) gather<8><<<grid, 128>>>(tab, idx, n, rowv, out);
        };
        run(); cudaDeviceSynchronize();
        cudaEventRecord(a); for (int r = 0; r < 5; ++r) run(); cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b); ms /= 5;
        printf("table %6.0f MB  blocks/SM %2d  U %d : %.3f ms  %.0f GB/s of rows\n", rows * 512 / 1e6,
               blocks_per_sm, U, ms, (double)n * 512 / ms / 1e6);
      }
    }
    cudaFree(tab); cudaFree(idx); cudaFree(out);
  }
  return 0;
}
