// Device-side helpers shared by the kernels of libsmoothe (sm_100a).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "internal.h"

namespace smoothe {

// Every per-seed array is [row][Bp] fp32, seed innermost.  A "row group" of
// LPR lanes covers one chunk of 4*LPR seeds of one row with float4 accesses
// (Bp = 32 -> LPR 8, Bp = 64 -> LPR 16, Bp >= 128 -> LPR 32 and Bp/128
// chunks).  Grids are 2-D: x over rows, y over chunks, so a row group never
// straddles chunks and block reductions are per seed.
constexpr int kBlock = 256;

__host__ __device__ inline int lanes_per_row(int Bp) { return Bp >= 128 ? 32 : Bp / 4; }
__host__ __device__ inline int num_chunks(int Bp) { return Bp >= 128 ? Bp / 128 : 1; }

template <int LPR, int BLOCK = kBlock>
struct RowGroup {
  int row;   // row index (class or node)
  int s0;    // first seed of this lane (multiple of 4)
  int sub;   // group index inside the block
  __device__ RowGroup() {
    const int lane = threadIdx.x % LPR;
    sub = threadIdx.x / LPR;
    row = blockIdx.x * (BLOCK / LPR) + sub;
    s0 = blockIdx.y * (4 * LPR) + lane * 4;
  }
};

inline dim3 row_grid(int rows, int Bp, int LPR, int block = kBlock) {
  return dim3((rows + block / LPR - 1) / (block / LPR), num_chunks(Bp));
}

// Class kernels (softmax, cost, update): blocks [0, num_big) each take one
// class with more than kBigClass e-nodes (its row groups stride over the
// class's e-nodes and reduce through shared memory, so no row group walks a
// 900-node class alone); later blocks hold one row group per class and skip
// the big ones.
inline dim3 class_grid(int rows, int Bp, int LPR, int num_big, int block = kBlock) {
  return dim3(num_big + (rows + block / LPR - 1) / (block / LPR), num_chunks(Bp));
}

// Sum of a float4 over the R = kBlock / LPR row groups of a block, in row
// group order (deterministic); every thread receives the total for its lane.
template <int LPR>
__device__ __forceinline__ float4 block_sum_rows(float4 (*red)[LPR], float4 v) {
  const int lane = threadIdx.x % LPR, sub = threadIdx.x / LPR;
  red[sub][lane] = v;
  __syncthreads();
  float4 acc = red[0][lane];
  for (int r = 1; r < kBlock / LPR; ++r) {
    const float4 w = red[r][lane];
    acc.x += w.x; acc.y += w.y; acc.z += w.z; acc.w += w.w;
  }
  __syncthreads();
  return acc;
}

// Per-class sums in a big-class block that do not depend on Bp: e-node
// k0 + i belongs to part i mod 32, each part is summed in e-node order by one
// row group (row group sub owns parts sub, sub + R, ...), and the 32 part sums
// are added in part order.  So a seed's result is the same bits whatever the
// batch it runs in (seed sharding stays bit-identical).
constexpr int kClassParts = 32;
template <int LPR>
struct PartSums {
  static constexpr int R = kBlock / LPR, PP = kClassParts / R;
  float4 acc[PP];
  __device__ PartSums() {
#pragma unroll
    for (int q = 0; q < PP; ++q) acc[q] = make_float4(0.f, 0.f, 0.f, 0.f);
  }
  // f(i, acc) for every e-node i of [k0, k1) this thread's parts own
  template <typename F>
  __device__ void run(int k0, int k1, F f) {
    const int sub = threadIdx.x / LPR;
#pragma unroll
    for (int q = 0; q < PP; ++q)
      for (int i = k0 + sub + q * R; i < k1; i += kClassParts) f(i, acc[q]);
  }
  __device__ float4 total(float4 (*red)[LPR]) const {  // red: [kClassParts][LPR]
    const int lane = threadIdx.x % LPR, sub = threadIdx.x / LPR;
#pragma unroll
    for (int q = 0; q < PP; ++q) red[sub + q * R][lane] = acc[q];
    __syncthreads();
    float4 t = red[0][lane];
    for (int r = 1; r < kClassParts; ++r) {
      const float4 w = red[r][lane];
      t.x += w.x; t.y += w.y; t.z += w.z; t.w += w.w;
    }
    __syncthreads();
    return t;
  }
};

__device__ __forceinline__ float4 ld4(const float* p) { return *reinterpret_cast<const float4*>(p); }
__device__ __forceinline__ int4 ld4i(const int32_t* p) { return *reinterpret_cast<const int4*>(p); }
__device__ __forceinline__ void st4(float* p, float4 v) { *reinterpret_cast<float4*>(p) = v; }
// evict-first ("streaming") variants for rows touched once per launch, so they
// do not displace the rows that are gathered many times from L2
__device__ __forceinline__ float4 ldcs4(const float* p) { return __ldcs(reinterpret_cast<const float4*>(p)); }
__device__ __forceinline__ void stcs4(float* p, float4 v) { __stcs(reinterpret_cast<float4*>(p), v); }
__device__ __forceinline__ void stcs4i(int32_t* p, int4 v) { __stcs(reinterpret_cast<int4*>(p), v); }
__device__ __forceinline__ void st4i(int32_t* p, int4 v) { *reinterpret_cast<int4*>(p) = v; }

__device__ __forceinline__ float comp(const float4& v, int c) {
  return c == 0 ? v.x : c == 1 ? v.y : c == 2 ? v.z : v.w;
}
__device__ __forceinline__ float& comp(float4& v, int c) {
  return c == 0 ? v.x : c == 1 ? v.y : c == 2 ? v.z : v.w;
}
__device__ __forceinline__ int comp(const int4& v, int c) {
  return c == 0 ? v.x : c == 1 ? v.y : c == 2 ? v.z : v.w;
}
__device__ __forceinline__ int& comp(int4& v, int c) {
  return c == 0 ? v.x : c == 1 ? v.y : c == 2 ? v.z : v.w;
}

#define SM_DISPATCH_LPR(Bp, ...)            \
  do {                                      \
    const int _lpr = lanes_per_row(Bp);     \
    if (_lpr == 32) {                       \
      constexpr int LPR = 32;               \
      __VA_ARGS__;                          \
    } else if (_lpr == 16) {                \
      constexpr int LPR = 16;               \
      __VA_ARGS__;                          \
    } else {                                \
      constexpr int LPR = 8;                \
      __VA_ARGS__;                          \
    }                                       \
  } while (0)

#define SM_LAUNCH_CHECK()                                        \
  do {                                                           \
    ++::smoothe::launch_counter();                               \
    SM_CUDA(cudaGetLastError());                                 \
  } while (0)

// ---------------------------------------------------------------------------
// tcgen05 / mbarrier helpers (the tensor-core kernels: MLP layer 1, the
// large-component matrix exponential)
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

// p advanced to the next 1 KB boundary of the shared window, by arithmetic on
// the shared pointer itself: a round trip through uintptr_t loses the address
// space and turns every access into a generic LD.E / ST.E.
__device__ __forceinline__ uint8_t* smem_align1024(uint8_t* p) {
  return p + ((1024u - (smem_u32(p) & 1023u)) & 1023u);
}
// no-swizzle UMMA shared-memory descriptor (sm_100 version 1)
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
         ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
      "@!P bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
      "r"(parity));
}
__device__ __forceinline__ float4 tf32_hi(float4 v) {
  auto h = [](float x) { return __uint_as_float(__float_as_uint(x) & 0xFFFFE000u); };
  return make_float4(h(v.x), h(v.y), h(v.z), h(v.w));
}
__device__ __forceinline__ float4 sub4(float4 a, float4 b) {
  return make_float4(a.x - b.x, a.y - b.y, a.z - b.z, a.w - b.w);
}

}  // namespace smoothe
