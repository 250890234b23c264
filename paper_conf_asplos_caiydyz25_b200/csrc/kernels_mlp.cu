// MLP cost model f_mlp(p) = W3 relu(W2 relu(W1 p + b1) + b2) + b3 (
// reading S22: N -> 64 -> 8 -> 1) and its gradient.
//
// Layer 1 is the only large contraction: z1[h][b] = sum_k W1[h][k] p[k][b]
// (2*H1*N*B flop) and g_p[k][b] += sum_h W1[h][k] gz1[h][b] (same); both run
// on the tensor cores.  Split-K partial sums are reduced in a fixed order, so
// results are deterministic.
#include <cstdlib>
#include <cstring>
#include <vector>

#include "kcommon.cuh"

namespace smoothe {

constexpr int kMlpMaxH1 = 64;
constexpr int kMlpMaxH2 = 16;

// ---------------------------------------------------------------------------
// Layer 1 on the 5th-generation tensor cores (tcgen05, kind::tf32, fp32
// accumulation in TMEM), split-K over the e-nodes.
//
// TF32 keeps 10 mantissa bits, too few for the 1e-4 parity bar, so both
// operands are split x = hi + lo (hi = x with the low 13 mantissa bits
// cleared, lo = x - hi exactly) and one M=128 x N=2Bc x K=8 MMA per K step
// computes all four products at once:
//   A = [W1_hi ; W1_lo]  (128 x K, K-major: W1 rows are K-contiguous)
//   B = [p_hi | p_lo]    (K x 2Bc, staged K-major: 4 x 4 blocks of p are
//                          transposed in registers; MN-major tf32 operands
//                          without swizzle read as zeros on sm_100a, measured)
//   D = A B,   z1 = D[h][b] + D[h][Bc+b] + D[64+h][b] + D[64+h][Bc+b]
// (the lo*lo term is ~2^-22 relative and harmless).  Each CTA owns one seed
// chunk of Bc <= 128 seeds and a contiguous e-node range, streams W1 and p
// once (register loads one K block ahead, hi/lo split on the way into the
// canonical no-swizzle UMMA layouts in shared memory), one thread issues the
// MMAs, tcgen05.commit releases each stage, and the 4 warps read their 32 TMEM
// lanes back at the end: z1_part[cta][128][Bp] (rows 64.. hold the W1_lo
// products), reduced in a fixed order by k_mlp_reduce.
// ---------------------------------------------------------------------------
#ifndef SMOOTHE_TC_KB
#define SMOOTHE_TC_KB 64
#endif
constexpr int kTcKB = SMOOTHE_TC_KB;  // e-nodes (K) per stage (16 float4 loads in flight per thread)
template <int BC>
#ifndef SMOOTHE_TC_S128
#define SMOOTHE_TC_S128 2
#endif
__host__ __device__ constexpr int tc_stages() { return BC >= 128 ? SMOOTHE_TC_S128 : 3; }  // <= 192 KB of shared memory
constexpr int kTcThreads = 128;

template <int BC>
__global__ void __launch_bounds__(kTcThreads, 1) k_mlp_l1_tc(int N, int Bp, int H1, int nsplit,
                                                            const float* __restrict__ W1,
                                                            const float* __restrict__ p,
                                                            float* __restrict__ z1_part) {
  constexpr int NM = 2 * BC;                       // MMA N
  constexpr int A_BYTES = 128 * kTcKB * 4;         // [W1_hi; W1_lo]
  constexpr int B_BYTES = kTcKB * NM * 4;          // [p_hi | p_lo]
  constexpr int STAGE = A_BYTES + B_BYTES;
  constexpr int A_LBO = 16 * 128;                  // K-chunk (4 elements) stride
  constexpr int B_LBO = (NM / 8) * 128;            // K-chunk (4 elements) stride
  constexpr int AV = 64 * kTcKB / 4 / kTcThreads;  // float4 of W1 per thread per stage
  constexpr int BBLK = (kTcKB / 4) * (BC / 4);     // 4 x 4 blocks of p per stage
  constexpr int BV = (BBLK + kTcThreads - 1) / kTcThreads;
  constexpr uint32_t TMEM_COLS = NM <= 32 ? 32 : NM <= 64 ? 64 : NM <= 128 ? 128 : 256;
  // kind::tf32, D f32, A and B K-major, M = 128, N = NM
  constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(NM >> 3) << 17) |
                             ((uint32_t)(128 >> 4) << 24);
  extern __shared__ __align__(1024) uint8_t tc_smem[];
  constexpr int kTcStages = tc_stages<BC>();
  __shared__ uint64_t bar[kTcStages + 1];
  __shared__ uint32_t tmem_base_sh;
  const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  const int seed0 = blockIdx.y * BC;
  const int64_t per = (((int64_t)N + nsplit - 1) / nsplit + kTcKB - 1) / kTcKB * kTcKB;
  const int64_t kb64 = (int64_t)blockIdx.x * per;
  const int k_begin = (int)(kb64 < N ? kb64 : N);
  const int k_end = (int)(k_begin + per < N ? k_begin + per : N);
  const int nkb = (k_end - k_begin + kTcKB - 1) / kTcKB;

  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(&tmem_base_sh)),
                 "n"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    for (int i = 0; i <= kTcStages; ++i) mbar_init(&bar[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_base_sh;

  float4 ra[AV], rb[BV][4];
  auto load = [&](int kb) {
    const int k0 = k_begin + kb * kTcKB;
#pragma unroll
    for (int i = 0; i < AV; ++i) {
      const int idx = tid + i * kTcThreads, h = idx / (kTcKB / 4), k = k0 + (idx % (kTcKB / 4)) * 4;
      ra[i] = make_float4(0.f, 0.f, 0.f, 0.f);
      if (h < H1) {
        const float* src = W1 + (size_t)h * N + k;
        if (k + 3 < k_end && ((reinterpret_cast<uintptr_t>(src) & 15) == 0)) {
          ra[i] = __ldcs(reinterpret_cast<const float4*>(src));
        } else {
          float t[4];
#pragma unroll
          for (int x = 0; x < 4; ++x) t[x] = k + x < k_end ? src[x] : 0.f;
          ra[i] = make_float4(t[0], t[1], t[2], t[3]);
        }
      }
    }
#pragma unroll
    for (int i = 0; i < BV; ++i) {
      const int idx = tid + i * kTcThreads;
      const int k = k0 + (idx / (BC / 4)) * 4, n = (idx % (BC / 4)) * 4;
#pragma unroll
      for (int r = 0; r < 4; ++r)
        rb[i][r] = idx < BBLK && k + r < k_end
                       ? __ldcs(reinterpret_cast<const float4*>(p + (size_t)(k + r) * Bp + seed0 + n))
                       : make_float4(0.f, 0.f, 0.f, 0.f);
    }
  };
  auto store = [&](int st) {
    uint8_t* sa = tc_smem + st * STAGE;
    uint8_t* sb = sa + A_BYTES;
#pragma unroll
    for (int i = 0; i < AV; ++i) {
      const int idx = tid + i * kTcThreads, h = idx / (kTcKB / 4), kc = idx % (kTcKB / 4);
      const float4 hi = tf32_hi(ra[i]), lo = sub4(ra[i], hi);
      // element (r, k): core (k/4, r/8) at (kc * 16 + r/8) * 128, + (r%8) * 16
      *reinterpret_cast<float4*>(sa + (kc * 16 + h / 8) * 128 + (h % 8) * 16) = hi;
      *reinterpret_cast<float4*>(sa + (kc * 16 + 8 + h / 8) * 128 + (h % 8) * 16) = lo;
    }
#pragma unroll
    for (int i = 0; i < BV; ++i) {
      const int idx = tid + i * kTcThreads;
      if (idx >= BBLK) continue;
      const int kc = idx / (BC / 4), n = (idx % (BC / 4)) * 4;  // K chunk, first seed
#pragma unroll
      for (int x = 0; x < 4; ++x) {  // seed n + x: its 4 K values, transposed
        const float4 col = make_float4(comp(rb[i][0], x), comp(rb[i][1], x), comp(rb[i][2], x),
                                       comp(rb[i][3], x));
        const float4 hi = tf32_hi(col), lo = sub4(col, hi);
        // element (k, m) (m = output column): core (k/4, m/8) at
        // ((k/4) * NM/8 + m/8) * 128, + (m%8) * 16 + (k%4) * 4
        const int m = n + x;
        *reinterpret_cast<float4*>(sb + (kc * (NM / 8) + m / 8) * 128 + (m % 8) * 16) = hi;
        *reinterpret_cast<float4*>(sb + (kc * (NM / 8) + (BC + m) / 8) * 128 + (m % 8) * 16) = lo;
      }
    }
  };

  if (nkb > 0) load(0);
  for (int kb = 0; kb < nkb; ++kb) {
    const int st = kb % kTcStages;
    if (kb >= kTcStages) mbar_wait(&bar[st], (uint32_t)((kb / kTcStages - 1) & 1));
    store(st);
    if (kb + 1 < nkb) load(kb + 1);  // next block in flight while this one multiplies
    asm volatile("fence.proxy.async.shared::cta;");
    __syncthreads();
    if (tid == 0) {
      asm volatile("tcgen05.fence::after_thread_sync;");
      const uint32_t sa = smem_u32(tc_smem + st * STAGE), sb = sa + A_BYTES;
#pragma unroll
      for (int ks = 0; ks < kTcKB / 8; ++ks) {
        const uint64_t da = umma_desc(sa + ks * 2 * A_LBO, A_LBO, 128);
        const uint64_t db = umma_desc(sb + ks * 2 * B_LBO, B_LBO, 128);
        const uint32_t acc = (kb > 0 || ks > 0) ? 1u : 0u;
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
            "l"(da), "l"(db), "r"(IDESC), "r"(acc));
      }
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
          smem_u32(&bar[st])));
    }
  }
  // all MMAs done -> accumulator readable
  if (tid == 0) {
    if (nkb > 0)
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
          smem_u32(&bar[kTcStages])));
    else
      asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&bar[kTcStages])));
  }
  mbar_wait(&bar[kTcStages], 0);
  __syncwarp();  // lanes leave the wait loop separately: converge before .sync.aligned tcgen05 ops
  asm volatile("tcgen05.fence::after_thread_sync;");
  // warp w reads TMEM lanes 32w..32w+31 = D rows; thread = one row
  const int row = warp * 32 + lane;
  float* out = z1_part + ((size_t)blockIdx.x * 128 + row) * Bp + seed0;
  if (nkb == 0) {  // no e-nodes in this CTA's range: the accumulator was never written
#pragma unroll
    for (int c = 0; c < BC; c += 4) *reinterpret_cast<float4*>(out + c) = make_float4(0.f, 0.f, 0.f, 0.f);
  }
#pragma unroll
  for (int c = 0; c < BC && nkb > 0; c += 16) {
    uint32_t v[16], w[16];
    const uint32_t ta = tmem + ((uint32_t)(warp * 32) << 16) + c;
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
          "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]),
          "=r"(v[14]), "=r"(v[15])
        : "r"(ta));
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]),
          "=r"(w[7]), "=r"(w[8]), "=r"(w[9]), "=r"(w[10]), "=r"(w[11]), "=r"(w[12]), "=r"(w[13]),
          "=r"(w[14]), "=r"(w[15])
        : "r"(ta + BC));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
#pragma unroll
    for (int x = 0; x < 16; x += 4)
      *reinterpret_cast<float4*>(out + c + x) =
          make_float4(__uint_as_float(v[x]) + __uint_as_float(w[x]),
                      __uint_as_float(v[x + 1]) + __uint_as_float(w[x + 1]),
                      __uint_as_float(v[x + 2]) + __uint_as_float(w[x + 2]),
                      __uint_as_float(v[x + 3]) + __uint_as_float(w[x + 3]));
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) {
    __syncwarp();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(TMEM_COLS));
  }
}

// ---------------------------------------------------------------------------
// Layer 1 with TMA-fed, warp-specialised stages (the default; SMOOTHE_MLP_TMA=0
// keeps the register-staged kernel above).
//  * A = [W1_hi; W1_lo] (M = 128, K-major).  The run keeps W1 in tiles of 32
//    e-nodes (`mlp_w1_tiles`, 8 KB, already in the no-swizzle K-major core
//    order); one 1-D bulk copy puts a tile into the A_hi half of a stage.
//  * The MMA reads an fp32 operand as tf32 by dropping the low 13 mantissa
//    bits (scripts/microbench/umma_layout.cu: operands with all 13 low bits
//    set give the exact products of the truncated values), so the raw W1 tile
//    IS A_hi; the converter warps only write A_lo = x - trunc(x) next to it,
//    element for element.
//  * B = [p_hi | p_lo] (N = 2 Bc, K-major).  p is stored seeds-contiguous,
//    i.e. MN-major for B, and a tf32 MMA with the MN-major bit set returned
//    zeros on this part (same microbenchmark), so p is transposed on chip:
//    tensor TMA brings the raw tile [32 e-nodes x Bc seeds], and each
//    converter thread builds one 16-byte K-major core row (4 e-nodes of one
//    seed) from four 4-byte loads; a warp reads whole 128-byte rows and
//    writes 512 contiguous bytes, so neither side has bank conflicts.
// One thread issues the MMAs (M=128 x N=2Bc x K=8, all four products as in
// k_mlp_l1_tc), tcgen05.commit hands each stage back to the producer; the
// converter warps read the accumulator back.  Output: z1_part as k_mlp_l1_tc.
//   warp 0: TMA producer, warp 1: MMA issuer, warps 2..2+kTmCW-1: converters +
//   epilogue (warp w reads TMEM lanes 32 (w % 4).., column part (w - 2) / 4)
// (C5 layer 1: W1 as 2-D TMA tiles of W1^T, both operands transposed as 4 x 4
// register blocks, 64 us; W1 stored pre-split -- twice the bytes -- 48.5 us;
// the 4 x 4 blocks' stores were 4-way bank-conflicted, and shared-memory
// bandwidth was the limit: 29 us with the converters skipped.)
// ---------------------------------------------------------------------------
constexpr int kTmKB = 32;                          // e-nodes per stage
constexpr int kTmWBytes = 64 * kTmKB * 4;          // one stored W1 tile (8 KB)
#ifndef SMOOTHE_TM_CW
#define SMOOTHE_TM_CW 8
#endif
constexpr int kTmCW = SMOOTHE_TM_CW;               // converter warps (C5: 8 -> 33.5 us, 4 -> 35.5)
constexpr int kTmThreads = 64 + 32 * kTmCW;
template <int BC>
__host__ __device__ constexpr int tm_stages() { return BC >= 128 ? 3 : BC >= 64 ? 5 : 7; }
template <int BC>  // A [hi; lo], B [hi | lo], raw p tile
__host__ __device__ constexpr int tm_stage_bytes() { return 2 * kTmWBytes + 3 * BC * kTmKB * 4; }
template <int BC>
__host__ __device__ constexpr int tm_smem() { return tm_stages<BC>() * tm_stage_bytes<BC>() + 1024; }

template <int BC>
__global__ void __launch_bounds__(kTmThreads, 1) k_mlp_l1_tma(const float* __restrict__ w1tiles,
                                                             const __grid_constant__ CUtensorMap tm_p,
                                                             int N, int Bp, int nsplit,
                                                             float* __restrict__ z1_part) {
  constexpr int NM = 2 * BC;
  constexpr int S = tm_stages<BC>(), SB = tm_stage_bytes<BC>();
  constexpr int A_BYTES = 2 * kTmWBytes;          // [hi; lo]
  constexpr int PB = BC * kTmKB * 4;              // the raw p tile
  constexpr int B_BYTES = 2 * PB;                 // [hi | lo]
  // A: core (e-node quad kc, hidden-unit octet g) at g * 1024 + kc * 128
  constexpr uint32_t A_LBO = 128, A_SBO = 1024;
  // B: core (e-node quad kc, seed octet) at kc * B_LBO + (n / 8) * 128
  constexpr uint32_t B_LBO = (NM / 8) * 128, B_SBO = 128;
  constexpr uint32_t TMEM_COLS = NM <= 32 ? 32 : NM <= 64 ? 64 : NM <= 128 ? 128 : 256;
  constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(NM >> 3) << 17) |
                             ((uint32_t)(128 >> 4) << 24);
  extern __shared__ __align__(1024) uint8_t tm_smem_raw[];
  uint8_t* smem = smem_align1024(tm_smem_raw);
  __shared__ uint64_t full[S], conv[S], empty[S], acc_full;
  __shared__ uint32_t tmem_sh;
  const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  const int seed0 = blockIdx.y * BC;
  const int64_t per = (((int64_t)N + nsplit - 1) / nsplit + kTmKB - 1) / kTmKB * kTmKB;
  const int64_t kb64 = (int64_t)blockIdx.x * per;
  const int k_begin = (int)(kb64 < N ? kb64 : N);
  const int k_end = (int)(k_begin + per < N ? k_begin + per : N);
  const int nkb = (k_end - k_begin + kTmKB - 1) / kTmKB;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(&tmem_sh)),
                 "n"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&conv[i], kTmCW);  // one arrival per converter warp
      mbar_init(&empty[i], 1);     // tcgen05.commit
    }
    mbar_init(&acc_full, 1);
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_sh;

  if (warp == 0) {  // producer: W1 tile (bulk copy) -> A_hi, p tile (tensor TMA) -> raw
    if (lane == 0)
      for (int kb = 0; kb < nkb; ++kb) {
        const int st = kb % S;
        const int k0 = k_begin + kb * kTmKB;
        if (kb >= S) mbar_wait(&empty[st], (uint32_t)((kb / S - 1) & 1));
        const uint32_t bar = smem_u32(&full[st]);
        const uint32_t dst = smem_u32(smem + st * SB);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar),
                     "r"(kTmWBytes + PB));
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                dst),
            "l"(w1tiles + (size_t)(k0 / kTmKB) * (kTmWBytes / 4)), "r"(kTmWBytes), "r"(bar)
            : "memory");
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
            " [%0], [%1, {%2, %3}], [%4];" ::"r"(dst + A_BYTES + B_BYTES),
            "l"(&tm_p), "r"(seed0), "r"(k0), "r"(bar)
            : "memory");
      }
  } else if (warp == 1) {  // MMA issuer
    if (lane == 0) {
      for (int kb = 0; kb < nkb; ++kb) {
        const int st = kb % S;
        mbar_wait(&conv[st], (uint32_t)((kb / S) & 1));
        asm volatile("tcgen05.fence::after_thread_sync;");
        const uint32_t sa = smem_u32(smem + st * SB), sb = sa + A_BYTES;
#pragma unroll
        for (int ks = 0; ks < kTmKB / 8; ++ks) {
          const uint64_t da = umma_desc(sa + ks * 2 * A_LBO, A_LBO, A_SBO);
          const uint64_t db = umma_desc(sb + ks * 2 * B_LBO, B_LBO, B_SBO);
          const uint32_t acc = (kb > 0 || ks > 0) ? 1u : 0u;
          asm volatile(
              "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
              "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
              "l"(da), "l"(db), "r"(IDESC), "r"(acc));
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
            smem_u32(&empty[st])));
      }
      if (nkb > 0)
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
            smem_u32(&acc_full)));
      else
        asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&acc_full)));
    }
  } else {  // converters: A_lo next to A_hi, B from the raw p tile; then the epilogue
    const int ct = tid - 64;
    for (int kb = 0; kb < nkb; ++kb) {
      const int st = kb % S;
      mbar_wait(&full[st], (uint32_t)((kb / S) & 1));
      uint8_t* sa = smem + st * SB;
      uint8_t* sb = sa + A_BYTES;
#pragma unroll
      for (int i = ct; i < kTmWBytes / 16; i += 32 * kTmCW) {
        const float4 w = *reinterpret_cast<const float4*>(sa + i * 16);
        *reinterpret_cast<float4*>(sa + kTmWBytes + i * 16) = sub4(w, tf32_hi(w));
      }
      // B core row (kc, n): p[4 kc .. 4 kc + 3][n], raw (k, n) at (k * BC + n) * 4
      const float* rp = reinterpret_cast<const float*>(sb + B_BYTES);
#pragma unroll
      for (int i = ct; i < (kTmKB / 4) * BC; i += 32 * kTmCW) {
        const int kc = i / BC, n = i % BC;
        const float4 x = make_float4(rp[(4 * kc) * BC + n], rp[(4 * kc + 1) * BC + n],
                                     rp[(4 * kc + 2) * BC + n], rp[(4 * kc + 3) * BC + n]);
        const int off = kc * B_LBO + (n / 8) * 128 + (n % 8) * 16;
        *reinterpret_cast<float4*>(sb + off) = x;  // the MMA truncates: x is B_hi
        *reinterpret_cast<float4*>(sb + off + (BC / 8) * 128) = sub4(x, tf32_hi(x));
      }
      asm volatile("fence.proxy.async.shared::cta;");
      __syncwarp();
      if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&conv[st])));
    }
    mbar_wait(&acc_full, 0);
    __syncwarp();  // lanes leave the wait loop separately: converge before .sync.aligned tcgen05 ops
    asm volatile("tcgen05.fence::after_thread_sync;");
    const int q = warp % 4;  // TMEM lanes 32q .. 32q + 31 = D rows
    constexpr int PARTS = kTmCW / 4, CH = BC / PARTS >= 16 ? BC / PARTS : 16;
    const int c0 = ((warp - 2) / 4) * CH;
    const int row = q * 32 + lane;
    float* out = z1_part + ((size_t)blockIdx.x * 128 + row) * Bp + seed0;
    if (c0 < BC && nkb == 0) {
#pragma unroll
      for (int c = 0; c < CH; c += 4)
        *reinterpret_cast<float4*>(out + c0 + c) = make_float4(0.f, 0.f, 0.f, 0.f);
    }
#pragma unroll
    for (int cc = 0; cc < CH; cc += 16) {
      const int c = c0 + cc;
      if (c >= BC || nkb == 0) break;
      uint32_t v[16], w[16];
      const uint32_t ta = tmem + ((uint32_t)(q * 32) << 16) + c;
      asm volatile(
          "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
          : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
            "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]),
            "=r"(v[14]), "=r"(v[15])
          : "r"(ta));
      asm volatile(
          "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
          : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]),
            "=r"(w[7]), "=r"(w[8]), "=r"(w[9]), "=r"(w[10]), "=r"(w[11]), "=r"(w[12]), "=r"(w[13]),
            "=r"(w[14]), "=r"(w[15])
          : "r"(ta + BC));
      asm volatile("tcgen05.wait::ld.sync.aligned;");
#pragma unroll
      for (int x = 0; x < 16; x += 4)
        *reinterpret_cast<float4*>(out + c + x) =
            make_float4(__uint_as_float(v[x]) + __uint_as_float(w[x]),
                        __uint_as_float(v[x + 1]) + __uint_as_float(w[x + 1]),
                        __uint_as_float(v[x + 2]) + __uint_as_float(w[x + 2]),
                        __uint_as_float(v[x + 3]) + __uint_as_float(w[x + 3]));
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) {
    __syncwarp();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(TMEM_COLS));
  }
}

// W1 laid out for k_mlp_l1_tma, once per run: ceil(N / 32) tiles of
// kTmWBytes, element (hidden unit h, e-node k) of tile kb at core (k/4, h/8):
// (h/8) * 1024 + (k/4) * 128 + (h%8) * 16 + (k%4) * 4 bytes; hidden units
// >= H1 and e-nodes >= N are zero.
std::vector<float> mlp_w1_tiles(const float* W1, int H1, int N) {
  const int nblk = (N + kTmKB - 1) / kTmKB;
  std::vector<float> t((size_t)nblk * (kTmWBytes / 4), 0.f);
  for (int kb = 0; kb < nblk; ++kb) {
    float* tile = t.data() + (size_t)kb * (kTmWBytes / 4);
    for (int kk = 0; kk < kTmKB && kb * kTmKB + kk < N; ++kk)
      for (int h = 0; h < H1 && h < 64; ++h)
        tile[((h / 8) * 1024 + (kk / 4) * 128 + (h % 8) * 16 + (kk % 4) * 4) / 4] =
            W1[(size_t)h * N + kb * kTmKB + kk];
  }
  return t;
}

// z1[h][b] = b1[h] + sum over CTAs (in order) of rows h and 64 + h.  One
// block per hidden unit and 32 seeds: 8 warps stage the per-CTA terms
// (coalesced, all loads in flight) in shared memory, then warp 0 adds them in
// CTA order (the in-order sum over 148 CTAs was latency-bound: 34 us on C5).
constexpr int kRedMaxSplit = 256;
__global__ void __launch_bounds__(256) k_mlp_reduce(int Bp, int H1, int nsplit, const float* __restrict__ b1,
                                                    const float* __restrict__ z1_part, float* __restrict__ z1) {
  __shared__ float xs[kRedMaxSplit][33];
  const int h = blockIdx.x, b = blockIdx.y * 32 + threadIdx.x % 32, w = threadIdx.x / 32;
  const size_t cs = (size_t)128 * Bp, lo = (size_t)64 * Bp;
  const float* q = z1_part + (size_t)h * Bp + b;
  for (int c = w; c < nsplit; c += 8) xs[c][threadIdx.x % 32] = q[c * cs] + q[c * cs + lo];
  __syncthreads();
  if (w != 0) return;
  float acc = 0.f;
  for (int c = 0; c < nsplit; ++c) acc += xs[c][threadIdx.x];
  z1[(size_t)h * Bp + b] = b1[h] + acc;
}

// Per seed (one warp, lanes over hidden units): layers 2-3, f_mlp, and
// gz1 = d f_mlp / d z1.  Layer-2 sums are warp trees in a fixed order.
__global__ void __launch_bounds__(128) k_mlp_head(int Bp, int H1, int H2, const float* __restrict__ z1g,
                                                  const float* __restrict__ W2, const float* __restrict__ b2,
                                                  const float* __restrict__ W3, const float* __restrict__ b3,
                                                  double* __restrict__ f_mlp, float* __restrict__ gz1) {
  const int b = blockIdx.x * 4 + threadIdx.x / 32, lane = threadIdx.x % 32;
  if (b >= Bp) return;
  constexpr int HL = kMlpMaxH1 / 32;  // hidden units per lane: lane, lane + 32
  float z1[HL];
#pragma unroll
  for (int r = 0; r < HL; ++r) {
    const int h = lane + 32 * r;
    z1[r] = h < H1 ? z1g[(size_t)h * Bp + b] : 0.f;
  }
  float y = b3[0];
  uint32_t pos = 0;  // bit h2: z2[h2] > 0
  for (int h2 = 0; h2 < H2; ++h2) {
    float part = 0.f;
#pragma unroll
    for (int r = 0; r < HL; ++r) {
      const int h = lane + 32 * r;
      if (h < H1) part = fmaf(W2[h2 * H1 + h], fmaxf(z1[r], 0.f), part);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
    const float z2 = b2[h2] + part;
    y += W3[h2] * fmaxf(z2, 0.f);
    if (z2 > 0.f) pos |= 1u << h2;
  }
  if (lane == 0) f_mlp[b] = (double)y;
  if (gz1) {
#pragma unroll
    for (int r = 0; r < HL; ++r) {
      const int h = lane + 32 * r;
      if (h >= H1) continue;
      float acc = 0.f;
      for (int h2 = 0; h2 < H2; ++h2)
        if (pos >> h2 & 1u) acc += W2[h2 * H1 + h] * W3[h2];
      gz1[(size_t)h * Bp + b] = z1[r] > 0.f ? acc : 0.f;  // ReLU'(0) = 0 (S25)
    }
  }
}

// ---------------------------------------------------------------------------
// Backward of layer 1 on the tensor cores: g_p[k][b] = u[k] + sum_h W1[h][k] gz1[h][b].
// One CTA per tile of 128 e-nodes (M) and seed chunk: A = W1^T tile (128 x H1,
// staged K-major: 4 x 4 blocks transposed in registers) split hi / lo into two
// tiles, B = [gz1_hi | gz1_lo] (H1 x 2Bc, K-major), two MMAs per K step:
//   D = A_hi B + A_lo B,   g_p = u + D[m][b] + D[m][Bc + b].
// ---------------------------------------------------------------------------
template <int BC>
__global__ void __launch_bounds__(kTcThreads) k_mlp_l1_back_tc(int N, int Bp, int H1,
                                                              const float* __restrict__ W1,
                                                              const float* __restrict__ u,
                                                              const float* __restrict__ gz1,
                                                              float* __restrict__ gp) {
  constexpr int NM = 2 * BC;
  constexpr int KH = kMlpMaxH1;                 // K = 64 (H1 padded with zeros)
  constexpr int A_BYTES = 128 * KH * 4;         // one of A_hi / A_lo
  constexpr int A_LBO = 16 * 128;               // K chunk stride (16 row groups of 8)
  constexpr int B_LBO = (NM / 8) * 128;
  constexpr uint32_t TMEM_COLS = NM <= 32 ? 32 : NM <= 64 ? 64 : NM <= 128 ? 128 : 256;
  constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(NM >> 3) << 17) |
                             ((uint32_t)(128 >> 4) << 24);
  extern __shared__ __align__(1024) uint8_t tc_smem[];
  __shared__ uint64_t bar;
  __shared__ uint32_t tmem_base_sh;
  uint8_t* sAh = tc_smem;
  uint8_t* sAl = tc_smem + A_BYTES;
  uint8_t* sB = tc_smem + 2 * A_BYTES;
  const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  const int k0 = blockIdx.x * 128, seed0 = blockIdx.y * BC;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(&tmem_base_sh)),
                 "n"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    mbar_init(&bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  // A: node m, hidden h -> core (h/4, m/8) at ((h/4) * 16 + m/8) * 128 + (m%8) * 16 + (h%4) * 4
  for (int blk = tid; blk < (KH / 4) * (128 / 4); blk += kTcThreads) {
    const int hc = blk / 32, m0 = (blk % 32) * 4;  // 4 hidden units x 4 nodes
    float4 r[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int h = hc * 4 + i;
      const float* src = W1 + (size_t)h * N + k0 + m0;
      if (h < H1 && k0 + m0 + 3 < N && ((reinterpret_cast<uintptr_t>(src) & 15) == 0)) {
        r[i] = __ldcs(reinterpret_cast<const float4*>(src));
      } else {
        float t[4];
#pragma unroll
        for (int x = 0; x < 4; ++x) t[x] = h < H1 && k0 + m0 + x < N ? src[x] : 0.f;
        r[i] = make_float4(t[0], t[1], t[2], t[3]);
      }
    }
#pragma unroll
    for (int x = 0; x < 4; ++x) {
      const int m = m0 + x;
      const float4 col = make_float4(comp(r[0], x), comp(r[1], x), comp(r[2], x), comp(r[3], x));
      const float4 hi = tf32_hi(col), lo = sub4(col, hi);
      const int off = (hc * 16 + m / 8) * 128 + (m % 8) * 16;
      *reinterpret_cast<float4*>(sAh + off) = hi;
      *reinterpret_cast<float4*>(sAl + off) = lo;
    }
  }
  // B: hidden h (K), column c (N) -> core (h/4, c/8) at ((h/4) * NM/8 + c/8) * 128 + (c%8) * 16 + (h%4) * 4
  for (int blk = tid; blk < (KH / 4) * (BC / 4); blk += kTcThreads) {
    const int hc = blk / (BC / 4), n0 = (blk % (BC / 4)) * 4;
    float4 r[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int h = hc * 4 + i;
      r[i] = h < H1 ? *reinterpret_cast<const float4*>(gz1 + (size_t)h * Bp + seed0 + n0)
                    : make_float4(0.f, 0.f, 0.f, 0.f);
    }
#pragma unroll
    for (int x = 0; x < 4; ++x) {
      const int c = n0 + x;
      const float4 col = make_float4(comp(r[0], x), comp(r[1], x), comp(r[2], x), comp(r[3], x));
      const float4 hi = tf32_hi(col), lo = sub4(col, hi);
      *reinterpret_cast<float4*>(sB + (hc * (NM / 8) + c / 8) * 128 + (c % 8) * 16) = hi;
      *reinterpret_cast<float4*>(sB + (hc * (NM / 8) + (BC + c) / 8) * 128 + (c % 8) * 16) = lo;
    }
  }
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_base_sh;
  if (tid == 0) {
    const uint32_t ah = smem_u32(sAh), al = smem_u32(sAl), bb = smem_u32(sB);
#pragma unroll
    for (int ks = 0; ks < KH / 8; ++ks) {
      const uint64_t db = umma_desc(bb + ks * 2 * B_LBO, B_LBO, 128);
#pragma unroll
      for (int part = 0; part < 2; ++part) {
        const uint64_t da = umma_desc((part ? al : ah) + ks * 2 * A_LBO, A_LBO, 128);
        const uint32_t acc = (ks > 0 || part > 0) ? 1u : 0u;
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
            "l"(da), "l"(db), "r"(IDESC), "r"(acc));
      }
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
        smem_u32(&bar)));
  }
  mbar_wait(&bar, 0);
  __syncwarp();  // lanes leave the wait loop separately: converge before .sync.aligned tcgen05 ops
  asm volatile("tcgen05.fence::after_thread_sync;");
  const int m = warp * 32 + lane, k = k0 + m;
  const float uk = k < N ? __ldg(u + k) : 0.f;
  float* out = gp + (size_t)k * Bp + seed0;
#pragma unroll
  for (int c = 0; c < BC; c += 16) {
    uint32_t v[16], w[16];
    const uint32_t ta = tmem + ((uint32_t)(warp * 32) << 16) + c;
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
          "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]),
          "=r"(v[14]), "=r"(v[15])
        : "r"(ta));
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]),
          "=r"(w[7]), "=r"(w[8]), "=r"(w[9]), "=r"(w[10]), "=r"(w[11]), "=r"(w[12]), "=r"(w[13]),
          "=r"(w[14]), "=r"(w[15])
        : "r"(ta + BC));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    if (k < N) {
#pragma unroll
      for (int x = 0; x < 16; x += 4)
        __stcs(reinterpret_cast<float4*>(out + c + x),
               make_float4(uk + (__uint_as_float(v[x]) + __uint_as_float(w[x])),
                           uk + (__uint_as_float(v[x + 1]) + __uint_as_float(w[x + 1])),
                           uk + (__uint_as_float(v[x + 2]) + __uint_as_float(w[x + 2])),
                           uk + (__uint_as_float(v[x + 3]) + __uint_as_float(w[x + 3]))));
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) {
    __syncwarp();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(TMEM_COLS));
  }
}

// ---------------------------------------------------------------------------
// Backward of layer 1, persistent and TMA-fed (the default; SMOOTHE_MLP_TMA=0
// keeps k_mlp_l1_back_tc): the same products in the same order as
// k_mlp_l1_back_tc, so g_p is bit for bit the same.  Per CTA: one seed chunk
// and every gridDim.x-th tile of 128 e-nodes.
//  * B = [gz1_hi | gz1_lo] (K = 64 hidden units) is built once per CTA and
//    stays in shared memory.
//  * A_hi = the W1^T tile, kept by the run in the K-major core order
//    (`mlp_w1_back_tiles`, 32 KB per tile): one bulk copy, used raw (the MMA
//    truncates to tf32); converter warps write A_lo = x - trunc(x) next to it.
//  * The accumulator is double-buffered in TMEM, so the epilogue of tile i
//    overlaps the MMAs of tile i + 1; the epilogue adds u, writes the tile
//    into a 128-byte-swizzled staging buffer (conflict-free) and one thread
//    stores it with tensor TMA (rows past N clipped).
//   warp 0: producer, warp 1: MMA issuer, warps 2-5: converters, warps 6-9: epilogue
// ---------------------------------------------------------------------------
constexpr int kBkABytes = 128 * kMlpMaxH1 * 4;  // one W1^T tile (32 KB)
constexpr int kBkThreads = 64 + 8 * 32;
template <int BC>
__host__ __device__ constexpr int bk_stages() { return BC >= 128 ? 1 : 2; }
template <int BC>
__host__ __device__ constexpr int bk_smem() {
  return bk_stages<BC>() * 2 * kBkABytes + kMlpMaxH1 * 2 * BC * 4 + 128 * BC * 4 + 1024;
}

template <int BC>
__global__ void __launch_bounds__(kBkThreads, 1) k_mlp_l1_back_tma(const float* __restrict__ w1b,
                                                                  const __grid_constant__ CUtensorMap tm_gp,
                                                                  int N, int Bp, int H1,
                                                                  const float* __restrict__ u,
                                                                  const float* __restrict__ gz1) {
  constexpr int NM = 2 * BC, KH = kMlpMaxH1, S = bk_stages<BC>();
  constexpr uint32_t A_LBO = 16 * 128, B_LBO = (NM / 8) * 128;
  constexpr uint32_t TMEM_COLS = 2 * NM <= 32 ? 32 : 2 * NM <= 64 ? 64 : 2 * NM <= 128 ? 128 : 2 * NM <= 256 ? 256 : 512;
  constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(NM >> 3) << 17) |
                             ((uint32_t)(128 >> 4) << 24);
  extern __shared__ __align__(1024) uint8_t bk_smem_raw[];
  uint8_t* smem = smem_align1024(bk_smem_raw);
  uint8_t* sA = smem;                                // S x [hi 32 KB | lo 32 KB]
  uint8_t* sB = smem + S * 2 * kBkABytes;            // KH x 2BC, K-major
  uint8_t* stg = sB + KH * NM * 4;                   // BC/32 blocks of [128 rows][128 B], swizzled
  __shared__ uint64_t a_full[S], a_conv[S], a_empty[S], acc_full[2], acc_empty[2];
  __shared__ uint32_t tmem_sh;
  const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  const int seed0 = blockIdx.y * BC;
  const int ntiles = (N + 127) / 128;
  const int nt = blockIdx.x < ntiles ? (ntiles - 1 - (int)blockIdx.x) / (int)gridDim.x + 1 : 0;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(&tmem_sh)),
                 "n"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&a_full[i], 1);
      mbar_init(&a_conv[i], 4);
      mbar_init(&a_empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&acc_full[i], 1);
      mbar_init(&acc_empty[i], 4);
    }
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  // B: hidden h (K), column c (N) -> core (h/4, c/8) at ((h/4) * NM/8 + c/8) * 128 + (c%8) * 16 + (h%4) * 4
  for (int blk = tid; blk < (KH / 4) * (BC / 4); blk += kBkThreads) {
    const int hc = blk / (BC / 4), n0 = (blk % (BC / 4)) * 4;
    float4 r[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int h = hc * 4 + i;
      r[i] = h < H1 ? *reinterpret_cast<const float4*>(gz1 + (size_t)h * Bp + seed0 + n0)
                    : make_float4(0.f, 0.f, 0.f, 0.f);
    }
#pragma unroll
    for (int x = 0; x < 4; ++x) {
      const int c = n0 + x;
      const float4 col = make_float4(comp(r[0], x), comp(r[1], x), comp(r[2], x), comp(r[3], x));
      const float4 hi = tf32_hi(col), lo = sub4(col, hi);
      *reinterpret_cast<float4*>(sB + (hc * (NM / 8) + c / 8) * 128 + (c % 8) * 16) = hi;
      *reinterpret_cast<float4*>(sB + (hc * (NM / 8) + (BC + c) / 8) * 128 + (c % 8) * 16) = lo;
    }
  }
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_sh;

  if (warp == 0) {  // producer
    if (lane == 0)
      for (int i = 0; i < nt; ++i) {
        const int st = i % S, tile = blockIdx.x + i * gridDim.x;
        if (i >= S) mbar_wait(&a_empty[st], (uint32_t)((i / S - 1) & 1));
        const uint32_t bar = smem_u32(&a_full[st]);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(kBkABytes));
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                smem_u32(sA + st * 2 * kBkABytes)),
            "l"(w1b + (size_t)tile * (kBkABytes / 4)), "r"(kBkABytes), "r"(bar)
            : "memory");
      }
  } else if (warp == 1) {  // MMA issuer
    if (lane == 0)
      for (int i = 0; i < nt; ++i) {
        const int st = i % S, d = i & 1;
        mbar_wait(&a_conv[st], (uint32_t)((i / S) & 1));
        if (i >= 2) mbar_wait(&acc_empty[d], (uint32_t)((i / 2 - 1) & 1));
        asm volatile("tcgen05.fence::after_thread_sync;");
        const uint32_t ah = smem_u32(sA + st * 2 * kBkABytes), al = ah + kBkABytes, bb = smem_u32(sB);
#pragma unroll
        for (int ks = 0; ks < KH / 8; ++ks) {
          const uint64_t db = umma_desc(bb + ks * 2 * B_LBO, B_LBO, 128);
#pragma unroll
          for (int part = 0; part < 2; ++part) {
            const uint64_t da = umma_desc((part ? al : ah) + ks * 2 * A_LBO, A_LBO, 128);
            const uint32_t acc = (ks > 0 || part > 0) ? 1u : 0u;
            asm volatile(
                "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem + d * NM),
                "l"(da), "l"(db), "r"(IDESC), "r"(acc));
          }
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
            smem_u32(&a_empty[st])));
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
            smem_u32(&acc_full[d])));
      }
  } else if (warp < 6) {  // converters: A_lo next to A_hi
    const int ct = tid - 64;
    for (int i = 0; i < nt; ++i) {
      const int st = i % S;
      mbar_wait(&a_full[st], (uint32_t)((i / S) & 1));
      uint8_t* ah = sA + st * 2 * kBkABytes;
#pragma unroll 4
      for (int j = ct; j < kBkABytes / 16; j += 128) {
        const float4 x = *reinterpret_cast<const float4*>(ah + j * 16);
        *reinterpret_cast<float4*>(ah + kBkABytes + j * 16) = sub4(x, tf32_hi(x));
      }
      asm volatile("fence.proxy.async.shared::cta;");
      __syncwarp();
      if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&a_conv[st])));
    }
  } else {  // epilogue: g_p = u + D_hi + D_lo -> swizzled staging -> tensor TMA store
    const int et = tid - 192, q = warp % 4, m = q * 32 + lane;
    for (int i = 0; i < nt; ++i) {
      const int d = i & 1, tile = blockIdx.x + i * gridDim.x;
      if (i > 0) {  // the previous tile's store has read the staging buffer
        if (et == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
        asm volatile("bar.sync 1, 128;" ::: "memory");
      }
      mbar_wait(&acc_full[d], (uint32_t)((i / 2) & 1));
      __syncwarp();
      asm volatile("tcgen05.fence::after_thread_sync;");
      const int k = tile * 128 + m;
      const float uk = k < N ? __ldg(u + k) : 0.f;
#pragma unroll
      for (int c = 0; c < BC; c += 16) {
        uint32_t v[16], w[16];
        const uint32_t ta = tmem + ((uint32_t)(q * 32) << 16) + d * NM + c;
        asm volatile(
            "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
            : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
              "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]),
              "=r"(v[14]), "=r"(v[15])
            : "r"(ta));
        asm volatile(
            "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
            : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]),
              "=r"(w[7]), "=r"(w[8]), "=r"(w[9]), "=r"(w[10]), "=r"(w[11]), "=r"(w[12]), "=r"(w[13]),
              "=r"(w[14]), "=r"(w[15])
            : "r"(ta + BC));
        asm volatile("tcgen05.wait::ld.sync.aligned;");
        uint8_t* rowp = stg + (c / 32) * (128 * 128) + m * 128;
#pragma unroll
        for (int x = 0; x < 16; x += 4) {
          const int j = ((c % 32) + x) / 4;  // 16-byte chunk within the 128-byte row
          *reinterpret_cast<float4*>(rowp + ((j ^ (m % 8)) * 16)) =
              make_float4(uk + (__uint_as_float(v[x]) + __uint_as_float(w[x])),
                          uk + (__uint_as_float(v[x + 1]) + __uint_as_float(w[x + 1])),
                          uk + (__uint_as_float(v[x + 2]) + __uint_as_float(w[x + 2])),
                          uk + (__uint_as_float(v[x + 3]) + __uint_as_float(w[x + 3])));
        }
      }
      asm volatile("tcgen05.fence::before_thread_sync;");
      __syncwarp();
      if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&acc_empty[d])));
      asm volatile("fence.proxy.async.shared::cta;");
      asm volatile("bar.sync 1, 128;" ::: "memory");
      if (et == 0) {
#pragma unroll
        for (int jb = 0; jb < BC / 32; ++jb)
          asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];" ::"l"(
                           &tm_gp),
                       "r"(seed0 + 32 * jb), "r"(tile * 128), "r"(smem_u32(stg + jb * 128 * 128))
                       : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
    }
    if (et == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) {
    __syncwarp();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(TMEM_COLS));
  }
}

// W1^T laid out for k_mlp_l1_back_tma, once per run: ceil(N / 128) tiles of
// kBkABytes, element (e-node m of the tile, hidden unit h) at core (h/4, m/8):
// ((h/4) * 16 + m/8) * 128 + (m%8) * 16 + (h%4) * 4 bytes (k_mlp_l1_back_tc's
// A layout); hidden units >= H1 and e-nodes >= N are zero.
std::vector<float> mlp_w1_back_tiles(const float* W1, int H1, int N) {
  const int ntiles = (N + 127) / 128;
  std::vector<float> t((size_t)ntiles * (kBkABytes / 4), 0.f);
  for (int tl = 0; tl < ntiles; ++tl) {
    float* tile = t.data() + (size_t)tl * (kBkABytes / 4);
    for (int h = 0; h < H1 && h < kMlpMaxH1; ++h)
      for (int m = 0; m < 128 && tl * 128 + m < N; ++m)
        tile[(((h / 4) * 16 + m / 8) * 128 + (m % 8) * 16 + (h % 4) * 4) / 4] =
            W1[(size_t)h * N + tl * 128 + m];
  }
  return t;
}

int mlp_nsplit(int device) { return num_sms(device); }

void launch_mlp_fwd(cudaStream_t s, const Shape& sh, int32_t H1, int32_t H2, const float* W1,
                    const float* W1t,
                    const float* b1, const float* W2, const float* b2, const float* W3,
                    const float* b3, const float* p, float* z1_part, float* z1, double* f_mlp,
                    float* gz1, int32_t nsplit) {
  const int Bc = sh.Bp < 128 ? sh.Bp : 128;
  const dim3 grid(nsplit, sh.Bp / Bc);
  const char* tenv = std::getenv("SMOOTHE_MLP_TMA");
  const bool tma = !(tenv && tenv[0] == '0') && W1t;
  if (tma) {
    const CUtensorMap tp = tensor_map_2d(p, false, (uint64_t)sh.Bp, (uint64_t)sh.N,
                                          (uint64_t)sh.Bp * 4, (uint32_t)Bc, kTmKB);
#define SM_L1T(BCV)                                                                             \
  do {                                                                                          \
    static bool attr = false;                                                                   \
    if (!attr) {                                                                                \
      SM_CUDA(cudaFuncSetAttribute(k_mlp_l1_tma<BCV>, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                                   tm_smem<BCV>()));                                            \
      attr = true;                                                                              \
    }                                                                                           \
    k_mlp_l1_tma<BCV><<<grid, kTmThreads, tm_smem<BCV>(), s>>>(W1t, tp, sh.N, sh.Bp, nsplit, z1_part); \
  } while (0)
    if (Bc == 128) SM_L1T(128);
    else if (Bc == 64) SM_L1T(64);
    else SM_L1T(32);
#undef SM_L1T
    SM_LAUNCH_CHECK();
  } else {
#define SM_L1(BCV)                                                                              \
  do {                                                                                          \
    constexpr int smem = tc_stages<BCV>() * (128 * kTcKB * 4 + kTcKB * 2 * BCV * 4) + 1024;     \
    static bool attr = false;                                                                   \
    if (!attr) {                                                                                \
      SM_CUDA(cudaFuncSetAttribute(k_mlp_l1_tc<BCV>, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                                   smem));                                                      \
      attr = true;                                                                              \
    }                                                                                           \
    k_mlp_l1_tc<BCV><<<grid, kTcThreads, smem, s>>>(sh.N, sh.Bp, H1, nsplit, W1, p, z1_part);   \
  } while (0)
  if (Bc == 128) SM_L1(128);
  else if (Bc == 64) SM_L1(64);
  else SM_L1(32);
#undef SM_L1
  SM_LAUNCH_CHECK();
  }
  SM_REQUIRE(nsplit <= kRedMaxSplit, SMOOTHE_E_CUDA, "k_mlp_reduce: more split-K partials than SMs expected");
  k_mlp_reduce<<<dim3(H1, sh.Bp / 32), 256, 0, s>>>(sh.Bp, H1, nsplit, b1, z1_part, z1);
  SM_LAUNCH_CHECK();
  k_mlp_head<<<(sh.Bp + 3) / 4, 128, 0, s>>>(sh.Bp, H1, H2, z1, W2, b2, W3, b3, f_mlp, gz1);
  SM_LAUNCH_CHECK();
}

void launch_mlp_bwd(cudaStream_t s, const Shape& sh, int32_t H1, const float* W1, const float* W1b,
                    const float* u, const float* gz1, float* gp, int32_t nsms) {
  const int Bc = sh.Bp < 128 ? sh.Bp : 128;
  const char* tenv = std::getenv("SMOOTHE_MLP_TMA");
  if (!(tenv && tenv[0] == '0') && W1b) {
    const int nchunks = sh.Bp / Bc, ntiles = (sh.N + 127) / 128;
    int gx = nsms / nchunks;
    gx = gx < 1 ? 1 : gx > ntiles ? ntiles : gx;
    const dim3 grid(gx, nchunks);
    const CUtensorMap tg = tensor_map_2d(gp, false, (uint64_t)sh.Bp, (uint64_t)sh.N,
                                          (uint64_t)sh.Bp * 4, 32, 128, true);
#define SM_L1BT(BCV)                                                                             \
  do {                                                                                           \
    static bool attr = false;                                                                    \
    if (!attr) {                                                                                 \
      SM_CUDA(cudaFuncSetAttribute(k_mlp_l1_back_tma<BCV>,                                       \
                                   cudaFuncAttributeMaxDynamicSharedMemorySize, bk_smem<BCV>()));\
      attr = true;                                                                               \
    }                                                                                            \
    k_mlp_l1_back_tma<BCV><<<grid, kBkThreads, bk_smem<BCV>(), s>>>(W1b, tg, sh.N, sh.Bp, H1, u, gz1); \
  } while (0)
    if (Bc == 128) SM_L1BT(128);
    else if (Bc == 64) SM_L1BT(64);
    else SM_L1BT(32);
#undef SM_L1BT
    SM_LAUNCH_CHECK();
    return;
  }
  const dim3 grid((sh.N + 127) / 128, sh.Bp / Bc);
#define SM_L1B(BCV)                                                                              \
  do {                                                                                           \
    constexpr int smem = 2 * 128 * kMlpMaxH1 * 4 + kMlpMaxH1 * 2 * BCV * 4 + 1024;               \
    static bool attr = false;                                                                    \
    if (!attr) {                                                                                 \
      SM_CUDA(cudaFuncSetAttribute(k_mlp_l1_back_tc<BCV>,                                        \
                                   cudaFuncAttributeMaxDynamicSharedMemorySize, smem));          \
      attr = true;                                                                               \
    }                                                                                            \
    k_mlp_l1_back_tc<BCV><<<grid, kTcThreads, smem, s>>>(sh.N, sh.Bp, H1, W1, u, gz1, gp);        \
  } while (0)
  if (Bc == 128) SM_L1B(128);
  else if (Bc == 64) SM_L1B(64);
  else SM_L1B(32);
#undef SM_L1B
  SM_LAUNCH_CHECK();
}

}  // namespace smoothe
