// NOTEARS acyclicity penalty per (penalty group, SCC) (sm_100a).
//
//   A_t[i][j] = sum_{k in m_i, m_j in ch_k} cp_k
//   h(A) = tr(e^A) - d, zero iff acyclic (Thm 3.1, Eqs. 8-9)
//   SCC decomposition: h = sum_S h(A_S)
//   batched approximation: exp of the seed-mean matrix (Eq. 11)  PAPER.md:320-325,
//     over groups of G seeds (reading S13)
//   gradient: dL/dcp_{k,b} += lambda * sum_{j in ch_k cap S} e^{Abar}[j][ec(k)]
//     (d tr e^A / dA = (e^A)^T)
//
// One CTA per (SCC, group).  Abar (|S| <= 64) lives in shared memory in fp64;
// e^A - I is formed directly (Horner form of the Taylor series of expm1 after
// scaling the inf-norm to <= 1/2, then Y <- Y^2 + 2Y per squaring), so
// h = tr(e^A - I) carries no cancellation.  The entry sums run over a fixed
// (entry, node, seed) order with a fixed warp-shuffle tree: h and the
// gradient are bit-identical at every GPU count.
#include <cstdlib>

#include "kcommon.cuh"

namespace smoothe {

constexpr int kNotearsMaxN = kSmallScc;
constexpr int kTaylorDeg = 16;

__device__ void smem_matmul(int n, const double* A, const double* B, double* C) {
  for (int idx = threadIdx.x; idx < n * n; idx += blockDim.x) {
    const int i = idx / n, j = idx % n;
    double acc = 0.0;
    for (int k = 0; k < n; ++k) acc += A[i * n + k] * B[k * n + j];
    C[idx] = acc;
  }
}

__global__ void __launch_bounds__(256) k_notears(
    int Bp, int G, int ngroups, double lambda, const int32_t* __restrict__ scc_class_ptr,
    const int32_t* __restrict__ ent_ptr, const int32_t* __restrict__ ent_i,
    const int32_t* __restrict__ ent_j, const int32_t* __restrict__ ent_node_ptr,
    const int32_t* __restrict__ ent_node, const int32_t* __restrict__ slot_ptr,
    const int32_t* __restrict__ slot_iloc, const int32_t* __restrict__ slot_jptr,
    const int32_t* __restrict__ slot_jloc, const float* __restrict__ cp,
    double* __restrict__ h_part, float* __restrict__ pen) {
  extern __shared__ double smem[];
  __shared__ int s_sq;
  const int scc = blockIdx.x, grp = blockIdx.y;
  const int n = scc_class_ptr[scc + 1] - scc_class_ptr[scc];
  if (n > kNotearsMaxN) return;  // large components: launch_notears_big
  double* X = smem;
  double* T = X + n * n;
  double* U = T + n * n;
  for (int idx = threadIdx.x; idx < n * n; idx += blockDim.x) X[idx] = 0.0;
  __syncthreads();
  // Abar_S[i][j] = (1/G) sum_{b in group} sum_{k in m_i, j in ch_k} cp_{k,b}
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nwarps = blockDim.x >> 5;
  const int b0 = grp * G;
  for (int e = ent_ptr[scc] + warp; e < ent_ptr[scc + 1]; e += nwarps) {
    double acc = 0.0;
    for (int a = ent_node_ptr[e]; a < ent_node_ptr[e + 1]; ++a) {
      const float* row = cp + (size_t)ent_node[a] * Bp + b0;
      for (int b = lane; b < G; b += 32) acc += (double)row[b];
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
    if (lane == 0) X[ent_i[e] * n + ent_j[e]] = acc / G;
  }
  __syncthreads();
  // scaling: 2^-s with s = max(0, ceil(log2 ||A||_inf) + 1)  =>  ||X|| <= 1/2
  if (threadIdx.x == 0) {
    double nrm = 0.0;
    for (int i = 0; i < n; ++i) {
      double r = 0.0;
      for (int j = 0; j < n; ++j) r += fabs(X[i * n + j]);
      nrm = fmax(nrm, r);
    }
    s_sq = nrm > 0.0 ? max(0, (int)ceil(log2(nrm)) + 1) : 0;
  }
  __syncthreads();
  const int sq = s_sq;
  const double scale = ldexp(1.0, -sq);
  for (int idx = threadIdx.x; idx < n * n; idx += blockDim.x) {
    X[idx] *= scale;
    const int i = idx / n, j = idx % n;
    T[idx] = (i == j ? 1.0 : 0.0) + X[idx] / kTaylorDeg;
  }
  __syncthreads();
  // Horner: T_m = I + X T_{m+1} / m, m = deg-1 .. 2;  Y = X T_2 = e^X - I
  for (int mdeg = kTaylorDeg - 1; mdeg >= 2; --mdeg) {
    smem_matmul(n, X, T, U);
    __syncthreads();
    for (int idx = threadIdx.x; idx < n * n; idx += blockDim.x) {
      const int i = idx / n, j = idx % n;
      T[idx] = (i == j ? 1.0 : 0.0) + U[idx] / mdeg;
    }
    __syncthreads();
  }
  smem_matmul(n, X, T, U);  // U = Y
  __syncthreads();
  double* Y = U;
  double* Z = T;
  for (int r = 0; r < sq; ++r) {  // e^{2A} - I = Y^2 + 2Y
    smem_matmul(n, Y, Y, Z);
    __syncthreads();
    for (int idx = threadIdx.x; idx < n * n; idx += blockDim.x) Z[idx] += 2.0 * Y[idx];
    __syncthreads();
    double* tmp = Y;
    Y = Z;
    Z = tmp;
  }
  if (threadIdx.x == 0) {
    double tr = 0.0;
    for (int i = 0; i < n; ++i) tr += Y[i * n + i];
    h_part[(size_t)scc * ngroups + grp] = tr;
  }
  // penalty gradient per e-node slot of this SCC (same for every seed of the group)
  for (int l = slot_ptr[scc] + threadIdx.x; l < slot_ptr[scc + 1]; l += blockDim.x) {
    const int il = slot_iloc[l];
    double acc = 0.0;
    for (int q = slot_jptr[l]; q < slot_jptr[l + 1]; ++q) {
      const int jl = slot_jloc[q];
      acc += Y[jl * n + il] + (jl == il ? 1.0 : 0.0);
    }
    pen[(size_t)l * ngroups + grp] = (float)(lambda * acc);
  }
}

// ---------------------------------------------------------------------------
// Components larger than kNotearsMaxN classes: the same
// computation on dense fp64 matrices in global memory, one batch of penalty
// groups at a time (z = group), with the matrix products on a tiled fp64 GEMM.
// The scaling uses the loader's structural bound (HostGraph::big_scc_sq), so
// the launch sequence is fixed and the step stays capturable in a CUDA graph.
// fp64 because e^A - I is squared s times (relative errors double per
// squaring) and h must match an fp64 reference; tcgen05 has no fp64 kind,
// and the CUDA-core DFMA rate of B200 makes |S| in the thousands cost
// milliseconds.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_big_abar(
    int Bp, int G, int g0, int n, double scale, int e0, int e1,
    const int32_t* __restrict__ ent_i, const int32_t* __restrict__ ent_j,
    const int32_t* __restrict__ ent_node_ptr, const int32_t* __restrict__ ent_node,
    const float* __restrict__ cp, double* __restrict__ X) {
  const int lane = threadIdx.x & 31;
  const int e = e0 + blockIdx.x * 8 + (threadIdx.x >> 5);
  if (e >= e1) return;
  const int b0 = (g0 + blockIdx.y) * G;
  double acc = 0.0;
  for (int a = ent_node_ptr[e]; a < ent_node_ptr[e + 1]; ++a) {
    const float* row = cp + (size_t)ent_node[a] * Bp + b0;
    for (int b = lane; b < G; b += 32) acc += (double)row[b];
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
  if (lane == 0)
    X[(size_t)blockIdx.y * n * n + (size_t)ent_i[e] * n + ent_j[e]] = acc / G * scale;
}

// T = I + c X, elementwise over the batch
__global__ void k_big_ipx(int n, size_t total, double c, const double* __restrict__ X,
                          double* __restrict__ T) {
  const size_t nn = (size_t)n * n;
  for (size_t idx = blockIdx.x * (size_t)blockDim.x + threadIdx.x; idx < total;
       idx += (size_t)gridDim.x * blockDim.x) {
    const size_t r = idx % nn;
    T[idx] = c * X[idx] + ((r / n) == (r % n) ? 1.0 : 0.0);
  }
}

// C = alpha A B + beta D + gamma I per batch entry z (row-major n x n, stride n^2).
// 64 x 64 tile per block, k-slabs of 16 in shared memory, 4 x 4 outputs per
// thread at stride 16 (conflict-free shared reads: a warp reads 2 A values
// (broadcast) and 16 consecutive B values).
constexpr int kGT = 64, kGK = 16;
__global__ void __launch_bounds__(256) k_big_gemm(int n, const double* __restrict__ A,
                                                  const double* __restrict__ B,
                                                  double* __restrict__ C, double alpha,
                                                  double beta, const double* __restrict__ D,
                                                  double gamma) {
  __shared__ double As[kGK][kGT + 1];
  __shared__ double Bs[kGK][kGT];
  const size_t off = (size_t)blockIdx.z * n * n;
  A += off;
  B += off;
  C += off;
  if (D) D += off;
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  const int i0 = blockIdx.y * kGT, j0 = blockIdx.x * kGT;
  double acc[4][4] = {};
  for (int k0 = 0; k0 < n; k0 += kGK) {
#pragma unroll
    for (int t = 0; t < 4; ++t) {  // A tile 64 x 16 (stored k-major), B tile 16 x 64
      const int idx = threadIdx.x + 256 * t;
      const int ai = idx >> 4, ak = idx & 15;
      const int gi = i0 + ai, gk = k0 + ak;
      As[ak][ai] = (gi < n && gk < n) ? A[(size_t)gi * n + gk] : 0.0;
      const int bk = idx >> 6, bj = idx & 63;
      const int hk = k0 + bk, hj = j0 + bj;
      Bs[bk][bj] = (hk < n && hj < n) ? B[(size_t)hk * n + hj] : 0.0;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kGK; ++k) {
      double a[4], b[4];
#pragma unroll
      for (int r = 0; r < 4; ++r) a[r] = As[k][ty + 16 * r];
#pragma unroll
      for (int c = 0; c < 4; ++c) b[c] = Bs[k][tx + 16 * c];
#pragma unroll
      for (int r = 0; r < 4; ++r)
#pragma unroll
        for (int c = 0; c < 4; ++c) acc[r][c] = fma(a[r], b[c], acc[r][c]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int r = 0; r < 4; ++r)
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      const int i = i0 + ty + 16 * r, j = j0 + tx + 16 * c;
      if (i < n && j < n) {
        const size_t o = (size_t)i * n + j;
        double x = alpha * acc[r][c];
        if (D) x += beta * D[o];
        if (i == j) x += gamma;
        C[o] = x;
      }
    }
}

// h_part[scc][g] = tr(Y_g) and the penalty gradient per e-node slot of the
// component (fixed-order block reduction: deterministic)
__global__ void __launch_bounds__(256) k_big_finish(
    int n, int scc, int ngroups, int g0, double lambda, const double* __restrict__ Y,
    int l0, int l1, const int32_t* __restrict__ slot_iloc, const int32_t* __restrict__ slot_jptr,
    const int32_t* __restrict__ slot_jloc, double* __restrict__ h_part, float* __restrict__ pen) {
  __shared__ double red[256];
  const int grp = g0 + blockIdx.y;
  Y += (size_t)blockIdx.y * n * n;
  if (blockIdx.x == 0) {
    double tr = 0.0;
    for (int i = threadIdx.x; i < n; i += blockDim.x) tr += Y[(size_t)i * n + i];
    red[threadIdx.x] = tr;
    __syncthreads();
    for (int o = blockDim.x / 2; o > 0; o >>= 1) {
      if (threadIdx.x < o) red[threadIdx.x] += red[threadIdx.x + o];
      __syncthreads();
    }
    if (threadIdx.x == 0) h_part[(size_t)scc * ngroups + grp] = red[0];
  }
  for (int l = l0 + blockIdx.x * blockDim.x + threadIdx.x; l < l1; l += gridDim.x * blockDim.x) {
    const int il = slot_iloc[l];
    double acc = 0.0;
    for (int q = slot_jptr[l]; q < slot_jptr[l + 1]; ++q) {
      const int jl = slot_jloc[q];
      acc += Y[(size_t)jl * n + il] + (jl == il ? 1.0 : 0.0);
    }
    pen[(size_t)l * ngroups + grp] = (float)(lambda * acc);
  }
}

// ---------------------------------------------------------------------------
// The same chain on the 5th-generation tensor cores (the default; SURVEY.md
// NEXT-1): matrices in fp32, padded to np = 64 * ceil(n / 64) (zero padding:
// the identity only on the first n diagonal entries, so padded rows and
// columns stay 0 through every product), each product C = alpha A B + beta D
// + gamma I with A B in "3xTF32": x = hi + lo (hi = x with the low 13 mantissa
// bits cleared, lo = x - hi exactly), and one M=128 x N=128 x K=8 tcgen05
// kind::tf32 MMA on A = [A_hi; A_lo] (a 64-row tile twice) and B = [B_hi |
// B_lo] (a 64-column tile twice) accumulates all four products of the
// 64 x 64 output tile in TMEM: AB = D[0:64,0:64] + D[0:64,64:128] +
// (D[64:128,0:64] + D[64:128,64:128]), summed in that fixed order.
// Precision (scripts/notears_precision_study.py, profiles/r2/notears_precision.md):
// on the 217- to 1112-class test components h is within 4e-7 of fp64 and
// every entry of e^Abar within 1.4% of the parity bar.  SMOOTHE_BIG_FP64=1
// keeps the fp64 CUDA-core GEMMs above.
// ---------------------------------------------------------------------------
constexpr int kBtT = 64, kBtK = 32, kBtStages = 3, kBtThreads = 128;
constexpr int kBtA = 128 * kBtK * 4, kBtB = kBtK * 128 * 4, kBtStage = kBtA + kBtB;
constexpr int kBtSmem = kBtStages * kBtStage + 1024;

__global__ void __launch_bounds__(kBtThreads, 1) k_big_gemm_tc(int n, int np,
                                                              const float* __restrict__ A,
                                                              const float* __restrict__ B,
                                                              float* __restrict__ C, float alpha,
                                                              float beta,
                                                              const float* __restrict__ D,
                                                              float gamma) {
  constexpr int LBO = 16 * 128;  // K-chunk (4 elements) stride of both operands: 16 core rows
  // kind::tf32, D f32, A and B K-major, M = 128, N = 128
  constexpr uint32_t IDESC =
      (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(128 >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
  extern __shared__ __align__(1024) uint8_t bt_smem[];
  uint8_t* smem = smem_align1024(bt_smem);
  __shared__ uint64_t bar[kBtStages + 1];
  __shared__ uint32_t tmem_sh;
  const int tid = threadIdx.x, warp = tid / 32, lane = tid % 32;
  const size_t off = (size_t)blockIdx.z * np * np;
  A += off;
  B += off;
  C += off;
  if (D) D += off;
  const int i0 = blockIdx.y * kBtT, j0 = blockIdx.x * kBtT;
  const int nkb = np / kBtK;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(&tmem_sh)),
                 "n"(128));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    for (int i = 0; i <= kBtStages; ++i) mbar_init(&bar[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_sh;
  // two K slabs in flight in registers (buffers p, q for even / odd slabs),
  // the third stage multiplying
  float4 pa[4], pb[4], qa[4], qb[4];
  auto load = [&](int kb, float4 (&ra)[4], float4 (&rb)[4]) {
    const int k0 = kb * kBtK;
#pragma unroll
    for (int i = 0; i < 4; ++i) {  // A: 64 rows x 8 K-chunks of 4 (row-coalesced)
      const int idx = tid + i * kBtThreads, r = idx / 8, kc = idx % 8;
      ra[i] = __ldg(reinterpret_cast<const float4*>(A + (size_t)(i0 + r) * np + k0 + 4 * kc));
    }
    const int kc = tid / 16, c = (tid % 16) * 4;  // B: the 4 x 4 block (K-chunk kc, columns c..c+3)
#pragma unroll
    for (int r = 0; r < 4; ++r)
      rb[r] = __ldg(reinterpret_cast<const float4*>(B + (size_t)(k0 + 4 * kc + r) * np + j0 + c));
  };
  auto store = [&](int st, const float4 (&ra)[4], const float4 (&rb)[4]) {
    uint8_t* sa = smem + st * kBtStage;
    uint8_t* sb = sa + kBtA;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int idx = tid + i * kBtThreads, r = idx / 8, kc = idx % 8;
      const float4 hi = tf32_hi(ra[i]), lo = sub4(ra[i], hi);
      // element (row, k): core (k/4, row/8) at (kc * 16 + row/8) * 128 + (row%8) * 16
      *reinterpret_cast<float4*>(sa + (kc * 16 + r / 8) * 128 + (r % 8) * 16) = hi;
      *reinterpret_cast<float4*>(sa + (kc * 16 + 8 + r / 8) * 128 + (r % 8) * 16) = lo;
    }
    // (bank-conflict-free store orders for A and B measured slower: they cost
    // the loads' coalescing or extra selects, and shared stores are not the limit)
    const int kc = tid / 16, c = (tid % 16) * 4;
#pragma unroll
    for (int x = 0; x < 4; ++x) {  // column c + x: its 4 K values, transposed to K-major
      const float4 col = make_float4(comp(rb[0], x), comp(rb[1], x), comp(rb[2], x), comp(rb[3], x));
      const float4 hi = tf32_hi(col), lo = sub4(col, hi);
      const int m = c + x;
      *reinterpret_cast<float4*>(sb + (kc * 16 + m / 8) * 128 + (m % 8) * 16) = hi;
      *reinterpret_cast<float4*>(sb + (kc * 16 + (64 + m) / 8) * 128 + (m % 8) * 16) = lo;
    }
  };
  auto step = [&](int kb, float4 (&ra)[4], float4 (&rb)[4]) {
    const int st = kb % kBtStages;
    if (kb >= kBtStages) mbar_wait(&bar[st], (uint32_t)((kb / kBtStages - 1) & 1));
    store(st, ra, rb);
    if (kb + 2 < nkb) load(kb + 2, ra, rb);
    asm volatile("fence.proxy.async.shared::cta;");
    __syncthreads();
    if (tid == 0) {
      asm volatile("tcgen05.fence::after_thread_sync;");
      const uint32_t sa = smem_u32(smem + st * kBtStage), sb = sa + kBtA;
#pragma unroll
      for (int ks = 0; ks < kBtK / 8; ++ks) {
        const uint64_t da = umma_desc(sa + ks * 2 * LBO, LBO, 128);
        const uint64_t db = umma_desc(sb + ks * 2 * LBO, LBO, 128);
        const uint32_t acc = (kb > 0 || ks > 0) ? 1u : 0u;
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
            "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
            "l"(da), "l"(db), "r"(IDESC), "r"(acc));
      }
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
          smem_u32(&bar[st])));
    }
  };
  load(0, pa, pb);
  if (nkb > 1) load(1, qa, qb);
  for (int kb = 0; kb < nkb; kb += 2) {  // np / 32 is even (np is a multiple of 64)
    step(kb, pa, pb);
    step(kb + 1, qa, qb);
  }
  if (tid == 0)
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
        smem_u32(&bar[kBtStages])));
  mbar_wait(&bar[kBtStages], 0);
  __syncwarp();  // lanes leave the wait loop separately: converge before .sync.aligned tcgen05 ops
  asm volatile("tcgen05.fence::after_thread_sync;");
  // warp w holds D rows 32w..32w+31: warps 2, 3 (the A_lo rows) hand their
  // (lo*hi + lo*lo) to warps 0, 1 through shared memory (the stages are idle)
  float* xch = reinterpret_cast<float*>(smem);  // [64][64 + 1]
  auto ld16 = [&](uint32_t col, float* out) {
    uint32_t v[16];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
          "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]),
          "=r"(v[14]), "=r"(v[15])
        : "r"(tmem + ((uint32_t)(warp * 32) << 16) + col));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
#pragma unroll
    for (int x = 0; x < 16; ++x) out[x] = __uint_as_float(v[x]);
  };
  const int row = (warp & 1) * 32 + lane;  // output row within the tile
  if (warp >= 2) {
    for (int c = 0; c < 64; c += 16) {
      float a[16], b[16];
      ld16(c, a);
      ld16(64 + c, b);
#pragma unroll
      for (int x = 0; x < 16; ++x) xch[row * 65 + c + x] = a[x] + b[x];
    }
  }
  __syncthreads();
  if (warp < 2) {
    const int i = i0 + row;
    for (int c = 0; c < 64; c += 16) {
      float a[16], b[16];
      ld16(c, a);
      ld16(64 + c, b);
#pragma unroll
      for (int x = 0; x < 16; ++x) {
        const int j = j0 + c + x;
        const size_t o = (size_t)i * np + j;
        float v = alpha * ((a[x] + b[x]) + xch[row * 65 + c + x]);
        if (D) v += beta * D[o];
        if (i == j && i < n) v += gamma;
        C[o] = v;
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) {
    __syncwarp();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(128));
  }
}

__global__ void __launch_bounds__(256) k_big_abar_f(
    int Bp, int G, int g0, int np, float scale, int e0, int e1, const int32_t* __restrict__ ent_i,
    const int32_t* __restrict__ ent_j, const int32_t* __restrict__ ent_node_ptr,
    const int32_t* __restrict__ ent_node, const float* __restrict__ cp, float* __restrict__ X) {
  const int lane = threadIdx.x & 31;
  const int e = e0 + blockIdx.x * 8 + (threadIdx.x >> 5);
  if (e >= e1) return;
  const int b0 = (g0 + blockIdx.y) * G;
  double acc = 0.0;
  for (int a = ent_node_ptr[e]; a < ent_node_ptr[e + 1]; ++a) {
    const float* row = cp + (size_t)ent_node[a] * Bp + b0;
    for (int b = lane; b < G; b += 32) acc += (double)row[b];
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
  if (lane == 0)
    X[(size_t)blockIdx.y * np * np + (size_t)ent_i[e] * np + ent_j[e]] = (float)(acc / G * scale);
}

// T = I_n + c X over the batch (identity on the first n diagonal entries)
__global__ void k_big_ipx_f(int n, int np, size_t total, float c, const float* __restrict__ X,
                            float* __restrict__ T) {
  const size_t nn = (size_t)np * np;
  for (size_t idx = blockIdx.x * (size_t)blockDim.x + threadIdx.x; idx < total;
       idx += (size_t)gridDim.x * blockDim.x) {
    const size_t r = idx % nn, i = r / np;
    T[idx] = c * X[idx] + (i == r % np && (int)i < n ? 1.f : 0.f);
  }
}

__global__ void __launch_bounds__(256) k_big_finish_f(
    int n, int np, int scc, int ngroups, int g0, double lambda, const float* __restrict__ Y,
    int l0, int l1, const int32_t* __restrict__ slot_iloc, const int32_t* __restrict__ slot_jptr,
    const int32_t* __restrict__ slot_jloc, double* __restrict__ h_part, float* __restrict__ pen) {
  __shared__ double red[256];
  const int grp = g0 + blockIdx.y;
  Y += (size_t)blockIdx.y * np * np;
  if (blockIdx.x == 0) {
    double tr = 0.0;
    for (int i = threadIdx.x; i < n; i += blockDim.x) tr += (double)Y[(size_t)i * np + i];
    red[threadIdx.x] = tr;
    __syncthreads();
    for (int o = blockDim.x / 2; o > 0; o >>= 1) {
      if (threadIdx.x < o) red[threadIdx.x] += red[threadIdx.x + o];
      __syncthreads();
    }
    if (threadIdx.x == 0) h_part[(size_t)scc * ngroups + grp] = red[0];
  }
  for (int l = l0 + blockIdx.x * blockDim.x + threadIdx.x; l < l1; l += gridDim.x * blockDim.x) {
    const int il = slot_iloc[l];
    double acc = 0.0;
    for (int q = slot_jptr[l]; q < slot_jptr[l + 1]; ++q) {
      const int jl = slot_jloc[q];
      acc += (double)Y[(size_t)jl * np + il] + (jl == il ? 1.0 : 0.0);
    }
    pen[(size_t)l * ngroups + grp] = (float)(lambda * acc);
  }
}

static bool big_fp64() {
  const char* e = std::getenv("SMOOTHE_BIG_FP64");
  return e && e[0] == '1';
}

static void launch_notears_big_tc(cudaStream_t s, const Shape& sh, const HostGraph& hg,
                                  const DevGraph& g, int32_t G, double lambda, const float* cp,
                                  double* h_part, float* pen, double* scratch_d, int gpb) {
  const int ngroups = sh.B / G;
  static bool attr = false;
  if (!attr) {
    SM_CUDA(cudaFuncSetAttribute(k_big_gemm_tc, cudaFuncAttributeMaxDynamicSharedMemorySize, kBtSmem));
    attr = true;
  }
  float* scratch = reinterpret_cast<float*>(scratch_d);
  for (size_t t = 0; t < hg.big_scc.size(); ++t) {
    const int scc = hg.big_scc[t], sq = hg.big_scc_sq[t];
    const int n = hg.scc_class_ptr[scc + 1] - hg.scc_class_ptr[scc];
    const int np = (n + kBtT - 1) / kBtT * kBtT;
    const size_t nn = (size_t)np * np;
    const int e0 = hg.ent_ptr[scc], e1 = hg.ent_ptr[scc + 1];
    const int l0 = hg.slot_ptr[scc], l1 = hg.slot_ptr[scc + 1];
    for (int g0 = 0; g0 < ngroups; g0 += gpb) {
      const int gc = std::min(gpb, ngroups - g0);
      float* X = scratch;
      float* T = X + nn * gc;
      float* U = T + nn * gc;
      const dim3 gz(np / kBtT, np / kBtT, gc);
      SM_CUDA(cudaMemsetAsync(X, 0, sizeof(float) * nn * gc, s));
      if (e1 > e0) {
        k_big_abar_f<<<dim3((e1 - e0 + 7) / 8, gc), 256, 0, s>>>(
            sh.Bp, G, g0, np, (float)ldexp(1.0, -sq), e0, e1, g.ent_i, g.ent_j, g.ent_node_ptr,
            g.ent_node, cp, X);
        SM_LAUNCH_CHECK();
      }
      const int eg = (int)std::min<size_t>((nn * gc + 255) / 256, 148 * 8);
      k_big_ipx_f<<<eg, 256, 0, s>>>(n, np, nn * gc, 1.f / kTaylorDeg, X, T);
      SM_LAUNCH_CHECK();
      for (int mdeg = kTaylorDeg - 1; mdeg >= 2; --mdeg) {  // T_m = I + X T_{m+1} / m
        k_big_gemm_tc<<<gz, kBtThreads, kBtSmem, s>>>(n, np, X, T, U, 1.f / mdeg, 0.f, nullptr, 1.f);
        SM_LAUNCH_CHECK();
        std::swap(T, U);
      }
      k_big_gemm_tc<<<gz, kBtThreads, kBtSmem, s>>>(n, np, X, T, U, 1.f, 0.f, nullptr, 0.f);
      SM_LAUNCH_CHECK();
      float* Y = U;
      float* Z = T;
      for (int r = 0; r < sq; ++r) {  // e^{2A} - I = Y^2 + 2Y
        k_big_gemm_tc<<<gz, kBtThreads, kBtSmem, s>>>(n, np, Y, Y, Z, 1.f, 2.f, Y, 0.f);
        SM_LAUNCH_CHECK();
        std::swap(Y, Z);
      }
      const int fb = std::max(1, std::min(148, (l1 - l0 + 255) / 256));
      k_big_finish_f<<<dim3(fb, gc), 256, 0, s>>>(n, np, scc, ngroups, g0, lambda, Y, l0, l1,
                                                  g.slot_iloc, g.slot_jptr, g.slot_jloc, h_part,
                                                  pen);
      SM_LAUNCH_CHECK();
    }
  }
}

size_t notears_big_scratch(const HostGraph& hg, int ngroups, int* groups_per_batch) {
  int nmax = 0;
  for (int s : hg.big_scc)
    nmax = std::max(nmax, hg.scc_class_ptr[s + 1] - hg.scc_class_ptr[s]);
  if (nmax == 0) {
    *groups_per_batch = 0;
    return 0;
  }
  // X, T, U per group: fp64 n x n (SMOOTHE_BIG_FP64) or fp32 padded to np
  const size_t np = (size_t)(nmax + kBtT - 1) / kBtT * kBtT;
  const size_t per = big_fp64() ? 3 * sizeof(double) * (size_t)nmax * nmax : 3 * sizeof(float) * np * np;
  const size_t budget = (size_t)4 << 30;
  *groups_per_batch = (int)std::max<size_t>(1, std::min<size_t>(ngroups, budget / per));
  return per * *groups_per_batch;
}

static void launch_notears_big(cudaStream_t s, const Shape& sh, const HostGraph& hg,
                               const DevGraph& g, int32_t G, double lambda, const float* cp,
                               double* h_part, float* pen, double* scratch, int gpb) {
  const int ngroups = sh.B / G;
  for (size_t t = 0; t < hg.big_scc.size(); ++t) {
    const int scc = hg.big_scc[t], sq = hg.big_scc_sq[t];
    const int n = hg.scc_class_ptr[scc + 1] - hg.scc_class_ptr[scc];
    const size_t nn = (size_t)n * n;
    const int e0 = hg.ent_ptr[scc], e1 = hg.ent_ptr[scc + 1];
    const int l0 = hg.slot_ptr[scc], l1 = hg.slot_ptr[scc + 1];
    const dim3 gg((n + kGT - 1) / kGT, (n + kGT - 1) / kGT, 1);
    for (int g0 = 0; g0 < ngroups; g0 += gpb) {
      const int gc = std::min(gpb, ngroups - g0);
      double* X = scratch;
      double* T = X + nn * gc;
      double* U = T + nn * gc;
      const dim3 gz(gg.x, gg.y, gc);
      SM_CUDA(cudaMemsetAsync(X, 0, sizeof(double) * nn * gc, s));
      if (e1 > e0) {
        k_big_abar<<<dim3((e1 - e0 + 7) / 8, gc), 256, 0, s>>>(
            sh.Bp, G, g0, n, ldexp(1.0, -sq), e0, e1, g.ent_i, g.ent_j, g.ent_node_ptr,
            g.ent_node, cp, X);
        SM_LAUNCH_CHECK();
      }
      const int eg = (int)std::min<size_t>((nn * gc + 255) / 256, 148 * 8);
      k_big_ipx<<<eg, 256, 0, s>>>(n, nn * gc, 1.0 / kTaylorDeg, X, T);
      SM_LAUNCH_CHECK();
      // Horner: T_m = I + X T_{m+1} / m, m = deg-1 .. 2;  Y = X T_2 = e^X - I
      for (int mdeg = kTaylorDeg - 1; mdeg >= 2; --mdeg) {
        k_big_gemm<<<gz, 256, 0, s>>>(n, X, T, U, 1.0 / mdeg, 0.0, nullptr, 1.0);
        SM_LAUNCH_CHECK();
        std::swap(T, U);
      }
      k_big_gemm<<<gz, 256, 0, s>>>(n, X, T, U, 1.0, 0.0, nullptr, 0.0);
      SM_LAUNCH_CHECK();
      double* Y = U;
      double* Z = T;
      for (int r = 0; r < sq; ++r) {  // e^{2A} - I = Y^2 + 2Y
        k_big_gemm<<<gz, 256, 0, s>>>(n, Y, Y, Z, 1.0, 2.0, Y, 0.0);
        SM_LAUNCH_CHECK();
        std::swap(Y, Z);
      }
      const int fb = std::max(1, std::min(148, (l1 - l0 + 255) / 256));
      k_big_finish<<<dim3(fb, gc), 256, 0, s>>>(n, scc, ngroups, g0, lambda, Y, l0, l1,
                                                g.slot_iloc, g.slot_jptr, g.slot_jloc, h_part,
                                                pen);
      SM_LAUNCH_CHECK();
    }
  }
}

void launch_notears(cudaStream_t s, const Shape& sh, const HostGraph& hg, const DevGraph& g,
                    int32_t G, double lambda, const float* cp, double* h_part, float* pen,
                    double* big_scratch, int big_groups_per_batch) {
  if (hg.num_scc == 0) return;
  const int ngroups = sh.B / G;
  if (hg.num_scc > (int)hg.big_scc.size()) {
    const int n = std::min(hg.scc_max, kNotearsMaxN);
    const size_t smem = 3 * sizeof(double) * (size_t)n * n;
    static bool attr_set = false;
    if (!attr_set) {
      SM_CUDA(cudaFuncSetAttribute(k_notears, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   3 * sizeof(double) * kNotearsMaxN * kNotearsMaxN));
      attr_set = true;
    }
    k_notears<<<dim3(hg.num_scc, ngroups), 256, smem, s>>>(
        sh.Bp, G, ngroups, lambda, g.scc_class_ptr, g.ent_ptr, g.ent_i, g.ent_j, g.ent_node_ptr,
        g.ent_node, g.slot_ptr, g.slot_iloc, g.slot_jptr, g.slot_jloc, cp, h_part, pen);
    SM_LAUNCH_CHECK();
  }
  if (!hg.big_scc.empty()) {
    if (big_fp64())
      launch_notears_big(s, sh, hg, g, G, lambda, cp, h_part, pen, big_scratch,
                         big_groups_per_batch);
    else
      launch_notears_big_tc(s, sh, hg, g, G, lambda, cp, h_part, pen, big_scratch,
                            big_groups_per_batch);
  }
}

}  // namespace smoothe
