// The two propagation sweeps of one SmoothE step (sm_100a): the forward
// Jacobi sweep of Eqs. 5-7 and its reverse mode.  Together they are ~90% of a
// step on deep graphs (2K launches per step), so their design is driven by
// measurement:
//
//  * seed-innermost rows: a row group of LPR lanes owns one class row of
//    4*LPR seeds (float4 per lane), so every parent / child gather is a
//    contiguous 512-byte access at 128 seeds;
//  * parent / child lists padded to multiples of 4 with inert entries, read as
//    aligned 16-byte index vectors one batch ahead, four row gathers per
//    array in flight per row group;
//  * 64-thread blocks, rows assigned round-robin across SMs (the concurrent
//    class "wavefront" shares parent / child rows through L2; contiguous
//    per-block ranges measured 1.3-1.8x slower);
//  * no division in the inner loops: the reverse sweep forms one reciprocal per
//    e-node (an IEEE divide per edge or per node cost ~30% of the sweep);
//  * deterministic: every output row has exactly one owner, no atomics.
#include <cuda.h>

#include <algorithm>
#include <cstdlib>
#include <mutex>
#include <vector>

#include "kcommon.cuh"

namespace smoothe {

constexpr int kSweepBlock = 64;
// 1 + tau of reading S7' (exact in fp32)
constexpr float kRouteTau1 = 1.0f + 1.0f / 1024.0f;

// ---------------------------------------------------------------------------
// Forward sweep t (readings S2-S4, S6-S8):
//   p^t_k = cp_k * q^{t-1}_{ec(k)}                                      (Eq. 5)
//   q^t_j = wI (1 - prod_{k in pa_j}(1 - p^t_k)) + wC max_{k in pa_j} p^t_k   (Eqs. 6b, 7)
// and, for the reverse sweep, pi = the product over the non-zero factors signed
// by the number of zero factors (+: none, -: exactly one, 0: two or more), and
// am = the route of the max (reading S7'): parents are
// scanned in ascending e-node id, the first is the champion, and a later one
// takes over iff its p exceeds the champion's by more than a factor 1 + tau
// (tau = 2^-10), so parents tied up to rounding route to the lowest id.  The
// max itself (the correlated term) is the exact fp32 max.  The independent
// term 1 - prod(1 - p) is accumulated as the union u <- u + p (1 - u), which
// keeps its relative accuracy when every p is small (1 - prod of factors
// rounded near 1 loses it: q ~ 1e-4 came out 5e-4 off in fp32); a zero factor
// (p = 1) gives exactly 1.  Products, the
// difference 1 - p and the max use explicit round-to-nearest intrinsics so the
// reverse sweep can recompute 1 - p_k bit for bit.
//
// Change propagation ("frozen classes"): q^t_j is a
// deterministic function of the rows q^{t-1}_c of its parent classes c, so
// if none of them changed in sweep t-1 (bitwise, any seed), q^t_j, pi^t_j and
// am^t_j equal their values of sweep t-1 bit for bit and the class is not
// recomputed.  A class whose q row changes marks its child classes dirty for
// the next sweep (stamp t+1 in dirty_next); sweep 1 computes the classes
// adjacent to the root (q^0 = e_root).  In fp32 the iterates of the whole
// graph freeze long before K (C4: by sweep ~60 of 207), so most sweeps
// compute almost nothing.  Results are identical to computing every class.
//
//   q_prev / q_cur   complete rows q^{t-1} / q^t (ping-pong; a class that
//                    changed in t-1 but is not recomputed copies its row)
//   P                the version pools (pooled version stacks):
//                    a recomputed class takes the next row of its seed
//                    chunk's pool for its q / pi / am rows and is listed for
//                    sweep t with its previous row (publish_version)
// ---------------------------------------------------------------------------
// Pooled versions: per seed chunk c (wc seeds) a pool of cap rows; rows
// [0, M) hold version 0 of every class (q^0 = e_root, pi = 1, am = the first
// parent).  The row group's leader takes the next row of its chunk's pool,
// every lane writes its seeds of the q / pi / am rows, and the leader lists
// (class, previous row, new row) for sweep t.  A full pool gives no row: the
// step is marked aborted (its update is skipped; the host grows the pool and
// repeats the step, smoothe_run_steps).
struct PoolArgs {
  float* q;
  float* pi;  // NULL for the correlated aggregator
  int32_t* am;
  int64_t cap;
  int wc, M, K;
  int32_t* pool_n;      // [nchunk] rows taken this step (may exceed cap: overflow)
  int32_t* lastrow;     // [nchunk][M]
  int4* list;           // [nchunk][K+1][M]
  int32_t* list_n;      // [nchunk][K+2]
  int32_t* abort_flag;  // [0]: this step overflowed
  int32_t* fchg;        // [K+2] or NULL: fchg[t] = 1 once some q row changed in sweep t
};
template <int LPR>
__device__ __forceinline__ void publish_version(const PoolArgs& P, int t, int j, int gl,
                                                unsigned gm, float4 qo, float4 po, int4 arg) {
  const int c = blockIdx.y;
  int r = 0;
  if (gl == 0) r = atomicAdd(P.pool_n + c, 1);
  r = __shfl_sync(gm, r, (int)(threadIdx.x % 32) / LPR * LPR);  // from the group's leader
  if (r >= P.cap) {
    if (gl == 0) P.abort_flag[0] = 1;
    return;
  }
  const size_t o = ((size_t)c * P.cap + r) * P.wc + gl * 4;
  stcs4(P.q + o, qo);
  if (P.pi) stcs4(P.pi + o, po);
  stcs4i(P.am + o, arg);
  if (gl == 0) {
    int32_t* lr = P.lastrow + (size_t)c * P.M + j;
    const int n = atomicAdd(P.list_n + (size_t)c * (P.K + 2) + t, 1);
    P.list[((size_t)c * (P.K + 1) + t) * P.M + n] = make_int4(j, *lr, r, 0);
    *lr = r;
  }
}
// read-only path for the gathers (as the former kernel-parameter version got)
__device__ __forceinline__ float4 ldg4(const float* p) { return __ldg(reinterpret_cast<const float4*>(p)); }
__device__ __forceinline__ int4 ldg4i(const int32_t* p) { return __ldg(reinterpret_cast<const int4*>(p)); }

#define SM_FWD_PARAMS                                                                        \
  int M, int Bp, int root, int t, int all, const int32_t* __restrict__ dmin,                   \
      const int32_t* __restrict__ dirty_cur, int32_t* __restrict__ dirty_next,                 \
      const int32_t* __restrict__ chg_prev, int32_t* __restrict__ chg_cur, PoolArgs P,          \
      const int32_t* __restrict__ cls_child_ptr, const int32_t* __restrict__ cls_child,        \
      const int32_t* __restrict__ pad_par_ptr, const int32_t* __restrict__ pad_par, float wI,  \
      float wC, const float* __restrict__ cp, const float* __restrict__ q_prev,                \
      float* __restrict__ q_cur
#define SM_FWD_ARGS                                                                            \
  M, Bp, root, t, all, dmin, dirty_cur, dirty_next, chg_prev, chg_cur, P, cls_child_ptr,       \
      cls_child, pad_par_ptr, pad_par, wI, wC, cp, q_prev, q_cur

// Recompute class j (its row group: LPR lanes, this lane's 4 seeds from s0).
template <int LPR>
__device__ __forceinline__ void forward_class(SM_FWD_PARAMS, int j, int gl, int s0, unsigned gm) {
  const size_t o = (size_t)j * Bp + s0;
  const float4 qold = ldg4(q_prev + o);
  // (node, class) pairs in batches of 4; padding pairs (N, root) read the zero
  // row N of cp, so p = 0: factor 1 and never a new max
  const int e0 = __ldg(pad_par_ptr + j), e1 = __ldg(pad_par_ptr + j + 1);
  float4 prod = make_float4(1.f, 1.f, 1.f, 1.f);
  float4 un = make_float4(0.f, 0.f, 0.f, 0.f);
  float4 mx = make_float4(-1.f, -1.f, -1.f, -1.f);
  float4 pc = mx;  // the routing champion's p (reading S7')
  int4 arg = make_int4(-1, -1, -1, -1);
  int4 zc = make_int4(0, 0, 0, 0);
  int4 n01 = make_int4(0, 0, 0, 0), n23 = n01;
  if (e0 < e1) {
    n01 = ldg4i(pad_par + 2 * (size_t)e0);
    n23 = ldg4i(pad_par + 2 * (size_t)e0 + 4);
  }
  for (int e = e0; e < e1; e += 4) {
    const int kk[4] = {n01.x, n01.z, n23.x, n23.z};
    const int cc[4] = {n01.y, n01.w, n23.y, n23.w};
    if (e + 4 < e1) {  // next batch's pairs, one step ahead
      n01 = ldg4i(pad_par + 2 * (size_t)e + 8);
      n23 = ldg4i(pad_par + 2 * (size_t)e + 12);
    }
    float4 cv[4], qv[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      cv[u] = ldg4(cp + (size_t)kk[u] * Bp + s0);
      qv[u] = ldg4(q_prev + (size_t)cc[u] * Bp + s0);
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
#pragma unroll
      for (int x = 0; x < 4; ++x) {
        const float p = __fmul_rn(comp(cv[u], x), comp(qv[u], x));
        const float f = __fsub_rn(1.f, p);
        comp(zc, x) += f == 0.f ? 1 : 0;
        comp(prod, x) = f == 0.f ? comp(prod, x) : __fmul_rn(comp(prod, x), f);
        comp(un, x) = __fmaf_rn(p, __fsub_rn(1.f, comp(un, x)), comp(un, x));
        comp(mx, x) = fmaxf(comp(mx, x), p);
        const bool gt = p > __fmul_rn(comp(pc, x), kRouteTau1);
        comp(pc, x) = gt ? p : comp(pc, x);
        comp(arg, x) = gt ? kk[u] : comp(arg, x);
      }
    }
  }
  float4 qo, po;
#pragma unroll
  for (int x = 0; x < 4; ++x) {
    const int z = comp(zc, x);
    const float U = z > 0 ? 1.f : comp(un, x);
    comp(qo, x) = __fadd_rn(__fmul_rn(wI, U), __fmul_rn(wC, fmaxf(comp(mx, x), 0.f)));
    comp(po, x) = z == 0 ? comp(prod, x) : (z == 1 ? -comp(prod, x) : 0.f);
  }
  st4(q_cur + o, qo);
  publish_version<LPR>(P, t, j, gl, gm, qo, po, arg);
  // bitwise change of the row (any seed of this chunk); chunks of a class write
  // the same stamps, so concurrent stores are benign
  const bool ne = __float_as_uint(qo.x) != __float_as_uint(qold.x) ||
                  __float_as_uint(qo.y) != __float_as_uint(qold.y) ||
                  __float_as_uint(qo.z) != __float_as_uint(qold.z) ||
                  __float_as_uint(qo.w) != __float_as_uint(qold.w);
  if (__ballot_sync(gm, ne) == 0u) return;
  if (gl == 0) {
    chg_cur[j] = t;
    if (P.fchg && __ldcg(P.fchg + t) == 0) {  // fchg[0]: the last sweep with a change
      __stcg(P.fchg + t, 1);
      atomicMax(P.fchg, t);
    }
  }
  for (int c = cls_child_ptr[j] + gl, ce = cls_child_ptr[j + 1]; c < ce; c += LPR)
    dirty_next[cls_child[c]] = t + 1;
}

// Persistent row groups over the classes in round-robin order (row group g of
// G takes classes g, g + G, ...: the classes in flight at any time are a
// window of consecutive ids, whose parent rows share L2).  Each row group
// reads the stamps of its next LPR classes at once (one per lane) and visits
// only those with work: recompute (dirty) or copy the q row (changed in the
// previous sweep, not dirty now).  A frozen sweep is thus a few loads per row
// group instead of one thread block per 2 classes.
#ifndef SMOOTHE_FWD_MINB
#define SMOOTHE_FWD_MINB 16  // min resident blocks per SM of the persistent forward (72 -> 64
                            // registers, small spills: C4 44.6 -> 43.5 ms per step; 14 / 18 / 20:
                            // 44.2 / 46.6 / 53.6)
#endif
template <int LPR>
__global__ void __launch_bounds__(kSweepBlock, SMOOTHE_FWD_MINB) k_sweep_forward(SM_FWD_PARAMS) {
  const int gl = threadIdx.x % LPR;
  const int G = gridDim.x * (kSweepBlock / LPR);
  const int g = blockIdx.x * (kSweepBlock / LPR) + (int)threadIdx.x / LPR;
  const int sh = (int)(threadIdx.x % 32) / LPR * LPR;
  const unsigned gm = LPR == 32 ? 0xffffffffu : ((1u << LPR) - 1u) << sh;
  const int s0 = blockIdx.y * (4 * LPR) + gl * 4;
  // the warp iterates together (row groups of LPR < 32 lanes share it): loop
  // bounds from the warp's first row group, and the union of the groups' work
  // bits, so the row groups of a warp run their classes side by side
  const int gw = g - sh / LPR;
  for (int64_t r0 = 0; r0 * G + gw < M; r0 += LPR) {
    const int64_t jl = (r0 + gl) * G + g;
    bool dirty = false, work = false;
    if (jl < M && jl != root) {
      dirty = all || (t == 1 ? __ldg(dmin + jl) == 1 : dirty_cur[jl] == t);
      work = dirty || chg_prev[jl] == t - 1;
    }
    const unsigned wall = __ballot_sync(0xffffffffu, work);
    const unsigned dall = __ballot_sync(0xffffffffu, dirty);
    const unsigned wb = wall >> sh, db = dall >> sh;  // this group's bits (low LPR)
    unsigned un = wall;
#pragma unroll
    for (int k = LPR; k < 32; k += LPR) un |= wall >> k;
    if (LPR < 32) un &= (1u << (LPR & 31)) - 1u;
    for (; un; un &= un - 1) {
      const int i = __ffs(un) - 1;
      if (!((wb >> i) & 1u)) continue;
      const int j = (int)((r0 + i) * G + g);
      if ((db >> i) & 1u) {
        forward_class<LPR>(SM_FWD_ARGS, j, gl, s0, gm);
      } else {  // q^t_j = q^{t-1}_j, which q_cur (written two sweeps ago) lacks
        const size_t o = (size_t)j * Bp + s0;
        st4(q_cur + o, ld4(q_prev + o));
      }
    }
  }
}

// One row group per class (graphs up to a few waves of resident blocks): the
// hardware block scheduler balances big classes.  The per-class code is the
// same as forward_class; kept as a kernel of its own because the inlined
// version schedules its loads worse (measured 15% slower on C5, same
// instruction and sector counts, more long-scoreboard stalls).
#ifndef SMOOTHE_FWDD_MINB
#define SMOOTHE_FWDD_MINB 1
#endif
template <int LPR>
__global__ void __launch_bounds__(kSweepBlock, SMOOTHE_FWDD_MINB) k_sweep_forward_direct(
    int M, int Bp, int root, int t, int all, const int32_t* __restrict__ dmin,
    const int32_t* __restrict__ dirty_cur, int32_t* __restrict__ dirty_next,
    const int32_t* __restrict__ chg_prev, int32_t* __restrict__ chg_cur, PoolArgs P,
    const int32_t* __restrict__ cls_child_ptr, const int32_t* __restrict__ cls_child,
    const int32_t* __restrict__ pad_par_ptr, const int32_t* __restrict__ pad_par, float wI,
    float wC, const float* __restrict__ cp, const float* __restrict__ q_prev,
    float* __restrict__ q_cur) {
  const int j = blockIdx.x * (kSweepBlock / LPR) + (int)threadIdx.x / LPR;
  if (j >= M) return;
  const int gl = threadIdx.x % LPR;
  const int s0 = blockIdx.y * (4 * LPR) + gl * 4;
  const size_t o = (size_t)j * Bp + s0;
  const bool dirty = j != root && (all || (t == 1 ? __ldg(dmin + j) == 1 : dirty_cur[j] == t));
  if (!dirty) {  // q^t_j = q^{t-1}_j; q_cur already holds it unless j changed in t-1
    if (chg_prev[j] == t - 1) st4(q_cur + o, ld4(q_prev + o));
    return;
  }
  const float4 qold = ld4(q_prev + o);
  // (node, class) pairs in batches of 4; padding pairs (N, root) read the zero
  // row N of cp, so p = 0: factor 1 and never a new max
  const int e0 = pad_par_ptr[j], e1 = pad_par_ptr[j + 1];
  float4 prod = make_float4(1.f, 1.f, 1.f, 1.f);
  float4 un = make_float4(0.f, 0.f, 0.f, 0.f);
  float4 mx = make_float4(-1.f, -1.f, -1.f, -1.f);
  float4 pc = mx;  // the routing champion's p (reading S7')
  int4 arg = make_int4(-1, -1, -1, -1);
  int4 zc = make_int4(0, 0, 0, 0);
  int4 n01 = make_int4(0, 0, 0, 0), n23 = n01;
  if (e0 < e1) {
    n01 = ld4i(pad_par + 2 * (size_t)e0);
    n23 = ld4i(pad_par + 2 * (size_t)e0 + 4);
  }
  for (int e = e0; e < e1; e += 4) {
    const int kk[4] = {n01.x, n01.z, n23.x, n23.z};
    const int cc[4] = {n01.y, n01.w, n23.y, n23.w};
    if (e + 4 < e1) {  // next batch's pairs, one step ahead
      n01 = ld4i(pad_par + 2 * (size_t)e + 8);
      n23 = ld4i(pad_par + 2 * (size_t)e + 12);
    }
    float4 cv[4], qv[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      cv[u] = ld4(cp + (size_t)kk[u] * Bp + s0);
      qv[u] = ld4(q_prev + (size_t)cc[u] * Bp + s0);
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
#pragma unroll
      for (int x = 0; x < 4; ++x) {
        const float p = __fmul_rn(comp(cv[u], x), comp(qv[u], x));
        const float f = __fsub_rn(1.f, p);
        comp(zc, x) += f == 0.f ? 1 : 0;
        comp(prod, x) = f == 0.f ? comp(prod, x) : __fmul_rn(comp(prod, x), f);
        comp(un, x) = __fmaf_rn(p, __fsub_rn(1.f, comp(un, x)), comp(un, x));
        comp(mx, x) = fmaxf(comp(mx, x), p);
        const bool gt = p > __fmul_rn(comp(pc, x), kRouteTau1);
        comp(pc, x) = gt ? p : comp(pc, x);
        comp(arg, x) = gt ? kk[u] : comp(arg, x);
      }
    }
  }
  float4 qo, po;
#pragma unroll
  for (int x = 0; x < 4; ++x) {
    const int z = comp(zc, x);
    const float U = z > 0 ? 1.f : comp(un, x);
    comp(qo, x) = __fadd_rn(__fmul_rn(wI, U), __fmul_rn(wC, fmaxf(comp(mx, x), 0.f)));
    comp(po, x) = z == 0 ? comp(prod, x) : (z == 1 ? -comp(prod, x) : 0.f);
  }
  st4(q_cur + o, qo);
  const unsigned gm = LPR == 32 ? 0xffffffffu : ((1u << LPR) - 1u) << ((threadIdx.x % 32) / LPR * LPR);
  publish_version<LPR>(P, t, j, gl, gm, qo, po, arg);
  // bitwise change of the row (any seed of this chunk); chunks of a class write
  // the same stamps, so concurrent stores are benign
  const bool ne = __float_as_uint(qo.x) != __float_as_uint(qold.x) ||
                  __float_as_uint(qo.y) != __float_as_uint(qold.y) ||
                  __float_as_uint(qo.z) != __float_as_uint(qold.z) ||
                  __float_as_uint(qo.w) != __float_as_uint(qold.w);
  if (__ballot_sync(gm, ne) == 0u) return;
  if (gl == 0) {
    chg_cur[j] = t;
    if (P.fchg && __ldcg(P.fchg + t) == 0) {  // fchg[0]: the last sweep with a change
      __stcg(P.fchg + t, 1);
      atomicMax(P.fchg, t);
    }
  }
  for (int c = cls_child_ptr[j] + gl, ce = cls_child_ptr[j + 1]; c < ce; c += LPR)
    dirty_next[cls_child[c]] = t + 1;
}

template <int LPR>
static int forward_grid(int device) {
  static int blocks[64] = {0};
  int& b = blocks[device & 63];
  if (!b) {
    SM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k_sweep_forward<LPR>, kSweepBlock, 0));
    // 4 waves of resident blocks: graphs up to that size keep one class per
    // row group (hardware block scheduling balances the big classes); larger
    // ones loop (C4: ~10 classes per row group)
    b = 4 * std::max(1, b) * num_sms(device);
  }
  return b;
}

static PoolArgs pool_args(const Shape& sh, const SweepState& st) {
  PoolArgs P;
  P.q = st.qpool;
  P.pi = st.pipool;
  P.am = st.apool;
  P.cap = st.cap;
  P.wc = st.wc;
  P.M = sh.M;
  P.K = st.K;
  P.pool_n = st.pool_n;
  P.lastrow = st.lastrow;
  P.list = st.list;
  P.list_n = st.list_n;
  P.abort_flag = st.abort_flag;
  P.fchg = st.fchg;
  return P;
}

void launch_sweep_forward(cudaStream_t s, const Shape& sh, const DevGraph& g, Agg a, int t,
                          const SweepState& st, const float* cp) {
  int dev = 0;
  SM_CUDA(cudaGetDevice(&dev));
  const PoolArgs P = pool_args(sh, st);
  SM_DISPATCH_LPR(sh.Bp, {
    const int rows_per_block = kSweepBlock / LPR;
    const int need = (sh.M + rows_per_block - 1) / rows_per_block;
    const int cap = forward_grid<LPR>(dev);
    const dim3 grid(need <= cap ? need : cap, num_chunks(sh.Bp));
    if (need <= cap)
      k_sweep_forward_direct<LPR><<<grid, kSweepBlock, 0, s>>>(
          sh.M, sh.Bp, sh.root, t, st.all ? 1 : 0, g.dmin, st.dirty[t & 1], st.dirty[(t + 1) & 1],
          st.chg[(t - 1) & 1], st.chg[t & 1], P, g.cls_child_ptr, g.cls_child, g.pad_par_ptr,
          g.pad_par, a.wI, a.wC, cp, st.qbuf[(t - 1) & 1], st.qbuf[t & 1]);
    else
      k_sweep_forward<LPR><<<grid, kSweepBlock, 0, s>>>(
          sh.M, sh.Bp, sh.root, t, st.all ? 1 : 0, g.dmin, st.dirty[t & 1], st.dirty[(t + 1) & 1],
          st.chg[(t - 1) & 1], st.chg[t & 1], P, g.cls_child_ptr, g.cls_child, g.pad_par_ptr,
          g.pad_par, a.wI, a.wC, cp, st.qbuf[(t - 1) & 1], st.qbuf[t & 1]);
  });
  SM_LAUNCH_CHECK();
}

// Before reverse sweep t: the reverse reads q^{t-1} (its own class) and
// pi^t / am^t (child classes) from complete rows cur_q / cur_pi / cur_am.
// Going from sweep t+1 to t, only the classes recomputed in forward sweep t+1
// (pi, am) or t (q) change version: copy their previous version's pool rows
// (the forward's lists, so the work is proportional to the recomputed
// classes).  t == K fills cur_pi / cur_am from every class's last row (cur_q
// is the forward's complete q^{K-1} buffer).  Grid y = seed chunk = pool.
// Dead gradients: the reverse sweeps are linear in g_q
// with no source term after the loss, so once every g_q^t row is zero, sweep t
// and all later ones add nothing.  live[t] (zeroed per step) is set by any
// writer that stores a non-zero g_q^t value; the kernels of reverse sweep t
// (transition, plain, frozen, combine) return at once when live_in = &live[t]
// is still 0.  (On C4 the gradient underflows to zero from sweep ~60 down.)
__device__ __forceinline__ bool g_dead(const int32_t* live_in) {
  return live_in && __ldcg(live_in) == 0;
}
// lane `leader` of the (sub)warp `mask` marks live_out when any lane's row is
// non-zero, and stamps the row (stamp = t - 1 for a g_q^{t-1} row, NULL: none)
// so that k_wspmv can skip the W rows of children whose g_q^t is all zero
__device__ __forceinline__ void g_mark(int32_t* live_out, unsigned mask, bool nz, bool leader,
                                       int32_t* stamp = nullptr, int tval = 0) {
  if (__any_sync(mask, nz) && leader) {
    if (live_out && __ldcg(live_out) == 0) __stcg(live_out, 1);
    if (stamp) __stcg(stamp, tval);
  }
}
template <int LPR>
__global__ void __launch_bounds__(kBlock) k_rev_restore_all(int M, int Bp, PoolArgs P,
                                                           float* __restrict__ cur_pi,
                                                           int32_t* __restrict__ cur_am) {
  const RowGroup<LPR> rg;
  const int j = rg.row;
  if (j >= M) return;
  const int c = blockIdx.y;
  const size_t o = (size_t)j * Bp + rg.s0;
  const size_t src = ((size_t)c * P.cap + P.lastrow[(size_t)c * M + j]) * P.wc + (rg.s0 - c * P.wc);
  if (cur_pi) st4(cur_pi + o, ld4(P.pi + src));
  st4i(cur_am + o, ld4i(P.am + src));
}

template <int LPR>
__global__ void __launch_bounds__(kBlock) k_rev_transition(int M, int Bp, int t, PoolArgs P,
                                                          float* __restrict__ cur_q,
                                                          float* __restrict__ cur_pi,
                                                          int32_t* __restrict__ cur_am,
                                                          int32_t* __restrict__ wm,
                                                          const int32_t* __restrict__ live_in) {
  if (g_dead(live_in)) return;  // reverse sweep t and all later ones add nothing
  const int groups = gridDim.x * (kBlock / LPR);
  const int c = blockIdx.y;
  const int32_t* ln = P.list_n + (size_t)c * (P.K + 2);
  const int4* l_pa = P.list + ((size_t)c * (P.K + 1) + t + 1) * M;  // recomputed in sweep t+1
  const int4* l_q = P.list + ((size_t)c * (P.K + 1) + t) * M;       // recomputed in sweep t
  const int n1 = ln[t + 1], n = n1 + ln[t];
  const int gl = threadIdx.x % LPR;
  const int s0 = c * (4 * LPR) + gl * 4;
  const size_t pbase = (size_t)c * P.cap;
  // seeds whose restored q row differs: a lane always covers seeds s0..s0+3,
  // so it keeps its own flags and the block clears wm once at the end (every
  // entry testing and storing the same 128 wm words serialised on them)
  __shared__ int changed[4 * LPR];
  if (wm && threadIdx.x < 4 * LPR) changed[threadIdx.x] = 0;
  bool chg[4] = {false, false, false, false};
  for (int i = blockIdx.x * (kBlock / LPR) + (int)threadIdx.x / LPR; i < n; i += groups) {
    if (i < n1) {
      const int4 e = l_pa[i];
      const size_t o = (size_t)e.x * Bp + s0, src = (pbase + e.y) * P.wc + gl * 4;
      if (cur_pi) st4(cur_pi + o, ld4(P.pi + src));
      st4i(cur_am + o, ld4i(P.am + src));
    } else {
      const int4 e = l_q[i - n1];
      const size_t o = (size_t)e.x * Bp + s0;
      const float4 prev = ld4(P.q + (pbase + e.y) * P.wc + gl * 4);
      if (wm) {  // a seed whose q row changed in forward sweep t leaves the K-state
        const float4 now = ld4(cur_q + o);
#pragma unroll
        for (int x = 0; x < 4; ++x)
          chg[x] = chg[x] || __float_as_uint(comp(prev, x)) != __float_as_uint(comp(now, x));
      }
      st4(cur_q + o, prev);
    }
  }
  if (!wm) return;
  __syncthreads();
#pragma unroll
  for (int x = 0; x < 4; ++x)
    if (chg[x]) changed[gl * 4 + x] = 1;  // benign same-value stores
  __syncthreads();
  if (threadIdx.x < 4 * LPR && changed[threadIdx.x] && __ldcg(wm + c * (4 * LPR) + threadIdx.x))
    __stcg(wm + c * (4 * LPR) + threadIdx.x, 0);
}

void launch_rev_transition(cudaStream_t s, const Shape& sh, const DevGraph& g, int t, int K,
                           const SweepState& st) {
  (void)g;
  const PoolArgs P = pool_args(sh, st);
  SM_DISPATCH_LPR(sh.Bp, {
    if (t == K) {
      k_rev_restore_all<LPR><<<row_grid(sh.M, sh.Bp, LPR), kBlock, 0, s>>>(sh.M, sh.Bp, P,
                                                                            st.cur_pi, st.cur_am);
    } else {
#ifndef SMOOTHE_TRANS_BPS
#define SMOOTHE_TRANS_BPS 8  // blocks per SM (2: 5.1 ms of transitions per C4 step, 8: 4.3, ncu)
#endif
      const dim3 grid(SMOOTHE_TRANS_BPS * st.num_sms, num_chunks(sh.Bp));
      k_rev_transition<LPR><<<grid, kBlock, 0, s>>>(sh.M, sh.Bp, t, P, st.qbuf[(K - 1) & 1],
                                                    st.cur_pi, st.cur_am,
                                                    st.wmode ? st.wm : nullptr,
                                                    st.glive ? st.glive + t : nullptr);
    }
  });
  SM_LAUNCH_CHECK();
}

// Version 0 of every class in rows [0, M) of each chunk's pool (a class never
// recomputed: every parent's q is 0): q = e_root, pi = +1 (every factor 1 - 0
// is non-zero), am = the first (lowest-id) parent, the forward kernel's tie
// rule; -1 for the root and parentless classes.
template <int LPR>
__global__ void __launch_bounds__(kBlock) k_pool_version0(int M, int root,
                                                          const int32_t* __restrict__ pad_par_ptr,
                                                          const int32_t* __restrict__ pad_par,
                                                          PoolArgs P) {
  const RowGroup<LPR> rg;
  const int j = rg.row;
  if (j >= M) return;
  const int c = blockIdx.y;
  const size_t o = ((size_t)c * P.cap + j) * P.wc + (rg.s0 - c * P.wc);
  const int e0 = pad_par_ptr[j];
  const int a = j != root && e0 < pad_par_ptr[j + 1] ? pad_par[2 * (size_t)e0] : -1;
  const float q0 = j == root ? 1.f : 0.f;
  st4(P.q + o, make_float4(q0, q0, q0, q0));
  if (P.pi) st4(P.pi + o, make_float4(1.f, 1.f, 1.f, 1.f));
  st4i(P.am + o, make_int4(a, a, a, a));
}

void launch_pool_version0(cudaStream_t s, const Shape& sh, const DevGraph& g, const SweepState& st) {
  const PoolArgs P = pool_args(sh, st);
  SM_DISPATCH_LPR(sh.Bp, {
    k_pool_version0<LPR><<<row_grid(sh.M, sh.Bp, LPR), kBlock, 0, s>>>(sh.M, sh.root, g.pad_par_ptr,
                                                                       g.pad_par, P);
  });
  SM_LAUNCH_CHECK();
}

// Per-step reset of the forward's state in one kernel (instead of a dozen
// memsets and a fill): stamps (dirty / chg, one allocation of 4 M) = -1, both
// q ping-pong rows = e_root (qbuf[1] follows qbuf[0] in one allocation), and
// per seed chunk: the pool's rows taken = M (version 0), every class's row =
// its version 0, list lengths 0; the step's abort flag 0.
__global__ void k_sweep_reset(int M, int Bp, int root, int nchunk, int K,
                              int32_t* __restrict__ stamps, float* __restrict__ qbuf,
                              int32_t* __restrict__ pool_n, int32_t* __restrict__ lastrow,
                              int32_t* __restrict__ list_n, int32_t* __restrict__ abort_flag,
                              int32_t* __restrict__ glive, int32_t* __restrict__ fchg) {
  const int64_t MB = (int64_t)M * Bp, n0 = 4 * (int64_t)M, n1 = n0 + 2 * MB,
                n2 = n1 + (int64_t)nchunk * M, n3 = n2 + (int64_t)nchunk * (K + 2);
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t e0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e0 == 0) abort_flag[0] = 0;
  if (glive && e0 < K + 2) glive[e0] = 0;
  if (fchg && e0 < K + 2) fchg[e0] = 0;
  if (e0 < nchunk) pool_n[e0] = M;
  for (int64_t e = e0; e < n3; e += stride) {
    if (e < n0) stamps[e] = -1;
    else if (e < n1) {
      const int64_t q = e - n0;
      qbuf[q] = (q % MB) / Bp == root ? 1.f : 0.f;
    } else if (e < n2) {
      lastrow[e - n1] = (int32_t)((e - n1) % M);
    } else {
      list_n[e - n2] = 0;
    }
  }
}

void launch_sweep_reset(cudaStream_t s, const Shape& sh, const SweepState& st) {
  // stamps: dirty[0], dirty[1], chg[0], chg[1] are consecutive (alloc_state)
  int dev = 0;
  SM_CUDA(cudaGetDevice(&dev));
  k_sweep_reset<<<4 * num_sms(dev), 256, 0, s>>>(sh.M, sh.Bp, sh.root, st.nchunk, st.K,
                                                 st.dirty[0], st.qbuf[0], st.pool_n, st.lastrow,
                                                 st.list_n, st.abort_flag, st.glive, st.fchg);
  SM_LAUNCH_CHECK();
}


// ---------------------------------------------------------------------------
// Reverse sweep t, one row group per class j'; for
// every e-node k in m_j' (contiguous), with p_k = cp_k q^{t-1}_{j'} recomputed
// bit-identically to the forward sweep and om = 1 - p_k:
//   g_p^t_k = sum_{j in ch_k} g_q^t_j (wI excl_{jk} + wC [k = a^t_j])
//   excl_{jk} = prod_{k' in pa_j, k' != k} (1 - p^t_k'):
//     pi_j > 0 (no zero factor):  pi_j / om   (k's own factor is the same fp32
//                                 value, so the quotient is exact to ~ulps)
//     pi_j < 0 (one zero factor): -pi_j if om = 0 (k's factor is that zero), else 0
//     pi_j = 0 (two or more):     0
//   so g_p = wI (A / om  or  T if om = 0) + wC R with A = sum_j g_j max(pi_j, 0),
//   T = sum_j g_j max(-pi_j, 0), R = sum_{j: a_j = k} g_j (carried in one
//   accumulator, see below);
//   g_cp_k += g_p^t_k q^{t-1}_{j'};   g_q^{t-1}_{j'} = sum_k g_p^t_k cp_k (0 at root).
// The class's padded child lists form one contiguous run of 4-wide batches;
// pad_batch_node gives each batch's e-node, so e-node boundaries are known one
// batch ahead (no dependent pointer chasing) and the next e-node's cp / g_cp
// rows are requested before the current one is finished.  Leaves own no batch
// (g_p = 0, nothing to update).
// ---------------------------------------------------------------------------
// V seeds per lane (V = 1, 2, 4: 32 lanes always own one class row slice of
// 32 V seeds, so no warp mixes classes; Bp > 128 uses V = 4 and Bp/128 slices).
template <int V>
struct Vec {
  float v[V];
};
template <int V>
struct IVec {
  int v[V];
};
template <int V>
__device__ __forceinline__ Vec<V> ldv(const float* p) {
  Vec<V> r;
  if (V == 4) *reinterpret_cast<float4*>(r.v) = *reinterpret_cast<const float4*>(p);
  else if (V == 2) *reinterpret_cast<float2*>(r.v) = *reinterpret_cast<const float2*>(p);
  else r.v[0] = *p;
  return r;
}
template <int V>
__device__ __forceinline__ Vec<V> ldv_cs(const float* p) {
  Vec<V> r;
  if (V == 4) *reinterpret_cast<float4*>(r.v) = __ldcs(reinterpret_cast<const float4*>(p));
  else if (V == 2) *reinterpret_cast<float2*>(r.v) = __ldcs(reinterpret_cast<const float2*>(p));
  else r.v[0] = __ldcs(p);
  return r;
}
template <int V>
__device__ __forceinline__ IVec<V> ldiv(const int32_t* p) {
  IVec<V> r;
  if (V == 4) *reinterpret_cast<int4*>(r.v) = *reinterpret_cast<const int4*>(p);
  else if (V == 2) *reinterpret_cast<int2*>(r.v) = *reinterpret_cast<const int2*>(p);
  else r.v[0] = *p;
  return r;
}
template <int V>
__device__ __forceinline__ void stv(float* p, const Vec<V>& x) {
  if (V == 4) *reinterpret_cast<float4*>(p) = *reinterpret_cast<const float4*>(x.v);
  else if (V == 2) *reinterpret_cast<float2*>(p) = *reinterpret_cast<const float2*>(x.v);
  else *p = x.v[0];
}
template <int V>
__device__ __forceinline__ void stv_cs(float* p, const Vec<V>& x) {
  if (V == 4) __stcs(reinterpret_cast<float4*>(p), *reinterpret_cast<const float4*>(x.v));
  else if (V == 2) __stcs(reinterpret_cast<float2*>(p), *reinterpret_cast<const float2*>(x.v));
  else __stcs(p, x.v[0]);
}

template <int V>
__device__ __forceinline__ Vec<V> ldv_cg(const float* p) {  // L2 only: rows other SMs wrote
  Vec<V> r;
  if (V == 4) *reinterpret_cast<float4*>(r.v) = __ldcg(reinterpret_cast<const float4*>(p));
  else if (V == 2) *reinterpret_cast<float2*>(r.v) = __ldcg(reinterpret_cast<const float2*>(p));
  else r.v[0] = __ldcg(p);
  return r;
}

template <int V>
__device__ __forceinline__ bool any_nz(const Vec<V>& v) {
  bool nz = false;
#pragma unroll
  for (int x = 0; x < V; ++x) nz = nz || v.v[x] != 0.f;
  return nz;
}

// Outputs of one reverse-sweep item: g_q^{t-1}_{j'} directly (the class's only
// item), else its partial row, and the class's last item to finish combines.
// CONV (convergence mode without the frozen-sweep path): seeds with pass = 1
// are past their convergence sweep; their g_q^{t-1}_{j'} is g_q^t_{j'}.
template <int V, bool CONV>
__device__ __forceinline__ Vec<V> pass_through(const Vec<V>& out, const Vec<V>& pass,
                                               const float* __restrict__ gq, int jp, int Bp,
                                               int s0) {
  if (!CONV) return out;
  bool any = false;
#pragma unroll
  for (int x = 0; x < V; ++x) any = any || pass.v[x] != 0.f;
  if (!__any_sync(0xffffffffu, any)) return out;
  const Vec<V> g = ldv_cg<V>(gq + (size_t)jp * Bp + s0);
  Vec<V> o = out;
#pragma unroll
  for (int x = 0; x < V; ++x)
    if (pass.v[x] != 0.f) o.v[x] = g.v[x];
  return o;
}

template <int V, bool HI, bool CONV>
__device__ __forceinline__ void reverse_epilogue(
    int lane, int jp, int info, bool piece, int Bp, int root, int s0, const Vec<V>& keep,
    const Vec<V>& qp,
    const Vec<V>& gqacc, const Vec<V>& X, const int4* __restrict__ items,
    const int32_t* __restrict__ class_item_ptr, const float* __restrict__ cp,
    float* __restrict__ gcp, float* __restrict__ gq_prev, float* __restrict__ part,
    int32_t* __restrict__ cnt, const Vec<V>& pass, const float* __restrict__ gq,
    int32_t* __restrict__ live_out, int32_t* __restrict__ gstamp, int t) {
  Vec<V> zero;
  int32_t* st = gstamp ? gstamp + (size_t)jp * gridDim.y + blockIdx.y : nullptr;  // [row][chunk]
#pragma unroll
  for (int x = 0; x < V; ++x) zero.v[x] = 0.f;
  if (info < 0) {  // the class's only item
    if (gq_prev) {
      const Vec<V> o = jp == root ? zero : pass_through<V, CONV>(gqacc, pass, gq, jp, Bp, s0);
      stv<V>(gq_prev + (size_t)jp * Bp + s0, o);
      g_mark(live_out, 0xffffffffu, any_nz<V>(o), lane == 0, st, t - 1);
    }
    return;
  }
  stv<V>(part + (size_t)(info >> 1) * Bp + s0, piece ? X : gqacc);
  __threadfence();
  __syncwarp();
  const int i0 = class_item_ptr[jp], i1 = class_item_ptr[jp + 1];
  int last = 0;
  int32_t* c = cnt + (size_t)jp * gridDim.y + blockIdx.y;  // one counter per seed slice
  if (lane == 0) last = atomicAdd(c, 1) == i1 - i0 - 1;
  if (!__shfl_sync(0xffffffffu, last, 0)) return;
  __threadfence();
  if (lane == 0) *c = 0;  // ready for the next launch
  Vec<V> acc = zero;
  for (int t = i0; t < i1;) {
    const int4 itm = items[2 * t];
    Vec<V> r = ldv_cg<V>(part + (size_t)(itm.w >> 1) * Bp + s0);
    if (!(itm.w & 1)) {
      ++t;
#pragma unroll
      for (int x = 0; x < V; ++x) acc.v[x] += r.v[x];
      continue;
    }
    const int k = items[2 * t + 1].x;  // pieces of e-node k: add up X, finalise
    for (++t; t < i1; ++t) {
      const int4 nx = items[2 * t];
      if (!(nx.w & 1) || items[2 * t + 1].x != k) break;
      const Vec<V> r2 = ldv_cg<V>(part + (size_t)(nx.w >> 1) * Bp + s0);
#pragma unroll
      for (int x = 0; x < V; ++x) r.v[x] += r2.v[x];
    }
    const size_t ok = (size_t)k * Bp + s0;
    const Vec<V> cv = ldv<V>(cp + ok);
    Vec<V> gc = ldv<V>(gcp + ok);
#pragma unroll
    for (int x = 0; x < V; ++x) {
      const float om = __fsub_rn(1.f, __fmul_rn(cv.v[x], qp.v[x]));
      const float gp = (HI && om != 0.f ? __fdividef(r.v[x], om) : r.v[x]) * keep.v[x];
      gc.v[x] += gp * qp.v[x];
      acc.v[x] += gp * cv.v[x];
    }
    stv<V>(gcp + ok, gc);
  }
  if (gq_prev) {
    const Vec<V> o = jp == root ? zero : pass_through<V, CONV>(acc, pass, gq, jp, Bp, s0);
    stv<V>(gq_prev + (size_t)jp * Bp + s0, o);
    g_mark(live_out, 0xffffffffu, any_nz<V>(o), lane == 0, st, t - 1);
  }
}

// One warp per work item (HostGraph::rev_item): a run of batches of class j'.
// Items holding whole e-nodes finalise them; a "piece" of a long e-node only
// accumulates its part of X.  A class with several items has each write one
// partial row (its g_q sum, or a piece's X); the last item to finish (a
// per-class counter) adds them in item order, finalises the pieced e-nodes and
// writes g_q^{t-1}_{j'} -- a fixed summation order, so the sweep stays
// deterministic.  The item header carries its first / last e-node, so the
// first rows are requested right after the header arrives.  (Persistent warps
// striding over items, with the next item staged by cp.async, measured 2.3x
// slower on C4: the in-flight window of classes spreads and L2 reuse drops.)
#ifndef SMOOTHE_REV_BLOCK
#define SMOOTHE_REV_BLOCK 64  // threads per block (one item per warp)
#endif
constexpr int kRevBlock = SMOOTHE_REV_BLOCK;
#ifndef SMOOTHE_REV_MINB4
#define SMOOTHE_REV_MINB4 (6 * 64 / SMOOTHE_REV_BLOCK)  // min resident blocks per SM at V = 4
#endif
template <int V, bool HI, bool HC, bool CONV, bool PERSIST = false>
__global__ void __launch_bounds__(kRevBlock, V == 4 ? SMOOTHE_REV_MINB4 : 8 * 64 / kRevBlock) k_sweep_reverse(
    int n_items, int Bp, int root, const int4* __restrict__ items,
    const int32_t* __restrict__ class_item_ptr, const int32_t* __restrict__ pad_child,
    const int32_t* __restrict__ pad_batch_node, float wI, float wC, const float* __restrict__ cp,
    const float* __restrict__ q_prev, const float* __restrict__ gq, const float* __restrict__ pi,
    const int32_t* __restrict__ am, float* __restrict__ gcp, float* __restrict__ gq_prev,
    float* __restrict__ part, int32_t* __restrict__ cnt, bool l2_prefetch, int t, int K,
    const int32_t* __restrict__ wm, const int32_t* __restrict__ lastchg,
    const int32_t* __restrict__ live_in, int32_t* __restrict__ live_out,
    int32_t* __restrict__ gstamp, int stride) {
  const int it0 = blockIdx.x * (kRevBlock / 32) + (int)threadIdx.x / 32;
  if (it0 >= n_items || g_dead(live_in)) return;
  const int lane = threadIdx.x % 32;
  // seeds in a frozen sweep (wm set) are the W kernel's: no contribution here
  Vec<V> keep, pass;
  bool allpass = false;
  if (CONV) {  // convergence mode: seeds past their convergence sweep pass g_q through
    const int sw = blockIdx.y * (32 * V) + lane * V;
    bool all = true;
#pragma unroll
    for (int x = 0; x < V; ++x) {
      const bool p = t > __ldg(lastchg + sw + x) + 1;
      pass.v[x] = p ? 1.f : 0.f;
      all = all && p;
    }
    allpass = __all_sync(0xffffffffu, all);
  } else {
#pragma unroll
    for (int x = 0; x < V; ++x) pass.v[x] = 0.f;
  }
  {
    const int sw = blockIdx.y * (32 * V) + lane * V;
    bool allw = true;
#pragma unroll
    for (int x = 0; x < V; ++x) {
      const bool w = wm && __ldg(wm + sw + x) != 0;
      keep.v[x] = w || pass.v[x] != 0.f ? 0.f : 1.f;
      allw = allw && w;
    }
    if (__all_sync(0xffffffffu, allw)) return;
  }
  // stride = n_items: one item per warp; else persistent warps (one wave of
  // blocks) take items it0, it0 + stride, ... (an all-frozen sweep then costs
  // one wave of blocks that exit at once instead of a block per two items)
  auto item = [&](const int it) {
  const int4 c0 = items[2 * it], c1 = items[2 * it + 1];
  if (c1.z > t - 1) return;  // q^{t-1}_{j'} = 0: nothing to add, g_q^{t-1}_{j'} never read
  const int jp = c0.x, bb = c0.y, be = c0.z, info = c0.w;
  const bool piece = info >= 0 && (info & 1);
  const int s0 = blockIdx.y * (32 * V) + lane * V;
  if (CONV && allpass) {  // the class's first item copies g_q^t_{j'} (root: 0)
    if (gq_prev && (info < 0 || it == class_item_ptr[jp])) {
      Vec<V> g = ldv_cg<V>(gq + (size_t)jp * Bp + s0);
      if (jp == root)
#pragma unroll
        for (int x = 0; x < V; ++x) g.v[x] = 0.f;
      stv<V>(gq_prev + (size_t)jp * Bp + s0, g);
      g_mark(live_out, 0xffffffffu, any_nz<V>(g), lane == 0,
             gstamp ? gstamp + (size_t)jp * gridDim.y + blockIdx.y : nullptr, t - 1);
    }
    return;
  }
  // Reverse window: the loss reads only q^K, so g_q^t_j is exactly 0 unless a
  // walk of length K - t leaves class j (t >= K - hmax_j); every child of j'
  // then has g_q^t = 0 while t <= K - hmax_j', and so has g_q^{t-1}_{j'}.  The
  // first two such sweeps write that zero row over the stale g_q^{t+1} /
  // g_q^{t+2} of the ping-pong buffer (parents may still be active).
  if ((int64_t)t + c1.w <= K) {
    if ((int64_t)t + c1.w >= K - 1 && gq_prev && (info < 0 || it == class_item_ptr[jp])) {
      Vec<V> z;
#pragma unroll
      for (int x = 0; x < V; ++x) z.v[x] = 0.f;
      stv<V>(gq_prev + (size_t)jp * Bp + s0, z);
    }
    return;
  }
  Vec<V> zero;
#pragma unroll
  for (int x = 0; x < V; ++x) zero.v[x] = 0.f;
  const Vec<V> qp = ldv<V>(q_prev + (size_t)jp * Bp + s0);
  Vec<V> gqacc = zero, X = zero;
  if (bb < be) {
    int k = c1.x;
    if (l2_prefetch) {
      // The item's e-nodes are consecutive ids; their cp / g_cp rows stream
      // from HBM once per sweep (no reuse): pull them into L2 now.
      const int nn = c1.y - k + 1;
      const int lines = 2 * nn * V;  // 128-byte lines: V per row
      for (int l = lane; l < lines; l += 32) {
        const int arr = l / (nn * V), r = l % (nn * V);
        const float* base = arr ? gcp : cp;
        const float* a = base + (size_t)(k + r / V) * Bp + blockIdx.y * (32 * V) + (r % V) * 32;
        asm volatile("prefetch.global.L2 [%0];" ::"l"(a));
      }
    }
    size_t ok = (size_t)k * Bp + s0;
    Vec<V> cv = ldv_cs<V>(cp + ok), gc = piece ? zero : ldv_cs<V>(gcp + ok);
    Vec<V> cvn = zero, gcn = zero;  // next e-node's cp / g_cp rows, requested one batch early
    // om = 1 - p_k, known at the e-node's start, lets one accumulator carry all
    // three terms: X = sum_j g_j (wI max(s pi_j, 0) + [a_j = k] wC r) with
    // (s, r) = (+1, om) if om != 0 (then g_p = X / om) and (-1, 1) if om = 0
    // (then g_p = X).  Per e-node constants: sI = s wI, cC = wC r, and
    // rom = 1 / om (approximate reciprocal, one MUFU per e-node; om is 0 or at
    // least 2^-24, so flushing denormals is exact) or 1 when om = 0.
    Vec<V> rom, sI, cC;
    auto node_consts = [&]() {
#pragma unroll
      for (int x = 0; x < V; ++x) {
        const float om = __fsub_rn(1.f, __fmul_rn(cv.v[x], qp.v[x]));
        const bool nz = om != 0.f;
        float r;
        asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(om));
        rom.v[x] = (HI && nz ? r : 1.f) * keep.v[x];
        sI.v[x] = nz ? wI : -wI;
        cC.v[x] = HI && nz ? wC * om : wC;  // without HI, g_p = X (no division)
      }
    };
    node_consts();
    // Double-buffered rows: batch b+1's are requested before batch b is
    // consumed; indices two batches ahead.  (Unrolling by two to drop the
    // buffer copies measured 10-25% slower.)  Padding slots point at the
    // root, whose g_q row is 0: no mask.
    Vec<V> gA[4], PA[4], gB[4], PB[4];
    IVec<V> aA[4], aB[4];
    // byte offset of (row, this lane's seeds): one 32 x 32 -> 64-bit
    // multiply-add per slot (class ids are non-negative)
    const uint32_t rowb = (uint32_t)Bp * 4u;
    const uint64_t s0b = (uint64_t)s0 * 4u;
    auto fetch = [&](int4 j, Vec<V>* gg, Vec<V>* PP, IVec<V>* aa) {
      const uint32_t jj[4] = {(uint32_t)j.x, (uint32_t)j.y, (uint32_t)j.z, (uint32_t)j.w};
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const uint64_t ob = (uint64_t)jj[u] * rowb + s0b;
        gg[u] = ldv<V>(reinterpret_cast<const float*>(reinterpret_cast<const char*>(gq) + ob));
        if (HI) PP[u] = ldv<V>(reinterpret_cast<const float*>(reinterpret_cast<const char*>(pi) + ob));
        if (HC) aa[u] = ldiv<V>(reinterpret_cast<const int32_t*>(reinterpret_cast<const char*>(am) + ob));
      }
    };
    fetch(ld4i(pad_child + 4 * (size_t)bb), gA, PA, aA);
    int4 j4 = bb + 1 < be ? ld4i(pad_child + 4 * (size_t)(bb + 1)) : make_int4(root, root, root, root);
    int kn = bb + 1 < be ? pad_batch_node[bb + 1] : -1;
    for (int b = bb; b < be; ++b) {
      const int knext = kn;  // e-node of batch b+1 (-1: none)
      if (b + 1 < be) {
        fetch(j4, gB, PB, aB);
        if (b + 2 < be) j4 = ld4i(pad_child + 4 * (size_t)(b + 2));
        kn = b + 2 < be ? pad_batch_node[b + 2] : -1;
      }
      if (knext >= 0 && knext != k) {
        cvn = ldv_cs<V>(cp + (size_t)knext * Bp + s0);
        if (!piece) gcn = ldv_cs<V>(gcp + (size_t)knext * Bp + s0);
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
#pragma unroll
        for (int x = 0; x < V; ++x) {
          if (HI) X.v[x] = fmaf(gA[u].v[x], fmaxf(sI.v[x] * PA[u].v[x], 0.f), X.v[x]);
          if (HC && aA[u].v[x] == k) X.v[x] = fmaf(gA[u].v[x], cC.v[x], X.v[x]);
        }
      }
      if (knext != k && !piece) {  // finalise e-node k (a piece hands X to the combine)
#pragma unroll
        for (int x = 0; x < V; ++x) {
          const float gp = X.v[x] * rom.v[x];
          gc.v[x] += gp * qp.v[x];
          gqacc.v[x] += gp * cv.v[x];
        }
        stv_cs<V>(gcp + ok, gc);
        if (knext >= 0) {
          k = knext;
          ok = (size_t)k * Bp + s0;
          cv = cvn;
          gc = gcn;
          node_consts();
          X = zero;
        }
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        gA[u] = gB[u];
        if (HI) PA[u] = PB[u];
        if (HC) aA[u] = aB[u];
      }
    }
  }
  reverse_epilogue<V, HI, CONV>(lane, jp, info, piece, Bp, root, s0, keep, qp, gqacc, X, items,
                                class_item_ptr, cp, gcp, gq_prev, part, cnt, pass, gq, live_out,
                                gstamp, t);
  };
  if (PERSIST) {
    for (int it = it0; it < n_items; it += stride) item(it);
  } else {
    item(it0);
  }
}

// ---------------------------------------------------------------------------
// The reverse sweep with its child rows staged by the tensor-memory
// accelerator (128-seed slices, fixed K).  The per-lane
// double buffer of the register kernel above (three gathered 512-byte rows
// per child slot, 12 per batch of 4 slots) is what holds its occupancy to ~12
// warps per SM at 124 registers.  Here each batch's rows come from three
// TMA gather4 instructions (cp.async.bulk.tensor.2d ... tile::gather4: the 4
// child rows of the batch for one array, 2 KB, into shared memory), issued by
// one lane a batch ahead into a 2-stage ring per warp and completed on an
// mbarrier: in-flight rows cost no registers, so 16 warps per SM each keep a
// batch in flight.  Items are taken in order from a per-(sweep, seed slice)
// cursor, so the warps in flight work on a compact window of classes whose
// child rows share L2; the next item's first batch is requested while the
// current item finishes.  The arithmetic, the e-node bookkeeping and the
// epilogue are the register kernel's (same results bit for bit).
// ---------------------------------------------------------------------------
#ifndef SMOOTHE_RT_WARPS
#define SMOOTHE_RT_WARPS 8   // warps per CTA
#endif
#ifndef SMOOTHE_RT_STAGES
#define SMOOTHE_RT_STAGES 3  // ring stages per warp (batches in flight: stages - 1 ahead)
#endif
#ifndef SMOOTHE_RT_CTAS
#define SMOOTHE_RT_CTAS 1    // CTAs per SM
#endif
constexpr int kRtWarps = SMOOTHE_RT_WARPS, kRtStages = SMOOTHE_RT_STAGES;
constexpr int kRtRow = 512;                        // bytes of a 128-seed row
constexpr int kRtStage = 3 * 4 * kRtRow;           // g, pi, am rows of a batch
constexpr int kRtSmem = kRtWarps * (kRtStages * kRtStage + kRtStages * 8);

__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P;\n\tWAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
      "@!P bra WAIT_%=;\n\t}" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_gather4(uint32_t dst, const CUtensorMap* map, uint32_t bar, int x,
                                            int4 rows) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4, %5, %6, %7}], [%2];" ::"r"(dst),
      "l"(map), "r"(bar), "r"(x), "r"(rows.x), "r"(rows.y), "r"(rows.z), "r"(rows.w)
      : "memory");
}
__device__ __forceinline__ int4 shfl4(int4 v, int src) {
  return make_int4(__shfl_sync(0xffffffffu, v.x, src), __shfl_sync(0xffffffffu, v.y, src),
                   __shfl_sync(0xffffffffu, v.z, src), __shfl_sync(0xffffffffu, v.w, src));
}

// One warp walks items it = w, w + T, w + 2T, ... (T warps in the slice's
// grid).  Per item, lane l holds the child classes (pad_child) and e-node
// (pad_batch_node) of the item's batch l (an item has at most 32 batches),
// loaded with one coalesced request; the next item's header and index rows
// are requested while the current item runs.  Batches flow through a ring of
// kRtStages stages: batch n + kRtStages - 1 is requested before batch n is
// consumed, across item boundaries.
template <bool HI, bool HC>
__global__ void __launch_bounds__(32 * kRtWarps, SMOOTHE_RT_CTAS) k_sweep_reverse_tma(
    const __grid_constant__ CUtensorMap tm_g, const __grid_constant__ CUtensorMap tm_pi,
    const __grid_constant__ CUtensorMap tm_am, int n_items, int Bp, int root,
    const int4* __restrict__ items, const int32_t* __restrict__ class_item_ptr,
    const int32_t* __restrict__ pad_child, const int32_t* __restrict__ pad_batch_node, float wI,
    float wC, const float* __restrict__ cp, const float* __restrict__ q_prev,
    const float* __restrict__ gq, float* __restrict__ gcp, float* __restrict__ gq_prev,
    float* __restrict__ part, int32_t* __restrict__ cnt, bool l2_prefetch, int t, int K,
    const int32_t* __restrict__ wm, int32_t* __restrict__ cursor,
    const int32_t* __restrict__ live_in, int32_t* __restrict__ live_out,
    int32_t* __restrict__ gstamp) {
  constexpr int V = 4, S = kRtStages;
  (void)cursor;
  if (g_dead(live_in)) return;
  extern __shared__ __align__(128) unsigned char rt_smem[];
  const int lane = threadIdx.x % 32, wi = threadIdx.x / 32;
  unsigned char* ring = rt_smem + (size_t)wi * S * kRtStage;
  const uint32_t bar0 = smem_addr(rt_smem + (size_t)kRtWarps * S * kRtStage + wi * 8 * S);
  const int slice = blockIdx.y;
  const int s0 = slice * 128 + lane * V, x0 = slice * 128;
  const int T = gridDim.x * kRtWarps;
  // seeds in a frozen sweep (wm set) are the W kernel's: no contribution here
  Vec<V> keep, zero;
  {
    bool allw = true;
#pragma unroll
    for (int x = 0; x < V; ++x) {
      const bool w = wm && __ldg(wm + s0 + x) != 0;
      keep.v[x] = w ? 0.f : 1.f;
      zero.v[x] = 0.f;
      allw = allw && w;
    }
    if (__all_sync(0xffffffffu, allw)) return;
  }
  if (lane == 0) {
#pragma unroll
    for (int st = 0; st < S; ++st) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar0 + 8 * st));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncwarp();
  constexpr uint32_t kTx = (1 + (HI ? 1 : 0) + (HC ? 1 : 0)) * 4 * kRtRow;
  uint32_t nb = 0, nc = 0;  // batches requested / consumed by this warp
  // one lane requests a batch (child classes j4) into the next stage, whose
  // previous batch every lane has consumed (__syncwarp; the generic-proxy
  // reads ordered before the async-proxy writes by the proxy fence)
  auto issue = [&](int4 j4) {
    __syncwarp();
    if (lane == 0) {
      asm volatile("fence.proxy.async.shared::cta;");
      const uint32_t st = nb % S, bar = bar0 + 8 * st;
      const uint32_t dst = smem_addr(ring + (size_t)st * kRtStage);
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(kTx));
      tma_gather4(dst, &tm_g, bar, x0, j4);
      if (HI) tma_gather4(dst + 4 * kRtRow, &tm_pi, bar, x0, j4);
      if (HC) tma_gather4(dst + 8 * kRtRow, &tm_am, bar, x0, j4);
    }
    ++nb;
  };
  auto active = [&](int4 c0, int4 c1) {  // the register kernel's exits
    return !(c1.z > t - 1) && !((int64_t)t + c1.w <= K) && c0.y < c0.z;
  };
  // A queue of items whose batches are requested: the current item, and up
  // to kRtStages - 1 batches of the following items.  Item state: header,
  // the lane-distributed index rows, batches requested so far.
  struct Item {
    int it;
    int4 c0, c1;
    int4 jl;   // lane l: child classes of batch c0.y + l
    int kl;    // lane l: e-node of batch c0.y + l
    bool act;
  };
  auto load_item = [&](int it) {
    Item m;
    m.it = it;
    m.c0 = make_int4(0, 0, 0, 0);
    m.c1 = m.c0;
    m.jl = m.c0;
    m.kl = -1;
    m.act = false;
    if (it < n_items) {
      m.c0 = items[2 * it];
      m.c1 = items[2 * it + 1];
      m.act = active(m.c0, m.c1);
      if (m.act && m.c0.y + lane < m.c0.z) {
        m.jl = ld4i(pad_child + 4 * (size_t)(m.c0.y + lane));
        m.kl = pad_batch_node[m.c0.y + lane];
      }
    }
    return m;
  };
  // request batches of the item queue [cur, nxt] up to S - 1 ahead of consumption
  Item cur = load_item(blockIdx.x * kRtWarps + wi);
  Item nxt = load_item(cur.it + T);
  int cur_req = 0, nxt_req = 0;  // batches requested of cur / nxt
  auto top_up = [&]() {
    while ((int)(nb - nc) < S - 1) {
      if (cur.act && cur_req < cur.c0.z - cur.c0.y) {
        issue(shfl4(cur.jl, cur_req));
        ++cur_req;
      } else if (cur_req >= cur.c0.z - cur.c0.y || !cur.act) {
        if (nxt.act && nxt_req < nxt.c0.z - nxt.c0.y) {
          issue(shfl4(nxt.jl, nxt_req));
          ++nxt_req;
        } else {
          break;
        }
      } else {
        break;
      }
    }
  };
  while (cur.it < n_items) {
    const int4 c0 = cur.c0, c1 = cur.c1;
    const int jp = c0.x, bb = c0.y, be = c0.z, info = c0.w;
    if (c1.z > t - 1) {  // q^{t-1}_{j'} = 0: nothing to add, g_q^{t-1}_{j'} never read
    } else if ((int64_t)t + c1.w <= K) {  // reverse window (see k_sweep_reverse)
      if ((int64_t)t + c1.w >= K - 1 && gq_prev && (info < 0 || cur.it == class_item_ptr[jp]))
        stv<V>(gq_prev + (size_t)jp * Bp + s0, zero);
    } else {
      const bool piece = info >= 0 && (info & 1);
      const Vec<V> qp = ldv<V>(q_prev + (size_t)jp * Bp + s0);
      Vec<V> gqacc = zero, X = zero;
      if (bb < be) {
        top_up();
        int k = c1.x;
        if (l2_prefetch) {
          const int nn = c1.y - k + 1;
          const int lines = 2 * nn * V;
          for (int l = lane; l < lines; l += 32) {
            const int arr = l / (nn * V), r = l % (nn * V);
            const float* base = arr ? gcp : cp;
            const float* a = base + (size_t)(k + r / V) * Bp + x0 + (r % V) * 32;
            asm volatile("prefetch.global.L2 [%0];" ::"l"(a));
          }
        }
        size_t ok = (size_t)k * Bp + s0;
        Vec<V> cv = ldv_cs<V>(cp + ok), gc = piece ? zero : ldv_cs<V>(gcp + ok);
        Vec<V> cvn = zero, gcn = zero;
        Vec<V> rom, sI, cC;
        auto node_consts = [&]() {
#pragma unroll
          for (int x = 0; x < V; ++x) {
            const float om = __fsub_rn(1.f, __fmul_rn(cv.v[x], qp.v[x]));
            const bool nz = om != 0.f;
            float r;
            asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(om));
            rom.v[x] = (HI && nz ? r : 1.f) * keep.v[x];
            sI.v[x] = nz ? wI : -wI;
            cC.v[x] = HI && nz ? wC * om : wC;
          }
        };
        node_consts();
        for (int b = bb; b < be; ++b) {
          const int rb = b - bb;
          const int knext = __shfl_sync(0xffffffffu, cur.kl, (rb + 1) & 31);
          const int kn1 = rb + 1 < be - bb ? knext : -1;  // e-node of batch b+1 (-1: none)
          if (kn1 >= 0 && kn1 != k) {
            cvn = ldv_cs<V>(cp + (size_t)kn1 * Bp + s0);
            if (!piece) gcn = ldv_cs<V>(gcp + (size_t)kn1 * Bp + s0);
          }
          const uint32_t st = nc % S;
          mbar_wait(bar0 + 8 * st, (nc / S) & 1);
          const unsigned char* stg = ring + (size_t)st * kRtStage;
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const float4 g4 = reinterpret_cast<const float4*>(stg + u * kRtRow)[lane];
            const float gA[4] = {g4.x, g4.y, g4.z, g4.w};
            float PA[4] = {0.f, 0.f, 0.f, 0.f};
            int aA[4] = {0, 0, 0, 0};
            if (HI) {
              const float4 p4 = reinterpret_cast<const float4*>(stg + (4 + u) * kRtRow)[lane];
              PA[0] = p4.x; PA[1] = p4.y; PA[2] = p4.z; PA[3] = p4.w;
            }
            if (HC) {
              const int4 a4 = reinterpret_cast<const int4*>(stg + (8 + u) * kRtRow)[lane];
              aA[0] = a4.x; aA[1] = a4.y; aA[2] = a4.z; aA[3] = a4.w;
            }
#pragma unroll
            for (int x = 0; x < V; ++x) {
              if (HI) X.v[x] = fmaf(gA[x], fmaxf(sI.v[x] * PA[x], 0.f), X.v[x]);
              if (HC && aA[x] == k) X.v[x] = fmaf(gA[x], cC.v[x], X.v[x]);
            }
          }
          ++nc;
          top_up();  // the stage just read is free: request the next batch
          if (kn1 != k && !piece) {  // finalise e-node k
#pragma unroll
            for (int x = 0; x < V; ++x) {
              const float gp = X.v[x] * rom.v[x];
              gc.v[x] += gp * qp.v[x];
              gqacc.v[x] += gp * cv.v[x];
            }
            stv_cs<V>(gcp + ok, gc);
            if (kn1 >= 0) {
              k = kn1;
              ok = (size_t)k * Bp + s0;
              cv = cvn;
              gc = gcn;
              node_consts();
              X = zero;
            }
          }
        }
      }
      Vec<V> pass = zero;
      reverse_epilogue<V, HI, false>(lane, jp, info, piece, Bp, root, s0, keep, qp, gqacc, X,
                                     items, class_item_ptr, cp, gcp, gq_prev, part, cnt, pass, gq,
                                     live_out, gstamp, t);
    }
    // advance the queue: nxt becomes current (with the batches already requested)
    cur = nxt;
    cur_req = nxt_req;
    nxt = load_item(cur.it + T);
    nxt_req = 0;
  }
}

// Tensor map of the [M][Bp] rows the TMA reverse sweep gathers (box: one
// 128-seed row)
static CUtensorMap row_map(const void* base, int M, int Bp, bool is_int) {
  return tensor_map_2d(base, is_int, (uint64_t)Bp, (uint64_t)M, (uint64_t)Bp * 4, 128, 1);
}

// Opt-in (SMOOTHE_REV_TMA=1): measured slower than the register kernel on C4
// ("tried"); read at every host-side launch (A/B, tests).
static bool reverse_tma_enabled() {
  const char* e = std::getenv("SMOOTHE_REV_TMA");
  return e && e[0] == '1';
}

void launch_sweep_reverse(cudaStream_t s, const Shape& sh, const DevGraph& g, Agg a, int t, int K,
                          const float* q_prev, const float* pi, const int32_t* am,
                          const int32_t* wm, const float* cp, const float* gq, float* gcp,
                          float* gq_prev, bool write_gq_prev, float* rev_part, int32_t* rev_cnt,
                          const int32_t* lastchg, int32_t* cursor, const int32_t* live_in,
                          int32_t* live_out, int32_t* gstamp, bool persist) {
  float* out = write_gq_prev ? gq_prev : nullptr;
  if (!out) live_out = gstamp = nullptr;
#ifndef SMOOTHE_REV_VMAX
#define SMOOTHE_REV_VMAX 4  // seeds per lane at Bp >= 128 (4: one warp per 128-seed slice)
#endif
  const int V = sh.Bp >= 32 * SMOOTHE_REV_VMAX ? SMOOTHE_REV_VMAX : sh.Bp / 32;
  const int n = g.num_rev_items;
  // cp / g_cp rows are L2-prefetched per item only when they cannot stay
  // L2-resident (measured: +7% on C4 at 512 MB, -9% on C3 at 13 MB)
  const bool l2_prefetch = (double)sh.N * sh.Bp * sizeof(float) > 64e6;
  if (V == 4 && !lastchg && cursor && reverse_tma_enabled()) {
    const bool HI = a.wI != 0.f, HC = a.wC != 0.f;
    const CUtensorMap mg = row_map(gq, sh.M, sh.Bp, false);
    const CUtensorMap mp = row_map(HI ? (const void*)pi : (const void*)gq, sh.M, sh.Bp, false);
    const CUtensorMap ma = row_map(HC ? (const void*)am : (const void*)gq, sh.M, sh.Bp, true);
    int dev = 0;
    SM_CUDA(cudaGetDevice(&dev));
    const dim3 grid(SMOOTHE_RT_CTAS * num_sms(dev), sh.Bp / 128);
#define SM_RT(HI_, HC_)                                                                           do {                                                                                              static bool attr = false;                                                                       if (!attr) {                                                                                      SM_CUDA(cudaFuncSetAttribute(k_sweep_reverse_tma<HI_, HC_>,                                                                  cudaFuncAttributeMaxDynamicSharedMemorySize, kRtSmem));            attr = true;                                                                                  }                                                                                               k_sweep_reverse_tma<HI_, HC_><<<grid, 32 * kRtWarps, kRtSmem, s>>>(                                 mg, mp, ma, n, sh.Bp, sh.root, reinterpret_cast<const int4*>(g.rev_item),                       g.rev_class_item_ptr, g.pad_child, g.pad_batch_node, a.wI, a.wC, cp, q_prev, gq, gcp,           out, rev_part, rev_cnt, l2_prefetch, t, K, wm, cursor, live_in, live_out, gstamp);                                   } while (0)
    if (HI && HC) SM_RT(true, true);
    else if (HI) SM_RT(true, false);
    else SM_RT(false, true);
#undef SM_RT
    SM_LAUNCH_CHECK();
    return;
  }
  dim3 grid((n + kRevBlock / 32 - 1) / (kRevBlock / 32), sh.Bp / (32 * V));
  int stride = n;
  persist = persist && V == 4 && !lastchg;
  if (persist) {  // one wave of resident blocks
    int dev = 0;
    SM_CUDA(cudaGetDevice(&dev));
    static int wave[64] = {0};
    int& nb = wave[dev & 63];
    if (!nb) {
      SM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(
          &nb, k_sweep_reverse<4, true, true, false, true>, kRevBlock, 0));
      nb = std::max(1, nb) * num_sms(dev);
    }
    grid.x = std::min<unsigned>(grid.x, (unsigned)nb);
    stride = (int)grid.x * (kRevBlock / 32);
  }
#define SM_REV3(VV, HI, HC, CV)                                                                \
  if (VV == 4 && !CV && persist)                                                               \
    k_sweep_reverse<VV, HI, HC, CV, VV == 4 && !CV><<<grid, kRevBlock, 0, s>>>(                \
        n, sh.Bp, sh.root, reinterpret_cast<const int4*>(g.rev_item), g.rev_class_item_ptr,    \
        g.pad_child, g.pad_batch_node, a.wI, a.wC, cp, q_prev, gq, pi, am, gcp, out,           \
        rev_part, rev_cnt, l2_prefetch, t, K, wm, lastchg, live_in, live_out, gstamp, stride); \
  else                                                                                         \
  k_sweep_reverse<VV, HI, HC, CV><<<grid, kRevBlock, 0, s>>>(                                  \
      n, sh.Bp, sh.root, reinterpret_cast<const int4*>(g.rev_item), g.rev_class_item_ptr,      \
      g.pad_child, g.pad_batch_node, a.wI, a.wC, cp, q_prev, gq, pi, am, gcp, out,             \
      rev_part, rev_cnt, l2_prefetch, t, K, wm, lastchg, live_in, live_out, gstamp, stride)
#define SM_REV2(VV, HI, HC)                                                                    \
  do {                                                                                         \
    if (lastchg) SM_REV3(VV, HI, HC, true);                                                    \
    else SM_REV3(VV, HI, HC, false);                                                           \
  } while (0)
#define SM_REV(VV)                                                                             \
  do {                                                                                         \
    if (a.wI != 0.f && a.wC != 0.f) SM_REV2(VV, true, true);                                   \
    else if (a.wI != 0.f) SM_REV2(VV, true, false);                                            \
    else SM_REV2(VV, false, true);                                                             \
  } while (0)
  if (V == 4) SM_REV(4);
  else if (V == 2) SM_REV(2);
  else SM_REV(1);
#undef SM_REV
#undef SM_REV2
#undef SM_REV3
  SM_LAUNCH_CHECK();
}


// ---------------------------------------------------------------------------
// Frozen reverse sweeps.  In fp32 the forward iterates
// freeze: from some sweep on, a seed's q^{t-1}, pi^t and am^t rows equal the
// K-state (q^{K-1}, pi^K, am^K) bit for bit.  Reverse sweep t is then linear
// in g_q^t with coefficients that no longer depend on t:
//   g_p^t_k = sum_{j in ch_k} c_kj g_q^t_j,
//   c_kj = (wI max(s pi_j, 0) + [am_j = k] wC r) * rom    (the reverse kernel's
//          per-e-node constants s, r, rom of the K-state),
//   g_q^{t-1}_i = sum_{k in m_i} cp_k g_p^t_k = sum_j W_ij g_q^t_j,
//   W_ij = sum_{k in m_i, j in ch_k} cp_k c_kj        (one row per class edge),
// and its g_cp contribution q_i g_p^t_k sums over the frozen sweeps to
// q_i sum_j c_kj S_j with S_j = sum_t g_q^t_j: one more reverse-kernel pass
// over the K-state with g = S at the end of the step.  A frozen sweep is thus
// one streamed W row and one gathered g_q row per class edge (C4: 3.5M class
// edges against 5.5M child slots x three gathered rows).  A seed is frozen in
// reverse sweep t while none of its q rows changed in forward sweeps t..K-1:
// every seed is at t = K, and the transition into sweep t (which restores the
// rows forward sweep t recomputed) clears wm[s] when a restored row differs
// in seed s.  Decisions are per seed, so results do not depend on the batch.
// ---------------------------------------------------------------------------
// One row group per EP class edges (i, j), interleaved so that their loads
// are in flight together (the kernel is bound by its dependent gathers):
// W_ij = sum over the edge's e-nodes k (ascending) of cp_k c_kj, with pi_j /
// am_j / q_i loaded once per edge.
#ifndef SMOOTHE_WBUILD_EP
#define SMOOTHE_WBUILD_EP 2
#endif
template <int LPR>
__global__ void __launch_bounds__(kBlock) k_wbuild(
    int64_t n_cedge, int Bp, float wI, float wC, const int32_t* __restrict__ cedge_class,
    const int32_t* __restrict__ cedge_ptr, const int32_t* __restrict__ cedge_node,
    const int32_t* __restrict__ cls_child, const float* __restrict__ cp,
    const float* __restrict__ kq, const float* __restrict__ kpi, const int32_t* __restrict__ kam,
    float* __restrict__ W) {
  constexpr int EP = SMOOTHE_WBUILD_EP;
  const RowGroup<LPR> rg;
  const int64_t ce0 = ((int64_t)blockIdx.x * (kBlock / LPR) + rg.sub) * EP;
  if (ce0 >= n_cedge) return;
  const bool HI = wI != 0.f, HC = wC != 0.f;
  int64_t ce[EP];
  int i[EP], j[EP], a0[EP], a1[EP];
#pragma unroll
  for (int e = 0; e < EP; ++e) {
    ce[e] = ce0 + e < n_cedge ? ce0 + e : ce0;  // a tail pair repeats its first edge (same value)
    i[e] = cedge_class[ce[e]];
    j[e] = cls_child[ce[e]];
    a0[e] = cedge_ptr[ce[e]];
    a1[e] = cedge_ptr[ce[e] + 1];
  }
  float4 qp[EP], P[EP], w[EP];
  int4 A[EP];
#pragma unroll
  for (int e = 0; e < EP; ++e) {
    qp[e] = ld4(kq + (size_t)i[e] * Bp + rg.s0);
    P[e] = HI ? ld4(kpi + (size_t)j[e] * Bp + rg.s0) : make_float4(0.f, 0.f, 0.f, 0.f);
    A[e] = ld4i(kam + (size_t)j[e] * Bp + rg.s0);
    w[e] = make_float4(0.f, 0.f, 0.f, 0.f);
  }
  int n = 0;
#pragma unroll
  for (int e = 0; e < EP; ++e) n = max(n, a1[e] - a0[e]);
  for (int u = 0; u < n; ++u) {
    int k[EP];
    float4 cv[EP];
#pragma unroll
    for (int e = 0; e < EP; ++e) {
      k[e] = a0[e] + u < a1[e] ? cedge_node[a0[e] + u] : -1;
      if (k[e] >= 0) cv[e] = ld4(cp + (size_t)k[e] * Bp + rg.s0);
    }
#pragma unroll
    for (int e = 0; e < EP; ++e) {
      if (k[e] < 0) continue;
#pragma unroll
      for (int x = 0; x < 4; ++x) {  // node_consts of k_sweep_reverse, then c_kj
        const float om = __fsub_rn(1.f, __fmul_rn(comp(cv[e], x), comp(qp[e], x)));
        const bool nz = om != 0.f;
        float r;
        asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(om));
        const float rom = HI && nz ? r : 1.f;
        const float cC = HI && nz ? wC * om : wC;
        float c = HI ? wI * fmaxf((nz ? 1.f : -1.f) * comp(P[e], x), 0.f) : 0.f;
        if (HC && comp(A[e], x) == k[e]) c += cC;
        comp(w[e], x) = fmaf(comp(cv[e], x), c * rom, comp(w[e], x));
      }
    }
  }
#pragma unroll
  for (int e = 0; e < EP; ++e)
    if (ce0 + e < n_cedge) st4(W + (size_t)ce[e] * Bp + rg.s0, w[e]);
}

void launch_wbuild(cudaStream_t s, const Shape& sh, const DevGraph& g, Agg a,
                   const SweepState& st, const float* cp) {
  SM_DISPATCH_LPR(sh.Bp, {
    k_wbuild<LPR><<<row_grid((int)((g.num_cedge + SMOOTHE_WBUILD_EP - 1) / SMOOTHE_WBUILD_EP),
                             sh.Bp, LPR), kBlock, 0, s>>>(
        g.num_cedge, sh.Bp, a.wI, a.wC, g.cedge_class, g.cedge_ptr, g.cedge_node, g.cls_child,
        cp, st.kq, st.kpi, st.kam, st.W);
  });
  SM_LAUNCH_CHECK();
}

#ifndef SMOOTHE_WSPMV_BLOCK
#define SMOOTHE_WSPMV_BLOCK 64
#endif
constexpr int kWBlock = SMOOTHE_WSPMV_BLOCK;
// min resident blocks for 128-seed rows: 12 (<= 85 registers, no spills);
// measured on C4 (ms per step): 10 -> 135.7, 12 -> 120.2, 14 -> 128.5, 16 ->
// 147.4.  None for narrower rows (C5: slower).  DEPTH edges in flight per row group.
#ifndef SMOOTHE_WSPMV_MINB
#define SMOOTHE_WSPMV_MINB 20
#endif
#ifndef SMOOTHE_WSPMV_DEPTH
#define SMOOTHE_WSPMV_DEPTH 6
#endif
#ifndef SMOOTHE_WSPMV_MINB16
#define SMOOTHE_WSPMV_MINB16 1  // min resident blocks for narrower rows (LPR <= 16)
#endif
#ifndef SMOOTHE_WSPMV_DEPTH32
#define SMOOTHE_WSPMV_DEPTH32 4
#endif
// One W work item (row group of LPR lanes; rows [s0, s0 + 4) of its seeds).
template <int LPR, bool STREAM, bool CONV>
__device__ __forceinline__ void wspmv_item(
    int row, int s0, int Bp, int root, int t, const int32_t* __restrict__ dmin,
    const int4* __restrict__ items, const int32_t* __restrict__ cls_child_ptr,
    const int32_t* __restrict__ cls_child, const float* __restrict__ W, int4 w4, unsigned gm,
    bool lead, bool check, const float* __restrict__ gq, float* __restrict__ S,
    float* __restrict__ gq_prev, float* __restrict__ part, const int32_t* __restrict__ lastchg,
    int32_t* __restrict__ live_out, int32_t* __restrict__ gstamp,
    const int32_t* __restrict__ gstamp_in, int32_t* __restrict__ wcnt) {
  const int4 itm = items[row];
  const int i = itm.x, e0 = itm.y, e1 = itm.z, slot = itm.w;
  const int d = __ldg(dmin + i);
  const size_t oi = (size_t)i * Bp + s0;
  // converge mode: a frozen seed's sweeps after its convergence sweep
  // lastchg + 1 were never performed: its g_q passes through unchanged
  int4 cp4 = make_int4(0, 0, 0, 0);  // copy mode per seed
  if (CONV) {
    const int4 lc = ld4i(lastchg + s0);
    cp4 = make_int4(w4.x && t > lc.x + 1, w4.y && t > lc.y + 1, w4.z && t > lc.z + 1,
                    w4.w && t > lc.w + 1);
  }
  if (d <= t && e0 == cls_child_ptr[i] &&
      (!check || __ldcg(gstamp_in + (size_t)i * gridDim.y + blockIdx.y) == t)) {
    // first item: S_i += g_q^t_i (a valid, non-zero row)
    const float4 gi = ld4(gq + oi);
    float4 si = ld4(S + oi);
#pragma unroll
    for (int x = 0; x < 4; ++x)
      if (comp(w4, x) && !comp(cp4, x)) comp(si, x) += comp(gi, x);
    st4(S + oi, si);
  }
  if (d > t - 1 || !gq_prev) return;  // q^{t-1}_i = 0: the row is never read
  const bool anyw = !CONV || __any_sync(gm, (comp(w4, 0) && !comp(cp4, 0)) || (comp(w4, 1) && !comp(cp4, 1)) ||
                                       (comp(w4, 2) && !comp(cp4, 2)) || (comp(w4, 3) && !comp(cp4, 3)));
  if (!anyw) {  // every frozen seed of the row group is past its convergence sweep
    if (e0 != cls_child_ptr[i]) return;  // the class's first item copies the row
    const float4 gi = ld4(gq + oi);
    float4 o = gi;
    if (!(w4.x && w4.y && w4.z && w4.w)) {
      const float4 cur = ld4(gq_prev + oi);
#pragma unroll
      for (int x = 0; x < 4; ++x)
        if (!comp(w4, x)) comp(o, x) = comp(cur, x);
    }
    st4(gq_prev + oi, o);
    g_mark(live_out, gm, o.x != 0.f || o.y != 0.f || o.z != 0.f || o.w != 0.f, lead,
           gstamp ? gstamp + (size_t)i * gridDim.y + blockIdx.y : nullptr, t - 1);
    return;
  }
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  // the row group loads LPR child indices at once (one per lane, coalesced)
  // and broadcasts them, so the W rows (streamed) and g_q rows (gathered) of
  // 8 edges are in flight together without a dependent index load each
  const int gl = threadIdx.x % LPR;
  for (int c0 = e0; c0 < e1; c0 += LPR) {
    const int n = min(LPR, e1 - c0);
    const int myj = gl < n ? __ldg(cls_child + c0 + gl) : 0;
    const bool myl = gl < n && (!check || __ldcg(gstamp_in + (size_t)myj * gridDim.y + blockIdx.y) == t);
    // the row group's live children (a child whose g_q^t is all zero adds
    // nothing: no W or g_q load), visited in ascending order, DP in flight
    unsigned lm = __ballot_sync(gm, myl);
    if (LPR < 32) lm = (lm >> ((threadIdx.x % 32) / LPR * LPR)) & (LPR == 32 ? 0xffffffffu : (1u << LPR) - 1u);
    const float* wrow = W + (size_t)c0 * Bp + s0;
    constexpr int DP = LPR == 32 ? SMOOTHE_WSPMV_DEPTH32 : SMOOTHE_WSPMV_DEPTH;
    while (lm) {
      float4 wv[DP], gv[DP];
#pragma unroll
      for (int v = 0; v < DP; ++v) {
        const int e = lm ? __ffs(lm) - 1 : 0;
        const bool has = lm != 0;
        lm &= lm - 1;
        const int j = __shfl_sync(gm, myj, e, LPR);
        if (has) {
          wv[v] = STREAM ? ldcs4(wrow + (size_t)e * Bp) : ld4(wrow + (size_t)e * Bp);
          gv[v] = ld4(gq + (size_t)j * Bp + s0);
        } else {
          wv[v] = make_float4(0.f, 0.f, 0.f, 0.f);
          gv[v] = wv[v];
        }
      }
#pragma unroll
      for (int v = 0; v < DP; ++v) {
        acc.x = fmaf(wv[v].x, gv[v].x, acc.x);
        acc.y = fmaf(wv[v].y, gv[v].y, acc.y);
        acc.z = fmaf(wv[v].z, gv[v].z, acc.z);
        acc.w = fmaf(wv[v].w, gv[v].w, acc.w);
      }
    }
  }
  if (slot >= 0) {  // one chunk of a long class
    st4(part + (size_t)slot * Bp + s0, acc);
    if (CONV || !wcnt) return;  // k_wcombine adds the chunks
    // the class's last chunk to finish adds the partial rows in slot order
    // (k_wcombine's order: bit-identical) and writes g_q^{t-1}_i.  Chunks sit
    // at ptr + 64 k (slots first + k), so the first slot and the count follow
    // from the class's child range; one counter per (class, seed chunk),
    // reset by the last arriver.
    const int ptr = cls_child_ptr[i], nsl = (cls_child_ptr[i + 1] - ptr + kWChunk - 1) / kWChunk;
    const int first = slot - (e0 - ptr) / kWChunk;
    __threadfence();
    __syncwarp(gm);
    int last = 0;
    int32_t* c = wcnt + (size_t)first * gridDim.y + blockIdx.y;
    if (lead) last = atomicAdd(c, 1) == nsl - 1;
    if (!__shfl_sync(gm, last, (threadIdx.x % 32) / LPR * LPR)) return;
    __threadfence();
    if (lead) *c = 0;
    acc = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int sl = first; sl < first + nsl; ++sl) {
      const float4 p = __ldcg(reinterpret_cast<const float4*>(part + (size_t)sl * Bp + s0));
      acc.x += p.x;
      acc.y += p.y;
      acc.z += p.z;
      acc.w += p.w;
    }
  }
  if (i == root) acc = make_float4(0.f, 0.f, 0.f, 0.f);
  float4 o = acc;
  if (CONV) {  // seeds past their convergence sweep pass g_q^t through
    const float4 gi = ld4(gq + oi);
#pragma unroll
    for (int x = 0; x < 4; ++x)
      if (comp(cp4, x)) comp(o, x) = comp(gi, x);
  }
  if (!(w4.x && w4.y && w4.z && w4.w)) {  // mixed: keep the reverse kernel's seeds
    const float4 cur = ld4(gq_prev + oi);
#pragma unroll
    for (int x = 0; x < 4; ++x)
      if (!comp(w4, x)) comp(o, x) = comp(cur, x);
  }
  st4(gq_prev + oi, o);
  g_mark(live_out, gm, o.x != 0.f || o.y != 0.f || o.z != 0.f || o.w != 0.f, lead,
         gstamp ? gstamp + (size_t)i * gridDim.y + blockIdx.y : nullptr, t - 1);
}


template <int LPR, bool STREAM, bool CONV, bool PERSIST>
__global__ void __launch_bounds__(kWBlock, LPR == 32 ? SMOOTHE_WSPMV_MINB * 64 / kWBlock : SMOOTHE_WSPMV_MINB16) k_wspmv(
    int n_items, int Bp, int root, int t, const int32_t* __restrict__ dmin,
    const int4* __restrict__ items, const int32_t* __restrict__ cls_child_ptr,
    const int32_t* __restrict__ cls_child, const float* __restrict__ W,
    const int32_t* __restrict__ wm, const float* __restrict__ gq, float* __restrict__ S,
    float* __restrict__ gq_prev, float* __restrict__ part, int64_t* __restrict__ frozen_count,
    const int32_t* __restrict__ lastchg, const int32_t* __restrict__ live_in,
    int32_t* __restrict__ live_out, int32_t* __restrict__ gstamp,
    const int32_t* __restrict__ gstamp_in, int32_t* __restrict__ wcnt) {
  const RowGroup<LPR, kWBlock> rg;
  if (frozen_count && blockIdx.x == 0 && blockIdx.y == 0 && threadIdx.x == 0 &&
      !g_dead(live_in)) {  // profiling: a working launch?
    bool any = false;
    for (int b = 0; b < Bp && !any; ++b) any = wm[b] != 0;
    if (any) atomicAdd(reinterpret_cast<unsigned long long*>(frozen_count), 1ull);
  }
  if (rg.row >= n_items || g_dead(live_in)) return;
  const int4 w4 = ld4i(wm + rg.s0);
  const unsigned gm = LPR == 32 ? 0xffffffffu
                                : ((1u << LPR) - 1u) << ((threadIdx.x % 32) / LPR * LPR);
  const bool lead = threadIdx.x % LPR == 0;
  // g_q^t_j may be non-zero only if sweep t + 1 stamped row j with t (every
  // writer of a non-zero row does); sweep K reads the cost's g_q^K rows
  const bool check = gstamp_in && live_in;
  if (!__any_sync(gm, (w4.x | w4.y | w4.z | w4.w) != 0)) return;  // row-group uniform
  // persistent launches (one wave of resident blocks): row group g takes
  // items g, g + G, ... (round robin keeps the items in flight a compact
  // window); otherwise one item per row group
  const int G = PERSIST ? gridDim.x * (kWBlock / LPR) : n_items;
  for (int row = rg.row; row < n_items; row += G)
    wspmv_item<LPR, STREAM, CONV>(row, rg.s0, Bp, root, t, dmin, items, cls_child_ptr, cls_child,
                                  W, w4, gm, lead, check, gq, S, gq_prev, part, lastchg, live_out,
                                  gstamp, gstamp_in, wcnt);
}

// g_q^{t-1}_i of the classes split into several chunks: their partial rows in
// item order (deterministic)
template <int LPR>
__global__ void __launch_bounds__(kBlock) k_wcombine(
    int n_multi, int Bp, int root, int t, const int32_t* __restrict__ dmin,
    const int32_t* __restrict__ wmulti, const int32_t* __restrict__ wmulti_ptr,
    const int32_t* __restrict__ wm, const float* __restrict__ part, float* __restrict__ gq_prev,
    const int32_t* __restrict__ lastchg, const float* __restrict__ gq,
    const int32_t* __restrict__ live_in, int32_t* __restrict__ live_out,
    int32_t* __restrict__ gstamp) {
  const RowGroup<LPR> rg;
  if (rg.row >= n_multi || g_dead(live_in)) return;
  const unsigned gm = LPR == 32 ? 0xffffffffu
                                : ((1u << LPR) - 1u) << ((threadIdx.x % 32) / LPR * LPR);
  const int4 w4 = ld4i(wm + rg.s0);
  if (!(w4.x | w4.y | w4.z | w4.w)) return;
  const int i = wmulti[rg.row];
  if (__ldg(dmin + i) > t - 1) return;
  int4 cp4 = make_int4(0, 0, 0, 0);
  if (lastchg) {
    const int4 lc = ld4i(lastchg + rg.s0);
    cp4 = make_int4(w4.x && t > lc.x + 1, w4.y && t > lc.y + 1, w4.z && t > lc.z + 1,
                    w4.w && t > lc.w + 1);
    // every frozen seed past its convergence sweep: k_wspmv's first item copied the row
    if ((!w4.x || cp4.x) && (!w4.y || cp4.y) && (!w4.z || cp4.z) && (!w4.w || cp4.w)) return;
  }
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int sl = wmulti_ptr[rg.row]; sl < wmulti_ptr[rg.row + 1]; ++sl) {
    const float4 p = ld4(part + (size_t)sl * Bp + rg.s0);
    acc.x += p.x;
    acc.y += p.y;
    acc.z += p.z;
    acc.w += p.w;
  }
  if (i == root) acc = make_float4(0.f, 0.f, 0.f, 0.f);
  const size_t oi = (size_t)i * Bp + rg.s0;
  float4 o = acc;
  if (lastchg) {
    const float4 gi = ld4(gq + oi);
#pragma unroll
    for (int x = 0; x < 4; ++x)
      if (comp(cp4, x)) comp(o, x) = comp(gi, x);
  }
  if (!(w4.x && w4.y && w4.z && w4.w)) {
    const float4 cur = ld4(gq_prev + oi);
#pragma unroll
    for (int x = 0; x < 4; ++x)
      if (!comp(w4, x)) comp(o, x) = comp(cur, x);
  }
  st4(gq_prev + oi, o);
  g_mark(live_out, gm, o.x != 0.f || o.y != 0.f || o.z != 0.f || o.w != 0.f,
         threadIdx.x % LPR == 0, gstamp ? gstamp + (size_t)i * gridDim.y + blockIdx.y : nullptr,
         t - 1);
}

// Profiling only (bench.py's roofline of k_wspmv): the (row, seed chunk)
// units frozen sweep t actually moves: out[0] += class edges (i, j) with i
// inside the window (dmin_i <= t - 1) and g_q^t_j live (W row loaded),
// out[1] += rows with a live g_q^t_i inside the window (g_q^t and S read, S
// written), out[2] += rows written (dmin_i <= t - 1).  stamp_in NULL: all live.
__global__ void k_count_live(int64_t n_cedge, int M, int nchunk, int t,
                             const int32_t* __restrict__ cedge_class,
                             const int32_t* __restrict__ cls_child,
                             const int32_t* __restrict__ dmin, const int32_t* __restrict__ stamp_in,
                             const int32_t* __restrict__ live_in, int64_t* __restrict__ out) {
  if (g_dead(live_in)) return;  // the sweep is skipped
  const int64_t ne = n_cedge * nchunk, nr = (int64_t)M * nchunk;
  unsigned long long c[3] = {0, 0, 0};
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < ne + nr;
       e += (int64_t)gridDim.x * blockDim.x) {
    if (e < ne) {
      const int64_t ce = e / nchunk;
      const int ch = (int)(e % nchunk), i = cedge_class[ce], j = cls_child[ce];
      c[0] += dmin[i] <= t - 1 && (!stamp_in || stamp_in[(size_t)j * nchunk + ch] == t);
    } else {
      const int64_t r = e - ne;
      const int i = (int)(r / nchunk), ch = (int)(r % nchunk);
      c[1] += dmin[i] <= t && (!stamp_in || stamp_in[(size_t)i * nchunk + ch] == t);
      c[2] += dmin[i] <= t - 1;
    }
  }
#pragma unroll
  for (int x = 0; x < 3; ++x) {
    for (int o = 16; o > 0; o >>= 1) c[x] += __shfl_xor_sync(0xffffffffu, c[x], o);
    if (threadIdx.x % 32 == 0 && c[x])
      atomicAdd(reinterpret_cast<unsigned long long*>(out + x), c[x]);
  }
}

void launch_count_live(cudaStream_t s, const Shape& sh, const DevGraph& g, int t,
                       const SweepState& st, int64_t* out) {
  const size_t sm_n = (size_t)st.nchunk * sh.M;
  const int32_t* stamp_in = st.gstamp && t < st.K ? st.gstamp + (t & 1) * sm_n : nullptr;
  k_count_live<<<4 * st.num_sms, 256, 0, s>>>(g.num_cedge, sh.M, st.nchunk, t, g.cedge_class,
                                              g.cls_child, g.dmin, stamp_in,
                                              st.glive && t < st.K ? st.glive + t : nullptr, out);
  SM_LAUNCH_CHECK();
}

void launch_wspmv(cudaStream_t s, const Shape& sh, const DevGraph& g, int t,
                  const SweepState& st, const float* gq, float* gq_prev, int64_t* frozen_count) {
  // W streams from HBM once per sweep (evict-first) unless it fits in L2 with
  // room to spare, where it stays resident across the frozen sweeps (C5: 69 MB)
  const bool stream = (double)g.num_cedge * sh.Bp * sizeof(float) > 96e6;
  const int4* items = reinterpret_cast<const int4*>(g.witem);
  const int32_t* live_in = st.glive && t < st.K ? st.glive + t : nullptr;
  int32_t* live_out = st.glive && gq_prev ? st.glive + (t - 1) : nullptr;
  // stamps by sweep parity: sweep t reads buffer t & 1 while writing (t - 1) & 1
  const size_t sm_n = (size_t)st.nchunk * sh.M;
  int32_t* gstamp = gq_prev && st.gstamp ? st.gstamp + ((t - 1) & 1) * sm_n : nullptr;
  const int32_t* gstamp_in = st.gstamp ? st.gstamp + (t & 1) * sm_n : nullptr;
#define SM_WSPMV(ST, CV)                                                                       \
  if (persist) {                                                                               \
    static int wave[64] = {0};                                                                 \
    int& nb = wave[dev & 63];                                                                  \
    if (!nb) {                                                                                 \
      SM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_wspmv<LPR, ST, CV, true>,   \
                                                            kWBlock, 0));                      \
      nb = std::max(1, nb) * num_sms(dev);                                                     \
    }                                                                                          \
    grid.x = std::min<unsigned>(grid.x, (unsigned)nb);                                         \
    k_wspmv<LPR, ST, CV, true><<<grid, kWBlock, 0, s>>>(                                       \
        g.num_witems, sh.Bp, sh.root, t, g.dmin, items, g.cls_child_ptr, g.cls_child, st.W,    \
        st.wm, gq, st.S, gq_prev, st.wpart, frozen_count, st.lastchg, live_in, live_out,       \
        gstamp, gstamp_in, wcnt);                                                              \
  } else                                                                                       \
  k_wspmv<LPR, ST, CV, false><<<grid, kWBlock, 0, s>>>(                                        \
      g.num_witems, sh.Bp, sh.root, t, g.dmin, items, g.cls_child_ptr, g.cls_child, st.W, st.wm, \
      gq, st.S, gq_prev, st.wpart, frozen_count, st.lastchg, live_in, live_out, gstamp, gstamp_in, \
      wcnt)
  // persistent row groups (one wave of resident blocks striding over the
  // items) for large item counts: the launch of ~85k blocks costs ~45 us per
  // sweep on C4 (SMOOTHE_WSPMV_PERSIST=0 / 1 forces)
  const bool persist = st.wpersist;
  // long classes: the last chunk combines inside k_wspmv (no k_wcombine
  // launch per sweep) except in convergence mode
  int32_t* wcnt = st.wcnt && !st.converge && gq_prev ? st.wcnt : nullptr;
  int dev = 0;
  SM_CUDA(cudaGetDevice(&dev));
  SM_DISPATCH_LPR(sh.Bp, {
    dim3 grid = row_grid(g.num_witems, sh.Bp, LPR, kWBlock);
    if (st.converge) {
      if (stream) SM_WSPMV(true, true);
      else SM_WSPMV(false, true);
    } else {
      if (stream) SM_WSPMV(true, false);
      else SM_WSPMV(false, false);
    }

    if (g.num_wmulti > 0 && gq_prev && !wcnt) {
      SM_LAUNCH_CHECK();
      k_wcombine<LPR><<<row_grid(g.num_wmulti, sh.Bp, LPR), kBlock, 0, s>>>(
          g.num_wmulti, sh.Bp, sh.root, t, g.dmin, g.wmulti, g.wmulti_ptr, st.wm, st.wpart,
          gq_prev, st.converge ? st.lastchg : nullptr, gq, live_in, live_out, gstamp);
    }
  });
#undef SM_WSPMV
  SM_LAUNCH_CHECK();
}


// Converge mode: lastchg[s] = max over sweeps t and classes j recomputed in t of
// t if version t of q_j differs from its previous version in seed s.  Grid
// (x: entries, y: sweep t - 1, z: seed chunk = pool); per-block flags, one
// atomicMax per seed and block.
template <int LPR>
__global__ void __launch_bounds__(kBlock) k_last_change(int M, PoolArgs P,
                                                       int32_t* __restrict__ lastchg) {
  __shared__ int flag[4 * LPR];
  const int t = blockIdx.y + 1, c = blockIdx.z;
  const int gl = threadIdx.x % LPR, sub = threadIdx.x / LPR;
  if (threadIdx.x < 4 * LPR) flag[threadIdx.x] = 0;
  __syncthreads();
  const int n = P.list_n[(size_t)c * (P.K + 2) + t];
  const int4* lt = P.list + ((size_t)c * (P.K + 1) + t) * M;
  const size_t pbase = (size_t)c * P.cap;
  for (int e = blockIdx.x * (kBlock / LPR) + sub; e < n; e += gridDim.x * (kBlock / LPR)) {
    const int4 en = lt[e];
    const float4 a = ld4(P.q + (pbase + en.z) * P.wc + gl * 4),
                 b = ld4(P.q + (pbase + en.y) * P.wc + gl * 4);
#pragma unroll
    for (int x = 0; x < 4; ++x)
      if (__float_as_uint(comp(a, x)) != __float_as_uint(comp(b, x))) flag[gl * 4 + x] = 1;
  }
  __syncthreads();
  if (threadIdx.x < 4 * LPR && flag[threadIdx.x])
    atomicMax(lastchg + c * (4 * LPR) + threadIdx.x, t);
}

void launch_last_change(cudaStream_t s, const Shape& sh, const SweepState& st) {
  SM_CUDA(cudaMemsetAsync(st.lastchg, 0, sizeof(int32_t) * sh.Bp, s));
  const PoolArgs P = pool_args(sh, st);
  SM_DISPATCH_LPR(sh.Bp, {
    const dim3 grid(64, st.K, num_chunks(sh.Bp));
    k_last_change<LPR><<<grid, kBlock, 0, s>>>(sh.M, P, st.lastchg);
  });
  SM_LAUNCH_CHECK();
}


// Conditional graph node of the plain reverse sweep: run it iff some seed is
// not frozen (the real seeds; padded columns carry nothing anyone reads).
__global__ void k_any_unfrozen(cudaGraphConditionalHandle h, const int32_t* __restrict__ wm,
                               int Bp) {
  int any = 0;
  for (int b = threadIdx.x; b < Bp; b += blockDim.x) any |= wm[b] == 0;
  any = __syncthreads_or(any);
  if (threadIdx.x == 0) cudaGraphSetConditional(h, any ? 1u : 0u);
}

void launch_any_unfrozen(cudaStream_t s, const Shape& sh, const int32_t* wm,
                         cudaGraphConditionalHandle h) {
  k_any_unfrozen<<<1, 256, 0, s>>>(h, wm, sh.B);
  SM_LAUNCH_CHECK();
}

// Reverse sweeps (t_low - 1, t] as a switch node: 2 (no body) when g_q^t is all
// zero, 1 (the whole sweeps) when a sweep of the block lies within one of the
// last forward sweep that changed a q row (fchg[0]) -- only there can a
// transition restore a row or a seed be unfrozen --, else 0 (k_wspmv alone:
// every seed frozen, no version to restore)
__global__ void k_rev_switch(cudaGraphConditionalHandle h, const int32_t* __restrict__ live,
                             const int32_t* __restrict__ fchg, int t_low) {
  const unsigned v = __ldcg(live) == 0 ? 2u : (t_low <= __ldcg(fchg) + 1 ? 1u : 0u);
  cudaGraphSetConditional(h, v);
}

void launch_rev_switch(cudaStream_t s, const int32_t* live, const int32_t* fchg, int t_low,
                       cudaGraphConditionalHandle h) {
  k_rev_switch<<<1, 1, 0, s>>>(h, live, fchg, t_low);
  SM_LAUNCH_CHECK();
}

__global__ void k_flag_if(cudaGraphConditionalHandle h, const int32_t* __restrict__ flag) {
  cudaGraphSetConditional(h, __ldcg(flag) != 0 ? 1u : 0u);
}

void launch_flag_if(cudaStream_t s, const int32_t* flag, cudaGraphConditionalHandle h) {
  k_flag_if<<<1, 1, 0, s>>>(h, flag);
  SM_LAUNCH_CHECK();
}

}  // namespace smoothe
