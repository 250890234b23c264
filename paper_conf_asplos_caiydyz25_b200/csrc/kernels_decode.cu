// Decode, validity and keep-best (sm_100a).
//
// Sampling: from the root, each selected class m_j takes the
// e-node c_j = argmax cp (= argmax theta, reading S17) and selects all of its
// child classes; completeness (a), (b) holds by construction (P105-107) and
// acyclicity (c) (P109) is checked.  Bit-sliced over seeds: word w of a row
// holds seeds 32w..32w+31.
//
//   sel[k][w]    bit set iff the seed chose e-node k in its class   (softmax kernel)
//   reach[j][w]  least fixpoint of  reach_root = 1,
//                reach_j = OR_{k in pa_j} (reach_{ec(k)} AND sel_k)       (top-down)
//   valid[w]     no selected cycle: checked per strongly connected component
//                (k_decode_levels below).
//
// Discrete cost (reading S19): sum of u over the chosen e-node of every reached
// class, each class once, accumulated in fp64 (exact for integer-valued u).
#include <cooperative_groups.h>

#include <cstdlib>

#include "kcommon.cuh"

namespace cg = cooperative_groups;

namespace smoothe {

// One cooperative kernel computes the reached sets and the validity masks,
// level by level over the condensation of the e-class graph (levels from the
// loader: longest path from the root's strongly connected component):
//  * a class in a trivial component has all its parents at lower levels, so
//    reach_j = OR_{k in pa_j} (reach_{ec(k)} AND sel_k) is final in one pass
//    (one warp per (class, 32-seed word), lanes over the parents);
//  * a non-trivial SCC S (|S| <= 64) is one block job per (SCC, word): its
//    classes' external reach comes from phase A; then, per seed (lane), the
//    chosen e-node of each class of S gives a 64-bit mask of its children
//    inside S, and the local reach closure R and settle closure
//    settle_j = !reach_j OR (children of c_j in S all settled) run in
//    registers on those masks;
//  * a component with more than 64 classes (kSmallScc) runs the same two
//    closures block-wide in place: reach words in `reach`, settle words in
//    `settle`, bit-OR atomics per seed (lane), passes repeated until one
//    changes nothing (__syncthreads_or).  The closures are monotone, so the
//    order of the updates inside a pass does not change the fixpoint;
//  * every cycle of a selection lies inside one SCC, so the selection is valid
//    iff, in every SCC, every reached class settles.  Unsettled reached classes
//    mark their seeds invalid (bit-OR atomics: order-independent, deterministic).
// One grid barrier per phase and level; each class is evaluated once per level.
// (The previous per-warp version walked every e-node of every class of S in
// each fixpoint pass: on C5, with 900-node classes, the slowest SCC set the
// pace of every level, 3.6 ms per decode.)
constexpr int kDecodeWarps = 8;

// Phase B for one (large component, 32-seed word), the whole block: lane =
// seed, warps over the component's classes.
__device__ void decode_big_scc(int n, int c0, int w, int W, int Bp, int root,
                               const int32_t* __restrict__ scc_class,
                               const int32_t* __restrict__ node_slot,
                               const int32_t* __restrict__ slot_jptr,
                               const int32_t* __restrict__ slot_jloc,
                               const int32_t* __restrict__ choice, uint32_t* reach,
                               uint32_t* settle, uint32_t* invalid) {
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t bit = 1u << lane;
  // reach closure: a reached class's chosen e-node reaches its children in S
  for (;;) {
    int chg = 0;
    for (int l = wib; l < n; l += kDecodeWarps) {
      const int j = scc_class[c0 + l];
      if (!(__ldcg(reach + (size_t)j * W + w) & bit)) continue;
      const int q = node_slot[choice[(size_t)j * Bp + 32 * w + lane]];
      if (q < 0) continue;
      for (int e = slot_jptr[q]; e < slot_jptr[q + 1]; ++e) {
        uint32_t* dst = reach + (size_t)scc_class[c0 + slot_jloc[e]] * W + w;
        if (!(__ldcg(dst) & bit)) {
          atomicOr(dst, bit);
          chg = 1;
        }
      }
    }
    if (!__syncthreads_or(chg)) break;
  }
  (void)root;  // the root's reach word is all ones (launch_decode)
  for (int l = wib; l < n; l += kDecodeWarps) {
    const size_t o = (size_t)scc_class[c0 + l] * W + w;
    if (lane == 0) __stcg(settle + o, ~__ldcg(reach + o));
  }
  __syncthreads();
  // settle closure: a reached class settles once every child of its chosen
  // e-node inside S has settled (children outside S settled at lower levels)
  for (;;) {
    int chg = 0;
    for (int l = wib; l < n; l += kDecodeWarps) {
      const int j = scc_class[c0 + l];
      uint32_t* sj = settle + (size_t)j * W + w;
      if (__ldcg(sj) & bit) continue;
      const int q = node_slot[choice[(size_t)j * Bp + 32 * w + lane]];
      bool ok = true;
      if (q >= 0)
        for (int e = slot_jptr[q]; e < slot_jptr[q + 1] && ok; ++e)
          ok = (__ldcg(settle + (size_t)scc_class[c0 + slot_jloc[e]] * W + w) & bit) != 0;
      if (ok) {
        atomicOr(sj, bit);
        chg = 1;
      }
    }
    if (!__syncthreads_or(chg)) break;
  }
  for (int l = wib; l < n; l += kDecodeWarps) {
    const size_t o = (size_t)scc_class[c0 + l] * W + w;
    const uint32_t bad = __ldcg(reach + o) & ~__ldcg(settle + o);
    if (lane == 0 && bad) atomicOr(invalid + w, bad);
  }
}

__global__ void __launch_bounds__(256) k_decode_levels(
    int W, int root, int num_levels, const int32_t* __restrict__ lvl_cptr,
    const int32_t* __restrict__ lvl_class, const int32_t* __restrict__ lvl_sptr,
    const int32_t* __restrict__ lvl_scc, const int32_t* __restrict__ par_ptr,
    const int32_t* __restrict__ par_node, const int32_t* __restrict__ par_class,
    const int32_t* __restrict__ class_ptr, const int32_t* __restrict__ scc_class_ptr,
    const int32_t* __restrict__ scc_class, const int32_t* __restrict__ scc_of_class,
    const int32_t* __restrict__ ent_ptr, const int32_t* __restrict__ ent_i,
    const int32_t* __restrict__ ent_j, const int32_t* __restrict__ ent_node_ptr,
    const int32_t* __restrict__ ent_node, const int32_t* __restrict__ node_slot,
    const int32_t* __restrict__ slot_ptr, const int32_t* __restrict__ slot_node,
    const int32_t* __restrict__ slot_jptr, const int32_t* __restrict__ slot_jloc,
    const uint32_t* __restrict__ sel, int Bp, const int32_t* __restrict__ choice, uint32_t* reach,
    uint32_t* settle, uint32_t* invalid, uint32_t* valid_out) {
  __shared__ uint64_t cm[64][32];  // phase B: children in S of the chosen e-node, per (class, seed)
  __shared__ uint32_t rs0[64];     // phase B: reach words after phase A
  cg::grid_group grid = cg::this_grid();
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int64_t gwarp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int L = 0; L < num_levels; ++L) {
    // phase A: every class of the level ORs in its parents outside its own SCC
    // (all final: they sit at lower levels); one warp per (class, word), lanes
    // over the parents.  For trivial classes this is the final reach.
    const int c0l = lvl_cptr[L];
    const int64_t nA = (int64_t)(lvl_cptr[L + 1] - c0l) * W;
    for (int64_t it = gwarp; it < nA; it += nwarps) {
      const int j = lvl_class[c0l + it / W];
      const int w = (int)(it % W);
      if (j == root) continue;
      const int sj = scc_of_class[j];
      uint32_t v = 0;
      const int e1 = par_ptr[j + 1];
      for (int e = par_ptr[j] + lane; e < e1; e += 4 * 32) {  // 4 parents per lane in flight
        int pc[4], pn[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int eu = e + 32 * u;
          pc[u] = eu < e1 ? par_class[eu] : -1;
          pn[u] = eu < e1 ? par_node[eu] : 0;
        }
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (pc[u] >= 0 && (sj < 0 || scc_of_class[pc[u]] != sj))
            v |= __ldcg(reach + (size_t)pc[u] * W + w) & sel[(size_t)pn[u] * W + w];
      }
      v = __reduce_or_sync(0xffffffffu, v);
      if (lane == 0) __stcg(reach + (size_t)j * W + w, v);
    }
    const int s0l = lvl_sptr[L];
    const int64_t nB = (int64_t)(lvl_sptr[L + 1] - s0l) * W;
    grid.sync();
    if (nB == 0) continue;
    // phase B: non-trivial SCCs, one block per (SCC, word)
    for (int64_t it = blockIdx.x; it < nB; it += gridDim.x) {
      const int s = lvl_scc[s0l + it / W];
      const int w = (int)(it % W);
      const int c0 = scc_class_ptr[s], n = scc_class_ptr[s + 1] - c0;
      if (n > kSmallScc) {
        decode_big_scc(n, c0, w, W, Bp, root, scc_class, node_slot, slot_jptr, slot_jloc, choice,
                       reach, settle, invalid);
        continue;
      }
      for (int l = wib; l < n; l += kDecodeWarps) {
        const int j = scc_class[c0 + l];
        const int c = choice[(size_t)j * Bp + 32 * w + lane];
        const int q = node_slot[c];
        uint64_t m = 0;
        if (q >= 0)
          for (int e = slot_jptr[q]; e < slot_jptr[q + 1]; ++e) m |= 1ull << slot_jloc[e];
        cm[l][lane] = m;
        if (lane == 0) rs0[l] = j == root ? 0xffffffffu : __ldcg(reach + (size_t)j * W + w);
      }
      __syncthreads();
      if (wib == 0) {
        uint64_t R = 0;
        for (int l = 0; l < n; ++l)
          if ((rs0[l] >> lane) & 1u) R |= 1ull << l;
        for (;;) {  // reach closure inside S for this seed
          const uint64_t o = R;
          for (int l = 0; l < n; ++l)
            if ((R >> l) & 1ull) R |= cm[l][lane];
          if (R == o) break;
        }
        const uint64_t all = n == 64 ? ~0ull : (1ull << n) - 1ull;
        uint64_t S = ~R & all;
        for (;;) {  // settle closure: a reached class settles once its children in S have
          const uint64_t o = S;
          for (int l = 0; l < n; ++l)
            if (!((S >> l) & 1ull) && (cm[l][lane] & ~S) == 0) S |= 1ull << l;
          if (S == o) break;
        }
        for (int l = 0; l < n; ++l) {
          const uint32_t word = __ballot_sync(0xffffffffu, (R >> l) & 1ull);
          if (lane == 0) __stcg(reach + (size_t)scc_class[c0 + l] * W + w, word);
        }
        const uint32_t bad = __ballot_sync(0xffffffffu, (R & ~S) != 0);
        if (lane == 0 && bad) atomicOr(invalid + w, bad);
      }
      __syncthreads();
    }
    grid.sync();
  }
  const int64_t gtid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (gtid < W) valid_out[gtid] = ~__ldcg(invalid + gtid);
}

static void coop_launch(const void* fn, int grid, void** args, cudaStream_t s) {
  SM_CUDA(cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(256), args, 0, s));
  SM_LAUNCH_CHECK();
}

void launch_decode(cudaStream_t s, const Shape& sh, const HostGraph& hg, const DevGraph& g,
                   const uint32_t* sel, const int32_t* choice, uint32_t* reach, uint32_t* settle,
                   uint32_t* invalid, uint32_t* valid_out, int32_t grid) {
  SM_CUDA(cudaMemsetAsync(invalid, 0, sizeof(uint32_t) * sh.W, s));
  SM_CUDA(cudaMemsetAsync(reach, 0, sizeof(uint32_t) * (size_t)sh.M * sh.W, s));
  SM_CUDA(cudaMemsetAsync(reach + (size_t)sh.root * sh.W, 0xff, sizeof(uint32_t) * sh.W, s));
  int W = sh.W, root = sh.root, L = hg.num_levels, Bp = sh.Bp;
  void* args[] = {&W, &root, &L, (void*)&g.lvl_cptr, (void*)&g.lvl_class, (void*)&g.lvl_sptr,
                  (void*)&g.lvl_scc, (void*)&g.par_ptr,
                  (void*)&g.par_node, (void*)&g.par_class, (void*)&g.class_ptr,
                  (void*)&g.scc_class_ptr, (void*)&g.scc_class, (void*)&g.scc_of_class,
                  (void*)&g.ent_ptr, (void*)&g.ent_i, (void*)&g.ent_j, (void*)&g.ent_node_ptr,
                  (void*)&g.ent_node, (void*)&g.node_slot, (void*)&g.slot_ptr,
                  (void*)&g.slot_node, (void*)&g.slot_jptr,
                  (void*)&g.slot_jloc, (void*)&sel, &Bp, (void*)&choice, &reach, &settle, &invalid,
                  &valid_out};
  coop_launch((const void*)k_decode_levels, grid, args, s);
}

int decode_grid(int device) {
  int per_sm = 0;
  SM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_decode_levels, 256, 0));
  const char* e = std::getenv("SMOOTHE_DECODE_BPS");  // blocks per SM (A/B)
  const int want = e ? std::max(1, std::atoi(e)) : 2;  // 2: measured best with the decode overlapped
  return std::max(1, std::min(per_sm, want)) * num_sms(device);
}

// Discrete linear cost per seed: part[blockIdx.x][b] = sum over the block's
// classes j with reach_j(b) of u[c_j(b)], fp64.
constexpr int kCostClasses = 64;

__global__ void k_decode_cost_linear(int M, int Bp, int W, const double* __restrict__ u,
                                     const int32_t* __restrict__ choice,
                                     const uint32_t* __restrict__ reach, double* __restrict__ part) {
  const int b = blockIdx.y * blockDim.x + threadIdx.x;
  if (b >= Bp) return;
  const int j0 = blockIdx.x * kCostClasses, j1 = min(M, j0 + kCostClasses);
  double acc = 0.0;
  for (int j = j0; j < j1; ++j)
    if ((reach[(size_t)j * W + (b >> 5)] >> (b & 31)) & 1u) acc += u[choice[(size_t)j * Bp + b]];
  part[(size_t)blockIdx.x * Bp + b] = acc;
}

void launch_decode_cost_linear(cudaStream_t s, const Shape& sh, const DevGraph&, const double* u,
                               const int32_t* choice, const uint32_t* reach, double* cost_part) {
  const int tpb = sh.Bp < 128 ? sh.Bp : 128;
  const dim3 grid((sh.M + kCostClasses - 1) / kCostClasses, sh.Bp / tpb);
  k_decode_cost_linear<<<grid, tpb, 0, s>>>(sh.M, sh.Bp, sh.W, u, choice, reach, cost_part);
  SM_LAUNCH_CHECK();
}

int decode_cost_rows(const Shape& sh) { return (sh.M + kCostClasses - 1) / kCostClasses; }

// s[k][b] = 1 iff class ec(k) is reached and chose k (the binary s of P99).
template <int LPR>
__global__ void __launch_bounds__(kBlock) k_decode_s(int M, int Bp, int W,
                                                     const int32_t* __restrict__ class_ptr,
                                                     const uint32_t* __restrict__ sel,
                                                     const uint32_t* __restrict__ reach,
                                                     float* __restrict__ s_out) {
  const RowGroup<LPR> rg;
  if (rg.row >= M) return;
  const int w = rg.s0 >> 5, sh = rg.s0 & 31;
  const uint32_t r = reach[(size_t)rg.row * W + w];
  for (int k = class_ptr[rg.row]; k < class_ptr[rg.row + 1]; ++k) {
    const uint32_t bits = (r & sel[(size_t)k * W + w]) >> sh;
    st4(s_out + (size_t)k * Bp + rg.s0,
        make_float4((float)(bits & 1u), (float)((bits >> 1) & 1u), (float)((bits >> 2) & 1u),
                    (float)((bits >> 3) & 1u)));
  }
}

void launch_decode_s(cudaStream_t s, const Shape& sh, const DevGraph& g, const uint32_t* sel,
                     const uint32_t* reach, float* s_out) {
  SM_DISPATCH_LPR(sh.Bp, {
    k_decode_s<LPR><<<row_grid(sh.M, sh.Bp, LPR), kBlock, 0, s>>>(sh.M, sh.Bp, sh.W, g.class_ptr,
                                                                 sel, reach, s_out);
  });
  SM_LAUNCH_CHECK();
}

// ---------------------------------------------------------------------------
// Keep-best (P297, readings S18, S20): the lowest (cost, step, global seed) of
// the valid samples.  best = {cost, step, seed, steps since improvement}.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_best_update(
    int B, int W, int root, const uint32_t* __restrict__ settle, const double* __restrict__ dcost,
    const double* __restrict__ dextra, int64_t seed_begin, int32_t* __restrict__ counter,
    double* __restrict__ best, int32_t* __restrict__ flag, double* __restrict__ cost_out,
    uint8_t* __restrict__ valid_out, double* __restrict__ trace, int trace_cap) {
  __shared__ double sc[256];
  __shared__ int sb[256];
  __shared__ int nvalid;
  if (threadIdx.x == 0) nvalid = 0;
  __syncthreads();
  double bc = INFINITY;
  int bb = 0x7fffffff, nv = 0;
  for (int b = threadIdx.x; b < B; b += blockDim.x) {
    const bool ok = (settle[(size_t)root * W + (b >> 5)] >> (b & 31)) & 1u;
    const double c = ok ? dcost[b] + (dextra ? dextra[b] : 0.0) : INFINITY;
    if (cost_out) cost_out[b] = c;
    if (valid_out) valid_out[b] = ok ? 1 : 0;
    nv += ok ? 1 : 0;
    if (c < bc) {
      bc = c;
      bb = b;
    }
  }
  if (trace) atomicAdd(&nvalid, nv);
  sc[threadIdx.x] = bc;
  sb[threadIdx.x] = bb;
  __syncthreads();
  for (int off = blockDim.x / 2; off > 0; off >>= 1) {
    if (threadIdx.x < off) {
      const double c2 = sc[threadIdx.x + off];
      const int b2 = sb[threadIdx.x + off];
      if (c2 < sc[threadIdx.x] || (c2 == sc[threadIdx.x] && b2 < sb[threadIdx.x])) {
        sc[threadIdx.x] = c2;
        sb[threadIdx.x] = b2;
      }
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    const int step = *counter;
    if (trace && step < trace_cap) {  // the sampled side of the step's record (k_loss)
      trace[4 * (size_t)step + 2] = sc[0];
      trace[4 * (size_t)step + 3] = (double)nvalid;
    }
    best[4] = sc[0];  // the step's candidate; k_best_commit decides once the step is complete
    best[5] = (double)(seed_begin + sb[0]);
  }
}

// Commit the step's candidate (cost, step, global seed) after the whole step
// ran (main stream): lexicographic keep-best (reading S20), patience counter
// best[3], step counter.  A step aborted by a full version pool (its update
// was skipped, it will be repeated) commits nothing and is counted in
// abort_flag[1]; abort_flag[2] tracks the most pool rows any chunk took.
__global__ void k_best_commit(int32_t* __restrict__ counter, double* __restrict__ best,
                              int32_t* __restrict__ flag, int32_t* __restrict__ abort_flag,
                              const int32_t* __restrict__ pool_n, int nchunk) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  if (abort_flag) {
    for (int c = 0; c < nchunk; ++c) abort_flag[2] = max(abort_flag[2], pool_n[c]);
    if (abort_flag[0]) {
      *flag = 0;
      abort_flag[1] += 1;
      return;
    }
  }
  const int step = *counter;
  if (best[4] < best[0]) {
    best[0] = best[4];
    best[1] = (double)step;
    best[2] = best[5];
    best[3] = 0.0;
    *flag = 1;
  } else {
    best[3] += 1.0;
    *flag = 0;
  }
  *counter = step + 1;
}

void launch_best_commit(cudaStream_t s, int32_t* counter, double* best, int32_t* flag,
                        int32_t* abort_flag, const int32_t* pool_n, int nchunk) {
  k_best_commit<<<1, 32, 0, s>>>(counter, best, flag, abort_flag, pool_n, nchunk);
  SM_LAUNCH_CHECK();
}

void launch_best_update(cudaStream_t s, const Shape& sh, const uint32_t* settle,
                        const double* dcost_lin, const double* dcost_extra, int64_t seed_begin,
                        const int32_t* step_counter, double* best, int32_t* best_flag,
                        double* valid_cost_out, uint8_t* valid_out, double* trace, int trace_cap) {
  k_best_update<<<1, 256, 0, s>>>(sh.B, sh.W, sh.root, settle, dcost_lin, dcost_extra, seed_begin,
                                  const_cast<int32_t*>(step_counter), best, best_flag,
                                  valid_cost_out, valid_out, trace, trace_cap);
  SM_LAUNCH_CHECK();
}

__global__ void k_best_snapshot(int M, int Bp, int W, const int32_t* __restrict__ choice,
                                const uint32_t* __restrict__ reach, const double* __restrict__ best,
                                const int32_t* __restrict__ flag, int64_t seed_begin,
                                int32_t* __restrict__ best_choice) {
  if (*flag == 0) return;
  const int b = (int)((int64_t)best[2] - seed_begin);
  for (int j = blockIdx.x * blockDim.x + threadIdx.x; j < M; j += gridDim.x * blockDim.x) {
    const bool r = (reach[(size_t)j * W + (b >> 5)] >> (b & 31)) & 1u;
    best_choice[j] = r ? choice[(size_t)j * Bp + b] : -1;
  }
}

void launch_best_snapshot(cudaStream_t s, const Shape& sh, const int32_t* choice,
                          const uint32_t* reach, const double* best, const int32_t* best_flag,
                          int64_t seed_begin, int32_t* best_choice) {
  const int grid = std::min((sh.M + 255) / 256, 148 * 4);
  k_best_snapshot<<<grid, 256, 0, s>>>(sh.M, sh.Bp, sh.W, choice, reach, best, best_flag,
                                       seed_begin, best_choice);
  SM_LAUNCH_CHECK();
}

}  // namespace smoothe
