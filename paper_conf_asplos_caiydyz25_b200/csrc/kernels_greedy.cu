// Greedy worklist extraction (the paper's "heuristic method")
// on the GPU (sm_100a): a comparator for SmoothE's extractions and an optional
// warm start of theta.
//
// The worklist computes the least fixpoint of
//   key(m_j) = min_{n_i in m_j} ( u_i + sum_{c in ch_i} cost(c),  1 + max_{c in ch_i} height(c),  i )
// (lexicographic; reading G1: costs decide as in the paper, then the shorter
// derivation, then the lowest id; height 0 for a leaf).  The fixpoint does
// not depend on the order the worklist processes e-nodes, so instead of a
// queue the kernel visits the condensation of the e-class graph bottom-up:
//  * level by level from the deepest (levels from the loader: longest path
//    from the root's component; every child of a class in a trivial component
//    sits at a deeper level, so its key is final after one evaluation: one
//    warp per class, lanes over its e-nodes);
//  * a non-trivial component S is one block job: keys start at infinity and
//    the block re-evaluates S's classes until a pass changes nothing
//    (Bellman-Ford inside S; keys only decrease, so stale reads inside a pass
//    only delay convergence).
// One grid barrier per phase and level.  Then the extraction is read top-down
// from the root: a frontier walk over the selected e-nodes' child classes
// (atomicExch marks; the reached set is unique, the frontier order is not
// used), and f_b(s) = sum over reached classes of u of the selected e-node is
// reduced in a fixed order (reading S19).
#include <cooperative_groups.h>

#include "kcommon.cuh"

namespace smoothe {

namespace cg = cooperative_groups;

struct GKey {
  double c;
  int h, id;
};
__device__ __forceinline__ bool key_less(const GKey& a, const GKey& b) {
  return a.c < b.c || (a.c == b.c && (a.h < b.h || (a.h == b.h && a.id < b.id)));
}

// best (aggregated cost, height, id) over the e-nodes of class j, warp-wide
__device__ GKey class_key(int j, const int32_t* __restrict__ class_ptr,
                          const int32_t* __restrict__ child_ptr,
                          const int32_t* __restrict__ child_class, const double* __restrict__ u,
                          const double* cost, const int32_t* height) {
  const int lane = threadIdx.x & 31;
  GKey best{INFINITY, INT32_MAX, INT32_MAX};
  for (int k = class_ptr[j] + lane; k < class_ptr[j + 1]; k += 32) {
    double agg = u[k];
    int h = 0;
    for (int e = child_ptr[k]; e < child_ptr[k + 1]; ++e) {
      const int c = child_class[e];
      agg += __ldcg(cost + c);
      h = max(h, __ldcg(height + c) + 1);
    }
    const GKey kk{agg, h, k};
    if (agg < INFINITY && key_less(kk, best)) best = kk;
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    GKey o;
    o.c = __shfl_xor_sync(0xffffffffu, best.c, off);
    o.h = __shfl_xor_sync(0xffffffffu, best.h, off);
    o.id = __shfl_xor_sync(0xffffffffu, best.id, off);
    if (key_less(o, best)) best = o;
  }
  return best;
}

constexpr int kGreedyWarps = 8;

__global__ void __launch_bounds__(256) k_greedy(
    int M, int root, int num_levels, const int32_t* __restrict__ lvl_cptr,
    const int32_t* __restrict__ lvl_class, const int32_t* __restrict__ lvl_sptr,
    const int32_t* __restrict__ lvl_scc, const int32_t* __restrict__ scc_of_class,
    const int32_t* __restrict__ scc_class_ptr, const int32_t* __restrict__ scc_class,
    const int32_t* __restrict__ class_ptr, const int32_t* __restrict__ child_ptr,
    const int32_t* __restrict__ child_class, const double* __restrict__ u, double* cost,
    int32_t* height, int32_t* sel, int32_t* reach, int32_t* frontier, int32_t* counts,
    double* part, int32_t* npart, int32_t* choice_out, double* result) {
  cg::grid_group grid = cg::this_grid();
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int64_t gwarp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  // bottom-up keys, deepest level first
  for (int L = num_levels - 1; L >= 0; --L) {
    for (int64_t it = gwarp; it < lvl_cptr[L + 1] - lvl_cptr[L]; it += nwarps) {
      const int j = lvl_class[lvl_cptr[L] + it];
      if (scc_of_class[j] >= 0) continue;
      const GKey k = class_key(j, class_ptr, child_ptr, child_class, u, cost, height);
      if (lane == 0) {
        __stcg(cost + j, k.c);
        __stcg(height + j, k.c < INFINITY ? k.h : INT32_MAX - 1);
        __stcg(sel + j, k.c < INFINITY ? k.id : -1);
      }
    }
    grid.sync();
    const int s0 = lvl_sptr[L], ns = lvl_sptr[L + 1] - s0;
    if (ns == 0) continue;
    for (int it = blockIdx.x; it < ns; it += gridDim.x) {
      const int s = lvl_scc[s0 + it];
      const int c0 = scc_class_ptr[s], n = scc_class_ptr[s + 1] - c0;
      for (int l = threadIdx.x; l < n; l += blockDim.x) {  // keys start at infinity
        const int j = scc_class[c0 + l];
        __stcg(cost + j, (double)INFINITY);
        __stcg(height + j, INT32_MAX - 1);
        __stcg(sel + j, -1);
      }
      __syncthreads();
      for (;;) {
        int chg = 0;
        for (int l = wib; l < n; l += kGreedyWarps) {
          const int j = scc_class[c0 + l];
          const GKey k = class_key(j, class_ptr, child_ptr, child_class, u, cost, height);
          const GKey cur{__ldcg(cost + j), __ldcg(height + j), __ldcg(sel + j) < 0 ? INT32_MAX : __ldcg(sel + j)};
          if (k.c < INFINITY && key_less(k, cur)) {
            if (lane == 0) {
              __stcg(cost + j, k.c);
              __stcg(height + j, k.h);
              __stcg(sel + j, k.id);
            }
            chg = 1;
          }
        }
        if (!__syncthreads_or(chg)) break;
      }
    }
    grid.sync();
  }
  // top-down: classes reached from the root through the selected e-nodes
  const int64_t gtid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t nthreads = (int64_t)gridDim.x * blockDim.x;
  for (int64_t j = gtid; j < M; j += nthreads) reach[j] = 0;
  if (gtid == 0) {
    counts[0] = sel[root] >= 0 ? 1 : 0;
    counts[1] = 0;
    counts[2] = 0;
    frontier[0] = root;
  }
  grid.sync();
  if (gtid == 0 && counts[0]) reach[root] = 1;
  int32_t* cur = frontier;
  int32_t* nxt = frontier + M;
  for (int r = 0;; ++r) {
    const int n = __ldcg(counts + (r % 3));
    if (n == 0) break;
    if (gtid == 0) counts[(r + 2) % 3] = 0;  // the round after next
    for (int64_t it = gwarp; it < n; it += nwarps) {
      const int j = __ldcg(cur + it);
      const int k = __ldcg(sel + j);
      for (int e = child_ptr[k] + lane; e < child_ptr[k + 1]; e += 32) {
        const int c = child_class[e];
        if (atomicExch(reach + c, 1) == 0) nxt[atomicAdd(counts + ((r + 1) % 3), 1)] = c;
      }
    }
    grid.sync();
    int32_t* t = cur;
    cur = nxt;
    nxt = t;
  }
  // f_b(s) = sum of u over the reached classes' selections; fixed order:
  // block b sums classes [b chunk, (b+1) chunk) in a fixed tree, block 0 adds
  // the block sums in block order
  __shared__ double red[256];
  __shared__ int redn[256];
  const int64_t chunk = (M + gridDim.x - 1) / gridDim.x;
  const int64_t j0 = blockIdx.x * chunk, j1 = min((int64_t)M, j0 + chunk);
  double acc = 0.0;
  int cnt = 0;
  for (int64_t j = j0 + threadIdx.x; j < j1; j += blockDim.x) {
    const bool r = __ldcg(reach + j) != 0;
    const int k = __ldcg(sel + j);
    if (r) {
      acc += u[k];
      ++cnt;
    }
    choice_out[j] = r ? k : -1;
  }
  red[threadIdx.x] = acc;
  redn[threadIdx.x] = cnt;
  __syncthreads();
  for (int o = blockDim.x / 2; o > 0; o >>= 1) {
    if (threadIdx.x < o) {
      red[threadIdx.x] += red[threadIdx.x + o];
      redn[threadIdx.x] += redn[threadIdx.x + o];
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    part[blockIdx.x] = red[0];
    npart[blockIdx.x] = redn[0];
  }
  grid.sync();
  if (gtid == 0) {
    double s = 0.0;
    int64_t c = 0;
    for (int b = 0; b < (int)gridDim.x; ++b) {
      s += __ldcg(part + b);
      c += __ldcg(npart + b);
    }
    const bool ok = __ldcg(sel + root) >= 0;
    result[0] = ok ? s : INFINITY;
    result[1] = __ldcg(cost + root);
    result[2] = ok ? 1.0 : 0.0;
    result[3] = (double)c;
  }
}

int greedy_grid(int device) {
  int per_sm = 0;
  SM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_greedy, 256, 0));
  return std::max(1, std::min(per_sm, 4)) * num_sms(device);
}

void launch_greedy(cudaStream_t s, const HostGraph& hg, const DevGraph& g, int grid,
                   const double* u, double* cost, int32_t* height, int32_t* sel, int32_t* reach,
                   int32_t* frontier, int32_t* counts, double* part, int32_t* npart,
                   int32_t* choice_out, double* result) {
  int M = hg.M, root = hg.root, L = hg.num_levels;
  void* args[] = {&M, &root, &L, (void*)&g.lvl_cptr, (void*)&g.lvl_class, (void*)&g.lvl_sptr,
                  (void*)&g.lvl_scc, (void*)&g.scc_of_class, (void*)&g.scc_class_ptr,
                  (void*)&g.scc_class, (void*)&g.class_ptr, (void*)&g.child_ptr,
                  (void*)&g.child_class, (void*)&u, &cost, &height, &sel, &reach, &frontier,
                  &counts, &part, &npart, &choice_out, &result};
  SM_CUDA(cudaLaunchCooperativeKernel((const void*)k_greedy, dim3(grid), dim3(256), args, 0, s));
  SM_LAUNCH_CHECK();
}

// theta_k += bias for the selected e-node k of every class with choice >= 0,
// every seed column (warm start from an extraction, e.g. the greedy one)
__global__ void k_warm_start(int M, int Bp, const int32_t* __restrict__ choice, float bias,
                             float* __restrict__ theta) {
  const int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (idx >= (int64_t)M * Bp) return;
  const int j = (int)(idx / Bp), b = (int)(idx % Bp);
  const int k = choice[j];
  if (k >= 0) theta[(size_t)k * Bp + b] += bias;
}

void launch_warm_start(cudaStream_t s, int M, int Bp, const int32_t* choice, float bias,
                       float* theta) {
  const int64_t n = (int64_t)M * Bp;
  k_warm_start<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(M, Bp, choice, bias, theta);
  SM_LAUNCH_CHECK();
}

}  // namespace smoothe
