// Internal declarations of libsmoothe (not part of the ABI).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <string>
#include <vector>

#include "../../include/smoothe.h"

namespace smoothe {

// ---------------------------------------------------------------------------
// Errors
// ---------------------------------------------------------------------------
void set_error(const std::string& msg);

struct Failure {
  smoothe_status status;
  std::string msg;
};

#define SM_CUDA(call)                                                                  \
  do {                                                                                 \
    cudaError_t _e = (call);                                                           \
    if (_e != cudaSuccess)                                                             \
      throw ::smoothe::Failure{SMOOTHE_E_CUDA, std::string(#call) + ": " +             \
                                                    cudaGetErrorString(_e)};           \
  } while (0)

#define SM_REQUIRE(cond, status, msg)                                                  \
  do {                                                                                 \
    if (!(cond)) throw ::smoothe::Failure{status, msg};                                \
  } while (0)

// ---------------------------------------------------------------------------
// E-graph: host analysis (egraph.cpp) and its device mirror
// ---------------------------------------------------------------------------
constexpr int32_t kBigClass = 32;  // e-nodes above which a class gets a block (kernels_step.cu)
// Components up to this many classes keep Abar / e^Abar in shared memory and
// their decode closures in 64-bit registers; larger ones take the global-memory
// paths (batched fp64 GEMMs for the penalty, block-wide fixpoints for decode).
constexpr int32_t kSmallScc = 64;
constexpr int32_t kWChunk = 64;  // class edges per frozen-sweep work item

// Max batches of 4 children per reverse-sweep item: 0 = from the graph's size
// (HostGraph::rev_chunk: small graphs need short items to fill the GPU, large ones pay
// for every split); a positive value fixes it (A/B experiments).
#ifndef SMOOTHE_REV_CHUNK
#define SMOOTHE_REV_CHUNK 0
#endif

struct HostGraph {
  int32_t M = 0, N = 0, root = 0;
  int64_t E = 0;
  std::vector<int32_t> class_ptr;                  // [M+1]
  std::vector<int32_t> ec;                         // [N]
  std::vector<int32_t> child_ptr, child_class;     // CSR: ch_i, sorted, deduplicated
  std::vector<int32_t> par_ptr, par_node, par_class;// CSC: pa_j sorted by node id, ec(node)
  // non-trivial strongly connected components (size > 1 or self-loop)
  int32_t num_scc = 0, scc_classes = 0, scc_max = 0;
  std::vector<int32_t> scc_of_class;               // [M] component id or -1
  std::vector<int32_t> scc_class_ptr, scc_class;   // members per component, by class id
  std::vector<int32_t> scc_local;                  // [M] position inside its component
  // Abar entries: unique (i_local, j_local) per component and their e-nodes k
  // (k in m_i, j in ch_k), SURVEY.md 8(a) a5.
  std::vector<int32_t> ent_ptr;                    // [num_scc+1]
  std::vector<int32_t> ent_i, ent_j;               // local indices
  std::vector<int32_t> ent_node_ptr, ent_node;     // contributing e-nodes
  // penalty slots: every e-node of a component's classes, with its children
  // inside the component (gradient scatter of App. B).
  std::vector<int32_t> slot_ptr;                   // [num_scc+1]
  std::vector<int32_t> slot_node, slot_iloc;       // [num_slots]
  std::vector<int32_t> slot_jptr, slot_jloc;       // children in the component (local)
  std::vector<int32_t> node_slot;                  // [N] slot id or -1
  // components with more than kSmallScc classes and, per component, the number
  // of squarings s of its matrix exponential: the row sums of Abar are
  // sum_{k in m_i} cp_k |ch_k cap S| <= max_k |ch_k cap S| (cp sums to 1 over
  // a class), so 2^-s Abar has inf-norm <= 1/2 with s = ceil(log2 max) + 1
  std::vector<int32_t> big_scc, big_scc_sq;
  int32_t K_auto = 0, max_class_size = 0, max_in_degree = 0;
  // Sweep layouts padded to multiples of 4 entries per list (aligned vector
  // index loads, 4 row gathers in flight):
  //   pad_child_ptr [N+1], pad_child [.]   child classes of e-node i; padding = root
  //                                        (g_q of the root is 0: inert, no mask)
  //   pad_par_ptr [M+1],  pad_par [.][2]   (parent e-node, its class) of class j;
  //                                        padding = (N, root): row N of cp is 0: p = 0
  // (Padding with masked copies of a list's first entry instead measured no
  // faster: the shared inert rows stay L1-resident.)
  std::vector<int32_t> pad_child_ptr, pad_child, pad_par_ptr, pad_par;
  std::vector<int32_t> pad_batch_node;  // [pad_child_ptr[N] / 4] e-node owning each batch of 4
  // [pad_child_ptr[N]] index of (ec(i), child) in cls_child for each padded
  // child slot of e-node i; -1 for padding (frozen-sweep matrix W, section 7)
  std::vector<int32_t> pad_cedge;
  // per class edge (i, j): its class i and the e-nodes k of m_i with j in ch_k
  // (ascending), CSR -- the rows of W are built one class edge at a time
  std::vector<int32_t> cedge_class, cedge_ptr, cedge_node;
  // frozen-sweep work items [n][4] = (class, first edge, end edge, partial
  // slot or -1): a class's edges in chunks of <= kWChunk (every class has at
  // least one item; the first carries the S update), and the classes with
  // several chunks, whose partial rows k_wcombine adds in item order
  std::vector<int32_t> witem, wmulti, wmulti_ptr;
  int32_t w_num_slots = 0;
  // classes with more than kBigClass e-nodes, largest first: the per-class
  // kernels (softmax, cost, update) give each a whole block
  std::vector<int32_t> big_class;
  std::vector<int32_t> dmin;  // [M] BFS depth from the root (INT32_MAX: unreachable)
  // class -> distinct child classes of its e-nodes (CSR, sorted): the forward
  // sweep marks these dirty for the next sweep when the class's q row changes
  std::vector<int32_t> cls_child_ptr, cls_child;
  std::vector<int32_t> hmax;  // [M] longest walk from the class (INT32_MAX: reaches a cycle)
  // Reverse-sweep work items, [n][8] = (class j, first batch, end batch, info,
  // first e-node, last e-node, dmin_j, hmax_j): a class's batches split into runs of <= rev_chunk cut at
  // e-node boundaries, an e-node with more batches cut into "pieces" of its own.
  // info = -1: the class's only item; else (slot << 1) | piece, slot = its
  // partial-sum row (the class's last item to finish combines them in order).
  // Without the split one warp walks the largest class serially and sets the
  // sweep time (C3: one e-node with 1507 children, 4x the rest of the sweep).
  std::vector<int32_t> rev_item, rev_class_item_ptr;  // rev_class_item_ptr [M+1]
  int32_t rev_num_slots = 0, rev_chunk = 0;
  // Decode schedule: levels of the SCC condensation reachable from the root
  // (level = longest path from the root's component).  Level L holds the
  // classes lvl_class[lvl_cptr[L] .. lvl_cptr[L+1]) and the non-trivial SCCs
  // lvl_scc[lvl_sptr[L] .. lvl_sptr[L+1]).
  int32_t num_levels = 0;
  std::vector<int32_t> lvl_cptr, lvl_class, lvl_sptr, lvl_scc;
};

void build_host_graph(int32_t M, int32_t N, const int32_t* class_ptr, const int64_t* child_ptr,
                      const int32_t* child_class, int32_t root, HostGraph& g);

struct DevGraph {
  int32_t *class_ptr = nullptr, *child_ptr = nullptr, *child_class = nullptr;
  int32_t *par_ptr = nullptr, *par_node = nullptr, *par_class = nullptr;
  int32_t *scc_class_ptr = nullptr, *scc_class = nullptr, *scc_of_class = nullptr, *ent_ptr = nullptr, *ent_i = nullptr, *ent_j = nullptr;
  int32_t *ent_node_ptr = nullptr, *ent_node = nullptr;
  int32_t *slot_ptr = nullptr, *slot_node = nullptr, *slot_iloc = nullptr;
  int32_t *slot_jptr = nullptr, *slot_jloc = nullptr, *node_slot = nullptr;
  int32_t *pad_child_ptr = nullptr, *pad_child = nullptr, *pad_par_ptr = nullptr, *pad_par = nullptr;
  int32_t* pad_batch_node = nullptr;
  int32_t* pad_cedge = nullptr;
  int32_t *cedge_class = nullptr, *cedge_ptr = nullptr, *cedge_node = nullptr;
  int64_t num_cedge = 0;
  int32_t *witem = nullptr, *wmulti = nullptr, *wmulti_ptr = nullptr;
  int32_t num_witems = 0, num_wmulti = 0, w_num_slots = 0;
  int32_t* big_class = nullptr;
  int32_t* dmin = nullptr;
  int32_t *cls_child_ptr = nullptr, *cls_child = nullptr;
  int32_t num_big = 0;
  int32_t *rev_item = nullptr, *rev_class_item_ptr = nullptr;
  int32_t num_rev_items = 0, rev_num_slots = 0;
  int32_t *lvl_cptr = nullptr, *lvl_class = nullptr, *lvl_sptr = nullptr, *lvl_scc = nullptr;
  int64_t bytes = 0;
};

}  // namespace smoothe

struct smoothe_egraph {
  smoothe::HostGraph host;
  smoothe::DevGraph dev;
  std::vector<void*> owned;  // device allocations (one arena)
  int device = -1;
  int refcount = 1;  // the handle itself + one per live run
  bool freed = false;
};

namespace smoothe {

// ---------------------------------------------------------------------------
// Kernel launch interface (kernels.cu).  Per-seed rows have Bp floats; Bp is
// num_seeds rounded up to 32, 64 or a multiple of 128.
// ---------------------------------------------------------------------------
struct Shape {
  int32_t M, N, root, B, Bp, W;  // W = Bp / 32 bitmask words per row
};

struct Agg {
  float wI, wC;  // independent / correlated weights
};

void launch_theta_init(cudaStream_t s, const Shape& sh, uint64_t key, int64_t seed_begin,
                       float* theta, float* m, float* v);
void launch_softmax_argmax(cudaStream_t s, const Shape& sh, const DevGraph& g, const float* theta,
                           float* cp, int32_t* choice, uint32_t* sel);
// Per-run sweep state (kernels_sweep.cu, "change propagation").  Versions
// live in pools: per seed chunk c (wc = min(Bp, 128) seeds,
// nchunk = Bp / wc) a pool of cap rows [cap][wc] for each of q, pi, am, rows
// [0, M) holding version 0 (q^0 = e_root, pi = 1, am = first parent); a class
// recomputed in forward sweep t takes the next row and is listed in
// list[c][t] with its previous row.  A step whose chunk needs more than cap
// rows is aborted and repeated after the host grows the pools.
struct SweepState {
  float* qpool = nullptr;     // [nchunk][cap][wc]
  float* pipool = nullptr;    // [nchunk][cap][wc] (NULL for the correlated aggregator)
  int32_t* apool = nullptr;   // [nchunk][cap][wc]
  int64_t cap = 0;            // rows per chunk pool
  int nchunk = 1, wc = 0;
  int32_t* pool_n = nullptr;  // [nchunk] rows taken this step (beyond cap: overflow)
  int32_t* lastrow = nullptr; // [nchunk][M] current row of each class (during the forward)
  int4* list = nullptr;       // [nchunk][K+1][M] (class, previous row, new row, -) of sweep t
  int32_t* list_n = nullptr;  // [nchunk][K+2] list lengths
  int32_t* abort_flag = nullptr;  // [0] this step overflowed a pool, [1] steps aborted, [2] max rows taken
  float* qbuf[2] = {nullptr, nullptr};  // complete q^t rows, buffer t & 1
  float* cur_pi = nullptr;    // [M][Bp] pi^t of every class during reverse sweep t
  int32_t* cur_am = nullptr;  // [M][Bp]
  int K = 0, num_sms = 148;
  int32_t* dirty[2] = {nullptr, nullptr};  // [M] stamp t: recompute in sweep t
  int32_t* chg[2] = {nullptr, nullptr};    // [M] stamp t: q row changed in sweep t
  bool all = false;  // recompute every class in every sweep (env SMOOTHE_SWEEP_ALL=1; A/B and tests)
  // Frozen reverse sweeps: W [num_cedge][Bp] class-level
  // reverse coefficients of the K-state, S [M][Bp] the sums of g_q over a
  // seed's frozen sweeps, the K-state rows kq / kpi / kam, wm [Bp] 1 while the
  // seed's rows still equal the K-state (env SMOOTHE_REV_W=0 disables).
  bool wmode = false;
  // "until convergence" (smoothe_options.converge, reading S1b): lastchg[s] =
  // the last forward sweep that changed a q row of seed s; the seed's step is
  // sweeps 1..lastchg+1 (its reverse skips the later, frozen sweeps)
  bool converge = false;
  int32_t* lastchg = nullptr;
  float *W = nullptr, *S = nullptr, *kq = nullptr, *kpi = nullptr, *wpart = nullptr;
  int32_t *kam = nullptr, *wm = nullptr;
  // live[t] [K + 2], zeroed per step: some g_q^t value is non-zero (set by the
  // reverse-phase writers; sweeps whose input is all zero are skipped).
  // NULL with SMOOTHE_GLIVE=0.
  int32_t* glive = nullptr;
  // gstamp[t & 1][row][chunk] = t: sweep t + 1 wrote a non-zero g_q^t row
  // (by parity: sweep t reads t & 1 and writes (t - 1) & 1; never reset, a
  // stale match only costs a read).  NULL with SMOOTHE_GLIVE=0.
  int32_t* gstamp = nullptr;
  // fchg[t] [K + 2], zeroed per step: some q row changed (bitwise) in forward
  // sweep t; fchg[0] = the last such sweep.  Once a sweep changes nothing, every later sweep is the identity
  // (no class is dirty, no row to copy forward): in the captured step of a
  // large graph, forward sweep t is a conditional node on fchg[t - 1].  NULL
  // with SMOOTHE_FSKIP=0.
  int32_t* fchg = nullptr;
  // k_wspmv as one wave of persistent row groups striding over the work items
  // (default for >= 100k items; SMOOTHE_WSPMV_PERSIST=0 / 1 forces)
  bool wpersist = false;
  // [w_num_slots][nchunk] arrival counters of the long classes' chunks (the
  // last chunk combines; zero between launches).  NULL: k_wcombine
  // (SMOOTHE_WFUSE=0)
  int32_t* wcnt = nullptr;
  // captured step of a large graph (>= 100k reverse items): conditional nodes
  // cost ~15 us each, so sweeps are gated in blocks: forward sweeps
  // [t, t + fblock) by one IF on fchg[t - 1] (0: no gating), reverse sweeps
  // (t - rblock, t] by one IF on live[t]; the plain reverse kernel runs as one
  // wave of persistent warps (an all-frozen sweep then costs a few us) unless
  // plain_if, which puts it under an IF on "some seed unfrozen"
  // (SMOOTHE_FBLOCK, SMOOTHE_RBLOCK, SMOOTHE_PLAIN_IF)
  bool big_sched = false;  // the gated schedule below (>= 100k reverse items; SMOOTHE_BIG_SCHED)
  int fblock = 0, rblock = 8;
  bool plain_if = false;
  // reverse blocks as a switch node whose k_wspmv-only body skips the
  // transitions and the plain kernel above the last changing forward sweep
  // (SMOOTHE_RSWITCH=0: the plain IF)
  bool rswitch = true;
};
// Reset the per-step sweep state (stamps, q buffers = q^0).
void launch_sweep_reset(cudaStream_t s, const Shape& sh, const SweepState& st);
// version 0 of every class in rows [0, M) of each chunk's pool (run creation, pool growth)
void launch_pool_version0(cudaStream_t s, const Shape& sh, const DevGraph& g, const SweepState& st);
// Forward sweep t: q^t (qbuf[t & 1]) from q^{t-1} and versions t of the stacks.
void launch_sweep_forward(cudaStream_t s, const Shape& sh, const DevGraph& g, Agg a, int t,
                          const SweepState& st, const float* cp);
void launch_cost_linear(cudaStream_t s, const Shape& sh, const DevGraph& g, const float* u,
                        const float* cp, const float* qK, float* gcp, float* gqK, float* f_part,
                        float* p_out, int32_t nblocks_hint);
void launch_cost_gp(cudaStream_t s, const Shape& sh, const DevGraph& g, const float* gp,
                    const float* cp, const float* qK, float* gcp, float* gqK);
// p = cp * q^K[ec]; with u != NULL also f_part = per-block partial sums of u^T p
void launch_materialize_p_f(cudaStream_t s, const Shape& sh, const DevGraph& g, const float* u,
                            const float* cp, const float* qK, float* p, float* f_part);
// quadratic cost over symmetric neighbour lists; u may be NULL (pair terms only)
void launch_quadratic(cudaStream_t s, const Shape& sh, const int32_t* qptr, const int32_t* qnbr,
                      const float* qw, const float* u, const float* p, float* gp, float* f_part);
// deterministic fp64 column sums; scratch holds 128 x Bp doubles
void launch_reduce_rows_f64(cudaStream_t s, const float* part, int32_t nrows, int32_t Bp,
                            double* out, double scale, double* scratch);
void launch_reduce_rows_f64d(cudaStream_t s, const double* part, int32_t nrows, int32_t Bp,
                             double* out, double* scratch);
// t: sweep index (items of classes with dmin > t - 1 are skipped: q^{t-1} = 0
// there, so they contribute nothing to g_cp and no active class reads their
// g_q^{t-1})
// Bring cur_q / cur_pi / cur_am to reverse sweep t (before each reverse sweep).
void launch_rev_transition(cudaStream_t s, const Shape& sh, const DevGraph& g, int t, int K,
                           const SweepState& st);
// Reverse sweep t over the rows q_prev (q^{t-1}), pi / am (pi^t, am^t); seeds
// with wm[s] != 0 are left to the frozen-sweep kernels (wm may be NULL).
void launch_sweep_reverse(cudaStream_t s, const Shape& sh, const DevGraph& g, Agg a, int t, int K,
                          const float* q_prev, const float* pi, const int32_t* am,
                          const int32_t* wm, const float* cp, const float* gq, float* gcp,
                          float* gq_prev, bool write_gq_prev, float* rev_part, int32_t* rev_cnt,
                          const int32_t* lastchg = nullptr, int32_t* cursor = nullptr,
                          const int32_t* live_in = nullptr, int32_t* live_out = nullptr,
                          int32_t* gstamp = nullptr, bool persist = false);
// sets the conditional handle to 1 iff some seed is not frozen (wm[s] == 0)
void launch_any_unfrozen(cudaStream_t s, const Shape& sh, const int32_t* wm,
                         cudaGraphConditionalHandle h);
// sets the conditional handle to 1 iff *flag != 0
void launch_flag_if(cudaStream_t s, const int32_t* flag, cudaGraphConditionalHandle h);
void launch_rev_switch(cudaStream_t s, const int32_t* live, const int32_t* fchg, int t_low,
                       cudaGraphConditionalHandle h);
// W from the K-state rows (before reverse sweep K)
void launch_wbuild(cudaStream_t s, const Shape& sh, const DevGraph& g, Agg a,
                   const SweepState& st, const float* cp);
// frozen reverse sweep t for the seeds with wm set: g_q^{t-1} = W g_q^t, S += g_q^t
void launch_wspmv(cudaStream_t s, const Shape& sh, const DevGraph& g, int t,
                  const SweepState& st, const float* gq, float* gq_prev, int64_t* frozen_count);
// profiling: live units of frozen sweep t into out[0..2] (kernels_sweep.cu)
void launch_count_live(cudaStream_t s, const Shape& sh, const DevGraph& g, int t,
                       const SweepState& st, int64_t* out);
// converge mode: lastchg[s] from the forward's version lists (per seed, the
// last sweep whose recomputed q rows differ from their previous versions)
void launch_last_change(cudaStream_t s, const Shape& sh, const SweepState& st);
void launch_notears(cudaStream_t s, const Shape& sh, const HostGraph& hg, const DevGraph& g,
                    int32_t G, double lambda, const float* cp, double* h_part, float* pen,
                    double* big_scratch, int big_groups_per_batch);
// bytes of fp64 scratch the large-component path needs, and how many penalty
// groups it processes per batch (0 when every component is small)
size_t notears_big_scratch(const HostGraph& hg, int ngroups, int* groups_per_batch);
void launch_update(cudaStream_t s, const Shape& sh, const DevGraph& g, int32_t G, const float* cp,
                   const float* gcp, const float* pen, float* theta, float* m, float* v,
                   const double* step_scalars, int32_t optimizer, float lr, float beta1,
                   float beta2, float eps, float* grad_theta_out, float* grad_cp_out,
                   const int32_t* abort_flag);
void launch_step_prologue(cudaStream_t s, int32_t* step_counter, double* step_scalars,
                          double beta1, double beta2, const int32_t* unused);
void launch_fill_rows(cudaStream_t s, float* base, int64_t stride, int count, int Bp, float value);
void launch_loss(cudaStream_t s, int B, int G, int ngroups, double lambda, const double* f,
                 const double* fextra, const double* h, double* ftot, double* loss,
                 const double* scal, double* trace, int trace_cap);
// reached sets and validity masks (kernels_decode.cu); valid_out[W]
void launch_decode(cudaStream_t s, const Shape& sh, const HostGraph& hg, const DevGraph& g,
                   const uint32_t* sel, const int32_t* choice, uint32_t* reach, uint32_t* settle,
                   uint32_t* invalid, uint32_t* valid_out, int32_t grid);
void launch_decode_cost_linear(cudaStream_t s, const Shape& sh, const DevGraph& g,
                               const double* u, const int32_t* choice, const uint32_t* reach,
                               double* cost_part);
void launch_decode_s(cudaStream_t s, const Shape& sh, const DevGraph& g, const uint32_t* sel,
                     const uint32_t* reach, float* s_out);
int decode_grid(int device);
// greedy worklist extraction (kernels_greedy.cu)
int greedy_grid(int device);
void launch_greedy(cudaStream_t s, const HostGraph& hg, const DevGraph& g, int grid,
                   const double* u, double* cost, int32_t* height, int32_t* sel, int32_t* reach,
                   int32_t* frontier, int32_t* counts, double* part, int32_t* npart,
                   int32_t* choice_out, double* result);
void launch_warm_start(cudaStream_t s, int M, int Bp, const int32_t* choice, float bias,
                       float* theta);
int decode_cost_rows(const Shape& sh);
// after the step (main stream): keep-best commit of the step's candidate (best[4..5])
void launch_best_commit(cudaStream_t s, int32_t* counter, double* best, int32_t* flag,
                        int32_t* abort_flag, const int32_t* pool_n, int nchunk);
void launch_best_update(cudaStream_t s, const Shape& sh, const uint32_t* settle,
                        const double* dcost_lin, const double* dcost_extra, int64_t seed_begin,
                        const int32_t* step_counter, double* best, int32_t* best_flag,
                        double* valid_cost_out, uint8_t* valid_out, double* trace = nullptr,
                        int trace_cap = 0);
void launch_best_snapshot(cudaStream_t s, const Shape& sh, const int32_t* choice,
                          const uint32_t* reach, const double* best, const int32_t* best_flag,
                          int64_t seed_begin, int32_t* best_choice);
// MLP (kernels_mlp.cu): f_mlp[b] (fp64) and gz1 = df/dz1 (may be NULL);
// gp = u + W1^T gz1.
// z1_part: [nsplit][128][Bp] split-K partials of the tensor-core layer 1
// (nsplit = mlp_nsplit(device) CTAs per seed chunk); z1: [H1][Bp]
// W1 in the tiles of the TMA layer-1 kernel (kernels_mlp.cu)
std::vector<float> mlp_w1_tiles(const float* W1, int H1, int N);
void launch_mlp_fwd(cudaStream_t s, const Shape& sh, int32_t H1, int32_t H2, const float* W1,
                    const float* W1t,
                    const float* b1, const float* W2, const float* b2, const float* W3,
                    const float* b3, const float* p, float* z1_part, float* z1, double* f_mlp,
                    float* gz1, int32_t nsplit);
int mlp_nsplit(int device);
// W1^T in the tiles of the TMA layer-1 backward kernel (kernels_mlp.cu)
std::vector<float> mlp_w1_back_tiles(const float* W1, int H1, int N);
void launch_mlp_bwd(cudaStream_t s, const Shape& sh, int32_t H1, const float* W1, const float* W1b,
                    const float* u, const float* gz1, float* gp, int32_t nsms);

int num_sms(int device);
int64_t& launch_counter();

// 2-D tensor map (tma.cu): dims {inner, outer} elements of fp32 / int32,
// rows row_bytes apart, box {box_inner, box_outer}, optionally written to
// shared memory with the 128-byte swizzle (box_inner * 4 must be 128); cached
CUtensorMap tensor_map_2d(const void* base, bool is_int, uint64_t inner, uint64_t outer,
                          uint64_t row_bytes, uint32_t box_inner, uint32_t box_outer,
                          bool swizzle128 = false);

}  // namespace smoothe
