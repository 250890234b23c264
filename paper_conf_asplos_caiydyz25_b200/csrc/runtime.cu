// libsmoothe runtime: the C ABI of include/smoothe.h.
//
// One optimisation step (Sec. 3.5) is a fixed sequence of
// kernel launches on the run's private stream (captured once into a CUDA graph
// and replayed, unless profiling):
//
//   prologue      Adam bias corrections of this step            (S10)
//   softmax       cp = softmax(theta), c_j = argmax theta, sel   (Eq. 3b, P277, P279)
//   forward x K   q^t from q^{t-1}                               (Eqs. 5-7, P215)
//   cost          f(p), backward initialisation                  (P101, P409, P425)
//   penalty       NOTEARS per (SCC, group)                       (Eqs. 8-11, P318-325)
//   reverse x K   g_cp, g_q                                      (App. C)
//   update        softmax backward + Adam                        (P277)
//   decode        reach, settle, discrete cost                   (P279, P103-111)
//   best          keep the best (cost, step, seed)               (P297, S20)
#include <algorithm>
#include <array>
#include <chrono>
#include <cmath>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <new>
#include <map>

#include "internal.h"

namespace smoothe {

static thread_local std::string g_last_error;
void set_error(const std::string& msg) { g_last_error = msg; }

// steps recorded by the per-step trace (relaxed vs sampled cost, E11)
constexpr int kTraceCap = 4096;

int64_t& launch_counter() {
  static int64_t counter = 0;
  return counter;
}

int num_sms(int device) {
  static int cached[64] = {0};
  if (device >= 0 && device < 64 && cached[device]) return cached[device];
  int n = 0;
  SM_CUDA(cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, device));
  if (device >= 0 && device < 64) cached[device] = n;
  return n;
}

template <typename T>
static T* dalloc(std::vector<void*>& owned, size_t count) {
  if (count == 0) count = 1;
  void* p = nullptr;
  cudaError_t e = cudaMalloc(&p, count * sizeof(T));
  if (e == cudaErrorMemoryAllocation) {
    (void)cudaGetLastError();
    throw Failure{SMOOTHE_E_OOM, "cudaMalloc of " + std::to_string(count * sizeof(T)) + " bytes failed"};
  }
  SM_CUDA(e);
  owned.push_back(p);
  return static_cast<T*>(p);
}

template <typename T>
static T* upload(std::vector<void*>& owned, const std::vector<T>& v, int64_t* bytes = nullptr) {
  T* d = dalloc<T>(owned, v.size());
  if (!v.empty()) SM_CUDA(cudaMemcpy(d, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice));
  if (bytes) *bytes += (int64_t)(v.size() * sizeof(T));
  return d;
}

// One device allocation for all arrays of an e-graph: run the upload sequence
// once to measure (base == nullptr), allocate, run it again to copy.
struct Arena {
  char* base = nullptr;
  size_t used = 0;
};

template <typename T>
static T* upload(Arena& A, const std::vector<T>& v, int64_t* bytes = nullptr) {
  const size_t off = (A.used + 255) & ~(size_t)255;
  A.used = off + std::max<size_t>(1, v.size()) * sizeof(T);
  if (!A.base) return nullptr;
  T* d = reinterpret_cast<T*>(A.base + off);
  if (!v.empty()) SM_CUDA(cudaMemcpy(d, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice));
  if (bytes) *bytes += (int64_t)(v.size() * sizeof(T));
  return d;
}

// Caching allocator for run state: a freed run's device blocks are kept (per
// device, the last freed run only) and handed to the next run that asks for
// blocks of the same sizes, so back-to-back runs of one configuration do not
// pay for unmapping and mapping tens of GB.  On an allocation failure the cache
// of the device is released and the allocation retried.
struct DevCache {
  std::mutex mu;
  std::multimap<std::pair<int, size_t>, void*> blocks;
};
DevCache& dev_cache() {
  static DevCache c;
  return c;
}
void cache_release(int device) {
  DevCache& c = dev_cache();
  std::lock_guard<std::mutex> lk(c.mu);
  int cur = 0;
  cudaGetDevice(&cur);
  for (auto it = c.blocks.begin(); it != c.blocks.end();) {
    if (device < 0 || it->first.first == device) {
      cudaSetDevice(it->first.first);
      cudaFree(it->second);
      it = c.blocks.erase(it);
    } else {
      ++it;
    }
  }
  cudaSetDevice(cur);
}

struct RunMem {
  std::vector<void*> p;
  std::vector<size_t> n;
  int device = 0;
};

template <typename T>
static T* dalloc(RunMem& m, size_t count) {
  if (count == 0) count = 1;
  const size_t bytes = count * sizeof(T);
  {
    DevCache& c = dev_cache();
    std::lock_guard<std::mutex> lk(c.mu);
    auto it = c.blocks.find({m.device, bytes});
    if (it != c.blocks.end()) {
      void* q = it->second;
      c.blocks.erase(it);
      m.p.push_back(q);
      m.n.push_back(bytes);
      return static_cast<T*>(q);
    }
  }
  void* q = nullptr;
  cudaError_t e = cudaMalloc(&q, bytes);
  if (e == cudaErrorMemoryAllocation) {
    (void)cudaGetLastError();
    cache_release(m.device);
    e = cudaMalloc(&q, bytes);
  }
  if (e == cudaErrorMemoryAllocation) {
    (void)cudaGetLastError();
    throw Failure{SMOOTHE_E_OOM, "cudaMalloc of " + std::to_string(bytes) + " bytes failed"};
  }
  SM_CUDA(e);
  m.p.push_back(q);
  m.n.push_back(bytes);
  return static_cast<T*>(q);
}

template <typename T>
static T* upload(RunMem& m, const std::vector<T>& v, int64_t* bytes = nullptr) {
  T* d = dalloc<T>(m, v.size());
  if (!v.empty()) SM_CUDA(cudaMemcpy(d, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice));
  if (bytes) *bytes += (int64_t)(v.size() * sizeof(T));
  return d;
}

// a freed run's blocks replace the device's cache
void runmem_free(RunMem& m, void* p) {  // one block, back to the driver
  for (size_t i = 0; i < m.p.size(); ++i)
    if (m.p[i] == p) {
      cudaFree(p);
      m.p.erase(m.p.begin() + i);
      m.n.erase(m.n.begin() + i);
      return;
    }
}

void runmem_recycle(RunMem& m) {
  cache_release(m.device);
  DevCache& c = dev_cache();
  std::lock_guard<std::mutex> lk(c.mu);
  for (size_t i = 0; i < m.p.size(); ++i) c.blocks.insert({{m.device, m.n[i]}, m.p[i]});
  m.p.clear();
  m.n.clear();
}

}  // namespace smoothe

using namespace smoothe;

struct smoothe_egraph_dev_owner {
  std::vector<void*> owned;
};

struct smoothe_run {
  smoothe_egraph* g = nullptr;
  smoothe_options opt{};
  Shape sh{};
  int K = 0, G = 1, ngroups = 1, device = 0, cost_kind = 0, H1 = 0, H2 = 0, nsplit = 0;
  int coop_grid = 0, f_rows = 0, dcost_rows = 0, rows_M = 0, rows_N = 0;
  Agg agg{0.f, 0.f};
  cudaStream_t stream = nullptr;
  // decode / keep-best run on a second stream, concurrently with the sweeps of
  // the same step (they only need the step's choices), joined at the step end
  cudaStream_t stream2 = nullptr;
  // graph capture: conditional bodies are captured on their own stream
  cudaStream_t stream_body = nullptr;
  cudaStream_t stream_body2 = nullptr;  // nested conditional bodies
  bool in_capture = false;
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr, ev_pen = nullptr;
  bool overlap = false;
  double* red_scratch_d = nullptr;  // the decode stream's own reduction / cost scratch
  float *f_part_d = nullptr, *z1_part_d = nullptr, *z1_d = nullptr;
  RunMem owned;  // device state (recycled through the caching allocator)
  // state
  float *theta = nullptr, *m = nullptr, *v = nullptr, *cp = nullptr, *gcp = nullptr;
  SweepState sw;  // q / pi / am version stacks, q buffers, change stamps
  float* gq[2] = {nullptr, nullptr};
  float* f_part = nullptr;
  double *f = nullptr, *fextra = nullptr, *ftot = nullptr, *h_part = nullptr, *h = nullptr,
         *loss = nullptr;
  float* pen = nullptr;
  double* big_scratch = nullptr;  // large-component penalty matrices
  int big_gpb = 0;
  int32_t* choice = nullptr;
  uint32_t *sel = nullptr, *reach = nullptr, *settle = nullptr, *invalid = nullptr;
  int32_t* flags = nullptr;
  double *dcost_part = nullptr, *dcost = nullptr, *dextra = nullptr;
  double* best = nullptr;
  int32_t *best_flag = nullptr, *best_choice = nullptr, *counter = nullptr;
  double* scal = nullptr;
  double* trace = nullptr;  // [kTraceCap][4] per-step record (smoothe_run_get_trace)
  double* red_scratch = nullptr;  // 128 x Bp, reductions
  float* rev_part = nullptr;       // reverse sweep partial rows [rev_num_slots][Bp]
  int32_t* rev_cnt = nullptr;      // [M][seed slices] items finished (self-resetting)
  int32_t* rev_cursor = nullptr;   // [K+2][Bp/128] item cursors of the TMA reverse sweeps (zeroed per step)
  // cost model
  float* u_f = nullptr;
  double* u_d = nullptr;
  int32_t *q_ptr = nullptr, *q_nbr = nullptr;
  float* q_w = nullptr;
  float* W1t = nullptr;  // W1 in k_mlp_l1_tma's tiles (mlp_w1_tiles)
  float* W1b = nullptr;  // W1^T in k_mlp_l1_back_tma's tiles (mlp_w1_back_tiles)
  float *W1 = nullptr, *b1 = nullptr, *W2 = nullptr, *b2 = nullptr, *W3 = nullptr, *b3 = nullptr;
  float *p = nullptr, *gp = nullptr, *sbin = nullptr, *z1_part = nullptr, *z1 = nullptr,
        *gz1 = nullptr;
  double* fmlp_s = nullptr;
  // debug outputs (set only during smoothe_debug_step)
  float *dbg_p = nullptr, *dbg_gth = nullptr, *dbg_gcp = nullptr;
  double* dbg_dcost = nullptr;
  uint8_t* dbg_valid = nullptr;
  bool debug = false;
  // timing / profiling
  cudaEvent_t ev_start = nullptr;
  std::vector<cudaEvent_t> ev_step;
  std::chrono::steady_clock::time_point t_create;
  bool profiling = false;
  std::vector<std::array<cudaEvent_t, SMOOTHE_NUM_PHASES + 1>> prof_ev;
  std::vector<cudaEvent_t> prof_pool;
  size_t prof_pool_used = 0;
  int64_t prof_launch[SMOOTHE_NUM_PHASES] = {0};
  int64_t prof_launch_total = 0, prof_steps = 0;
  std::vector<std::array<cudaEvent_t, 2>> prof_kev[3];  // around each sweep kernel
  int64_t* frozen_count = nullptr;  // device: k_wspmv launches with frozen seeds (profiling)
  // graph
  cudaGraphExec_t graph_exec = nullptr;
  bool graph_failed = false;
  int64_t graph_steps = 0;  // steps replayed from graph_exec
  int64_t pool_high = 0;    // most version-pool rows a chunk took in a step (checked steps)
  int32_t pool_grows = 0;   // times the pools grew
  bool poisoned = false;
  int steps_run = 0;
};

namespace {

template <typename F>
smoothe_status guarded(smoothe_run* run, F&& fn) {
  try {
    fn();
    return SMOOTHE_OK;
  } catch (const Failure& f) {
    set_error(f.msg);
    if (run && f.status == SMOOTHE_E_CUDA) run->poisoned = true;
    return f.status;
  } catch (const std::bad_alloc&) {
    set_error("host allocation failed");
    return SMOOTHE_E_OOM;
  } catch (...) {
    set_error("unknown internal error");
    return SMOOTHE_E_INVALID_ARG;
  }
}

void check_run(smoothe_run* run) {
  SM_REQUIRE(run != nullptr, SMOOTHE_E_INVALID_ARG, "NULL run");
  SM_REQUIRE(!run->poisoned, SMOOTHE_E_STATE, "run is poisoned by an earlier CUDA error");
  SM_CUDA(cudaSetDevice(run->device));
}

cudaEvent_t pool_event(smoothe_run* r) {
  if (r->prof_pool_used == r->prof_pool.size()) {
    cudaEvent_t e;
    SM_CUDA(cudaEventCreate(&e));
    r->prof_pool.push_back(e);
  }
  return r->prof_pool[r->prof_pool_used++];
}

// Record the boundary event before `phase` when profiling.
struct PhaseMarks {
  smoothe_run* r;
  std::array<cudaEvent_t, SMOOTHE_NUM_PHASES + 1> ev{};
  int64_t last = 0;
  int cur = -1;
  explicit PhaseMarks(smoothe_run* run) : r(run) {}
  void mark(int phase) {
    if (!r->profiling) return;
    if (cur >= 0) r->prof_launch[cur] += launch_counter() - last;
    last = launch_counter();
    cur = phase;
    ev[phase] = pool_event(r);
    SM_CUDA(cudaEventRecord(ev[phase], r->stream));
  }
  void finish() {
    if (!r->profiling) return;
    r->prof_launch[cur] += launch_counter() - last;
    ev[SMOOTHE_NUM_PHASES] = pool_event(r);
    SM_CUDA(cudaEventRecord(ev[SMOOTHE_NUM_PHASES], r->stream));
    r->prof_ev.push_back(ev);
  }
};

// Inside a graph capture on stream s: `set` launches a kernel that sets the
// conditional handle it is given, `body` enqueues the work run only when the
// handle is non-zero (a conditional IF node; its body captured on sb).
template <class SetF, class BodyF>
void enqueue_if(cudaStream_t s, cudaStream_t sb, SetF set, BodyF body) {
  cudaStreamCaptureStatus st;
  cudaGraph_t graph = nullptr;
  const cudaGraphNode_t* deps = nullptr;
  size_t ndeps = 0;
  SM_CUDA(cudaStreamGetCaptureInfo(s, &st, nullptr, &graph, &deps, &ndeps));
  cudaGraphConditionalHandle h;
  SM_CUDA(cudaGraphConditionalHandleCreate(&h, graph, 0, 0));
  set(h);
  SM_CUDA(cudaStreamGetCaptureInfo(s, &st, nullptr, &graph, &deps, &ndeps));
  cudaGraphNodeParams p = {};
  p.type = cudaGraphNodeTypeConditional;
  p.conditional.handle = h;
  p.conditional.type = cudaGraphCondTypeIf;
  p.conditional.size = 1;
  cudaGraphNode_t node;
  SM_CUDA(cudaGraphAddNode(&node, graph, deps, ndeps, &p));
  cudaGraph_t bg = p.conditional.phGraph_out[0];
  SM_CUDA(cudaStreamBeginCaptureToGraph(sb, bg, nullptr, nullptr, 0, cudaStreamCaptureModeThreadLocal));
  body(sb);
  SM_CUDA(cudaStreamEndCapture(sb, &bg));
  SM_CUDA(cudaStreamUpdateCaptureDependencies(s, &node, 1, cudaStreamSetCaptureDependencies));
}

// A two-body switch node: `set` launches the kernel that sets the handle;
// value 0 runs body0, 1 runs body1, anything else nothing.
template <class SetF, class B0, class B1>
void enqueue_switch2(cudaStream_t s, cudaStream_t sb, SetF set, B0 body0, B1 body1) {
  cudaStreamCaptureStatus st;
  cudaGraph_t graph = nullptr;
  const cudaGraphNode_t* deps = nullptr;
  size_t ndeps = 0;
  SM_CUDA(cudaStreamGetCaptureInfo(s, &st, nullptr, &graph, &deps, &ndeps));
  cudaGraphConditionalHandle h;
  SM_CUDA(cudaGraphConditionalHandleCreate(&h, graph, 0, 0));
  set(h);
  SM_CUDA(cudaStreamGetCaptureInfo(s, &st, nullptr, &graph, &deps, &ndeps));
  cudaGraphNodeParams p = {};
  p.type = cudaGraphNodeTypeConditional;
  p.conditional.handle = h;
  p.conditional.type = cudaGraphCondTypeSwitch;
  p.conditional.size = 2;
  cudaGraphNode_t node;
  SM_CUDA(cudaGraphAddNode(&node, graph, deps, ndeps, &p));
  cudaGraph_t b0 = p.conditional.phGraph_out[0], b1 = p.conditional.phGraph_out[1];
  SM_CUDA(cudaStreamBeginCaptureToGraph(sb, b0, nullptr, nullptr, 0, cudaStreamCaptureModeThreadLocal));
  body0(sb);
  SM_CUDA(cudaStreamEndCapture(sb, &b0));
  SM_CUDA(cudaStreamBeginCaptureToGraph(sb, b1, nullptr, nullptr, 0, cudaStreamCaptureModeThreadLocal));
  body1(sb);
  SM_CUDA(cudaStreamEndCapture(sb, &b1));
  SM_CUDA(cudaStreamUpdateCaptureDependencies(s, &node, 1, cudaStreamSetCaptureDependencies));
}

// Decode (P279, P103-111), its discrete cost and keep-best (P297) on stream ds.
// With the decode stream (overlap), it uses its own scratch buffers.
void enqueue_decode(smoothe_run* r, cudaStream_t ds, PhaseMarks* pm) {
  const Shape& sh = r->sh;
  const DevGraph& g = r->g->dev;
  const HostGraph& hg = r->g->host;
  const bool side = ds != r->stream;
  double* red = side ? r->red_scratch_d : r->red_scratch;
  float* fpart = side ? r->f_part_d : r->f_part;
  float* z1p = side ? r->z1_part_d : r->z1_part;
  float* z1 = side ? r->z1_d : r->z1;
  launch_decode(ds, sh, hg, g, r->sel, r->choice, r->reach, r->settle, r->invalid,
                r->settle + (size_t)sh.root * sh.W, r->coop_grid);
  launch_decode_cost_linear(ds, sh, g, r->u_d, r->choice, r->reach, r->dcost_part);
  launch_reduce_rows_f64d(ds, r->dcost_part, r->dcost_rows, sh.Bp, r->dcost, red);
  const double* dextra = nullptr;
  if (r->cost_kind == SMOOTHE_COST_QUADRATIC) {
    launch_decode_s(ds, sh, g, r->sel, r->reach, r->sbin);
    launch_quadratic(ds, sh, r->q_ptr, r->q_nbr, r->q_w, nullptr, r->sbin, nullptr, fpart);
    launch_reduce_rows_f64(ds, fpart, r->rows_N, sh.Bp, r->dextra, 1.0, red);
    dextra = r->dextra;
  } else if (r->cost_kind == SMOOTHE_COST_MLP) {
    launch_decode_s(ds, sh, g, r->sel, r->reach, r->sbin);
    launch_mlp_fwd(ds, sh, r->H1, r->H2, r->W1, r->W1t, r->b1, r->W2, r->b2, r->W3, r->b3, r->sbin,
                   z1p, z1, r->dextra, nullptr, r->nsplit);
    dextra = r->dextra;
  }
  if (pm) pm->mark(SMOOTHE_PHASE_BEST);
  launch_best_update(ds, sh, r->settle, r->dcost, dextra, r->opt.seed_begin, r->counter, r->best,
                     r->best_flag, r->debug ? r->dbg_dcost : nullptr,
                     r->debug ? r->dbg_valid : nullptr, r->trace, kTraceCap);
}

void enqueue_step(smoothe_run* r) {
  const Shape& sh = r->sh;
  const DevGraph& g = r->g->dev;
  const HostGraph& hg = r->g->host;
  cudaStream_t s = r->stream;
  const size_t MB = (size_t)sh.M * sh.Bp;
  const int K = r->K;
  const int64_t l0 = launch_counter();
  PhaseMarks pm(r);

  pm.mark(SMOOTHE_PHASE_SOFTMAX);
  launch_step_prologue(s, r->counter, r->scal, r->opt.beta1, r->opt.beta2, nullptr);
  launch_softmax_argmax(s, sh, g, r->theta, r->cp, r->choice, r->sel);
  const bool overlap_now = r->overlap && !r->profiling && !r->debug;
  if (overlap_now) {  // penalty and decode of this step alongside the sweeps
    SM_CUDA(cudaEventRecord(r->ev_fork, s));
    SM_CUDA(cudaStreamWaitEvent(r->stream2, r->ev_fork, 0));
    if (hg.num_scc > 0) {  // needs cp only; joined before the loss
      launch_notears(r->stream2, sh, hg, g, r->G, r->opt.lambda, r->cp, r->h_part, r->pen,
                     r->big_scratch, r->big_gpb);
      launch_reduce_rows_f64d(r->stream2, r->h_part, hg.num_scc, r->ngroups, r->h,
                              r->red_scratch_d);
      SM_CUDA(cudaEventRecord(r->ev_pen, r->stream2));
    }
    enqueue_decode(r, r->stream2, nullptr);
    SM_CUDA(cudaEventRecord(r->ev_join, r->stream2));
  }

  pm.mark(SMOOTHE_PHASE_FORWARD);
  launch_sweep_reset(s, sh, r->sw);
  SM_CUDA(cudaMemsetAsync(r->rev_cursor, 0, sizeof(int32_t) * (r->K + 2) * std::max(1, sh.Bp / 128), s));
  // (when profiling, events bracket each sweep kernel: bench.py's roofline)
  auto kmark = [&](int which, int at) {
    if (!r->profiling) return;
    if (at == 0) r->prof_kev[which].push_back({pool_event(r), nullptr});
    else r->prof_kev[which].back()[1] = pool_event(r);
    SM_CUDA(cudaEventRecord(r->prof_kev[which].back()[at], s));
  };
  // In the captured step of a large graph, forward sweeps [t, t + fblock)
  // (t >= 2) are one conditional node on fchg[t - 1]: once a sweep changes no
  // q row, it and every later sweep are the identity (C4: the rows freeze by
  // sweep ~46 of 207), so the blocks after it launch nothing.  Gated in blocks
  // because a conditional node costs more than an empty sweep (~10 us).
  // (Direct launches: the kernels of such a sweep find no dirty class.)
  const bool big = r->in_capture && r->sw.big_sched;
  const int fb = big && r->sw.fchg ? r->sw.fblock : 0;
  for (int t = 1; t <= K;) {
    if (fb > 0 && t >= 2) {
      const int t1 = std::min(K + 1, t + fb);
      enqueue_if(
          s, r->stream_body,
          [&](cudaGraphConditionalHandle h) { launch_flag_if(s, r->sw.fchg + (t - 1), h); },
          [&](cudaStream_t bs) {
            for (int u = t; u < t1; ++u) launch_sweep_forward(bs, sh, g, r->agg, u, r->sw, r->cp);
          });
      t = t1;
      continue;
    }
    kmark(0, 0);
    launch_sweep_forward(s, sh, g, r->agg, t, r->sw, r->cp);
    kmark(0, 1);
    ++t;
  }
  if (r->profiling && std::getenv("SMOOTHE_FREEZE_STATS")) {
    // diagnostic (stderr): per class the last forward sweep that recomputed
    // it, and F_i = the first reverse sweep (going down) at which class i's
    // reverse item no longer sees final rows: max(last(i) + 1, max_j last(j))
    std::vector<int32_t> ln(K + 2);
    std::vector<int4> lst((size_t)(K + 1) * sh.M);
    SM_CUDA(cudaMemcpyAsync(ln.data(), r->sw.list_n, sizeof(int32_t) * ln.size(), cudaMemcpyDeviceToHost, s));
    SM_CUDA(cudaMemcpyAsync(lst.data(), r->sw.list, sizeof(int4) * lst.size(), cudaMemcpyDeviceToHost, s));
    SM_CUDA(cudaStreamSynchronize(s));
    std::vector<int32_t> last(sh.M, 0);
    for (int t = 1; t <= K; ++t)
      for (int i = 0; i < ln[t]; ++i) last[lst[(size_t)t * sh.M + i].x] = t;
    std::vector<int64_t> hist(K + 2, 0), lasth(K + 2, 0);
    int64_t items_plain = 0;
    for (int j = 0; j < sh.M; ++j) {
      int F = last[j] + 1;
      for (int c = hg.cls_child_ptr[j]; c < hg.cls_child_ptr[j + 1]; ++c)
        F = std::max(F, last[hg.cls_child[c]]);
      F = std::min(F, K + 1);
      hist[F]++;
      lasth[last[j]]++;
      items_plain += F - 1;  // reverse sweeps t < F_i
    }
    int64_t seedf = 0;
    for (int t = 0; t <= K; ++t) if (ln[t] > 0) seedf = t;
    std::fprintf(stderr, "[freeze] K=%d last recompute sweep (any class) %lld; mean F %.2f; "
                 "plain (class,sweep) pairs %.3f of K*M\n", K, (long long)seedf,
                 (double)items_plain / sh.M + 1.0, (double)items_plain / ((double)K * sh.M));
    std::fprintf(stderr, "[freeze] F histogram (F: classes):");
    for (int t = 0; t <= K + 1; ++t) if (hist[t]) std::fprintf(stderr, " %d:%lld", t, (long long)hist[t]);
    std::fprintf(stderr, "\n");
  }

  pm.mark(SMOOTHE_PHASE_COST);
  const float* qK = r->sw.qbuf[K & 1];
  float* gqK = r->gq[K & 1];
  if (r->cost_kind == SMOOTHE_COST_LINEAR) {
    launch_cost_linear(s, sh, g, r->u_f, r->cp, qK, r->gcp, gqK, r->f_part,
                       r->debug ? r->dbg_p : nullptr, 0);
    launch_reduce_rows_f64(s, r->f_part, r->rows_M, sh.Bp, r->f, 1.0, r->red_scratch);
  } else if (r->cost_kind == SMOOTHE_COST_QUADRATIC) {
    launch_materialize_p_f(s, sh, g, nullptr, r->cp, qK, r->p, nullptr);
    launch_quadratic(s, sh, r->q_ptr, r->q_nbr, r->q_w, r->u_f, r->p, r->gp, r->f_part);
    launch_reduce_rows_f64(s, r->f_part, r->rows_N, sh.Bp, r->f, 1.0, r->red_scratch);
    launch_cost_gp(s, sh, g, r->gp, r->cp, qK, r->gcp, gqK);
  } else {
    launch_materialize_p_f(s, sh, g, r->u_f, r->cp, qK, r->p, r->f_part);
    launch_reduce_rows_f64(s, r->f_part, r->rows_M, sh.Bp, r->f, 1.0, r->red_scratch);
    launch_mlp_fwd(s, sh, r->H1, r->H2, r->W1, r->W1t, r->b1, r->W2, r->b2, r->W3, r->b3, r->p,
                   r->z1_part, r->z1, r->fextra, r->gz1, r->nsplit);
    launch_mlp_bwd(s, sh, r->H1, r->W1, r->W1b, r->u_f, r->gz1, r->gp, r->nsplit);
    launch_cost_gp(s, sh, g, r->gp, r->cp, qK, r->gcp, gqK);
  }

  pm.mark(SMOOTHE_PHASE_PENALTY);
  if (overlap_now && hg.num_scc > 0) {
    SM_CUDA(cudaStreamWaitEvent(s, r->ev_pen, 0));  // computed on the second stream
  } else if (hg.num_scc > 0) {
    launch_notears(s, sh, hg, g, r->G, r->opt.lambda, r->cp, r->h_part, r->pen, r->big_scratch,
                   r->big_gpb);
    launch_reduce_rows_f64d(s, r->h_part, hg.num_scc, r->ngroups, r->h, r->red_scratch);
  }
  launch_loss(s, sh.B, r->G, r->ngroups, r->opt.lambda, r->f,
              r->cost_kind == SMOOTHE_COST_MLP ? r->fextra : nullptr, hg.num_scc > 0 ? r->h : nullptr,
              r->ftot, r->loss, r->scal, r->trace, kTraceCap);

  pm.mark(SMOOTHE_PHASE_REVERSE);
  SweepState& sw = r->sw;
  const float* cur_q = sw.qbuf[(K - 1) & 1];
  // In the captured step of a large graph (C4), each sweep t < K is a
  // conditional node on live[t] (the sweep's input g_q^t not all zero), so
  // the sweeps after the gradient has died launch nothing; the plain kernel
  // inside is itself conditional on some seed being unfrozen.  (Direct
  // launches: every kernel of a dead sweep returns at once.)
  auto sweep = [&](int t, cudaStream_t ss, cudaStream_t sbody) {
      launch_rev_transition(ss, sh, g, t, K, sw);
      if (sw.wmode && t == K) {  // K-state rows, W, every seed frozen at t = K
        SM_CUDA(cudaMemcpyAsync(sw.kq, cur_q, sizeof(float) * MB, cudaMemcpyDeviceToDevice, ss));
        if (sw.kpi)
          SM_CUDA(cudaMemcpyAsync(sw.kpi, sw.cur_pi, sizeof(float) * MB, cudaMemcpyDeviceToDevice, ss));
        SM_CUDA(cudaMemcpyAsync(sw.kam, sw.cur_am, sizeof(int32_t) * MB, cudaMemcpyDeviceToDevice, ss));
        SM_CUDA(cudaMemsetAsync(sw.wm, 1, sizeof(int32_t) * sh.Bp, ss));
        SM_CUDA(cudaMemsetAsync(sw.S, 0, sizeof(float) * MB, ss));
        launch_wbuild(ss, sh, g, r->agg, sw, r->cp);
      }
      if (sw.converge && t == K) launch_last_change(ss, sh, sw);
      if (sw.wmode && r->profiling && std::getenv("SMOOTHE_REV_W_STATS")) {
        // diagnostic: seeds still frozen before reverse sweep t (stderr, one line per sweep)
        std::vector<int32_t> h(sh.Bp);
        SM_CUDA(cudaMemcpyAsync(h.data(), sw.wm, sizeof(int32_t) * sh.Bp, cudaMemcpyDeviceToHost, ss));
        SM_CUDA(cudaStreamSynchronize(ss));
        int n = 0, slices = 0;
        for (int b = 0; b < sh.B; ++b) n += h[b] != 0;
        for (int c = 0; c * 128 < sh.Bp; ++c) {
          bool all = true;
          for (int b = c * 128; b < std::min(sh.Bp, (c + 1) * 128); ++b) all = all && h[b] != 0;
          slices += all;
        }
        fprintf(stderr, "[wstats] t=%d frozen_seeds=%d full_slices=%d\n", t, n, slices);
      }
      kmark(1, 0);
      // converge mode: a seed's loss reads q^{t*} (t* = its convergence sweep),
      // so the reverse window (g_q^t_j = 0 while t + hmax_j <= K) does not hold
      // for K; no window then (the window argument with t* would be per seed)
      auto plain = [&](cudaStream_t ps) {
        launch_sweep_reverse(ps, sh, g, r->agg, t, sw.converge ? -1 : K, cur_q, sw.cur_pi,
                             sw.cur_am, sw.wmode ? sw.wm : nullptr, r->cp, r->gq[t & 1], r->gcp,
                             r->gq[(t - 1) & 1], t > 1, r->rev_part, r->rev_cnt,
                             sw.converge && !sw.wmode ? sw.lastchg : nullptr,
                             r->rev_cursor + (size_t)t * std::max(1, sh.Bp / 128),
                             sw.glive && t < K ? sw.glive + t : nullptr,
                             sw.glive && t > 1 ? sw.glive + (t - 1) : nullptr,
                             sw.gstamp ? sw.gstamp + ((t - 1) & 1) * (size_t)sw.nchunk * sh.M : nullptr,
                             big && sw.wmode && t < K && !sw.plain_if);
      };
      if (big && sw.wmode && t < K && sw.plain_if) {
        // the plain sweep as a conditional node, skipped once every seed is
        // frozen (the default instead launches it as one wave of persistent
        // warps, which exit at once then: cheaper than the conditional)
        enqueue_if(
            ss, sbody,
            [&](cudaGraphConditionalHandle h) { launch_any_unfrozen(ss, sh, sw.wm, h); }, plain);
      } else {
        plain(ss);
      }
      kmark(1, 1);
      if (sw.wmode) {
        if (r->profiling) launch_count_live(ss, sh, g, t, sw, r->frozen_count + 1);
        kmark(2, 0);
        launch_wspmv(ss, sh, g, t, sw, r->gq[t & 1], t > 1 ? r->gq[(t - 1) & 1] : nullptr,
                     r->profiling ? r->frozen_count : nullptr);
        kmark(2, 1);
      }
    };
  // In the captured step of a large graph, reverse sweeps (t - rblock, t]
  // (t < K) are one conditional node on live[t]: the sweeps after the
  // gradient has died launch nothing (the kernels of a dead sweep inside a
  // live block return at once)
  for (int t = K; t >= 1;) {
    if (big && sw.glive && t < K && sw.wmode && sw.fchg && sw.rswitch) {
      // a switch node: nothing (dead), k_wspmv alone (every seed frozen and
      // no row to restore: the block lies above the last forward sweep with
      // a change), or the whole sweeps
      const int t1 = std::max(0, t - sw.rblock);
      enqueue_switch2(
          s, r->stream_body,
          [&](cudaGraphConditionalHandle h) {
            launch_rev_switch(s, sw.glive + t, sw.fchg, t1 + 1, h);
          },
          [&](cudaStream_t bs) {
            for (int u = t; u > t1; --u)
              launch_wspmv(bs, sh, g, u, sw, r->gq[u & 1], u > 1 ? r->gq[(u - 1) & 1] : nullptr,
                           nullptr);
          },
          [&](cudaStream_t bs) {
            for (int u = t; u > t1; --u) sweep(u, bs, r->stream_body2);
          });
      t = t1;
    } else if (big && sw.glive && t < K) {
      const int t1 = std::max(0, t - sw.rblock);
      enqueue_if(
          s, r->stream_body,
          [&](cudaGraphConditionalHandle h) { launch_flag_if(s, sw.glive + t, h); },
          [&](cudaStream_t bs) {
            for (int u = t; u > t1; --u) sweep(u, bs, r->stream_body2);
          });
      t = t1;
    } else {
      sweep(t, s, r->stream_body);
      --t;
    }
  }
  if (sw.wmode)  // the frozen sweeps' g_cp: one pass over the K-state with g = S
    launch_sweep_reverse(s, sh, g, r->agg, K, K, sw.kq, sw.kpi, sw.kam, nullptr, r->cp, sw.S,
                         r->gcp, nullptr, false, r->rev_part, r->rev_cnt, nullptr,
                         r->rev_cursor + (size_t)(K + 1) * std::max(1, sh.Bp / 128));

  pm.mark(SMOOTHE_PHASE_UPDATE);
  launch_update(s, sh, g, r->G, r->cp, r->gcp, hg.num_scc > 0 ? r->pen : nullptr, r->theta, r->m,
                r->v, r->scal, r->opt.optimizer, (float)r->opt.lr, (float)r->opt.beta1,
                (float)r->opt.beta2, (float)r->opt.eps, r->debug ? r->dbg_gth : nullptr,
                r->debug ? r->dbg_gcp : nullptr, r->sw.abort_flag);

  if (!overlap_now) {
    pm.mark(SMOOTHE_PHASE_DECODE);
    enqueue_decode(r, s, &pm);
  } else {
    SM_CUDA(cudaStreamWaitEvent(s, r->ev_join, 0));
  }
  // keep-best of the complete step (an aborted step commits nothing)
  launch_best_commit(s, r->counter, r->best, r->best_flag, r->sw.abort_flag, r->sw.pool_n,
                     r->sw.nchunk);
  launch_best_snapshot(s, sh, r->choice, r->reach, r->best, r->best_flag, r->opt.seed_begin,
                       r->best_choice);
  pm.finish();
  if (r->profiling) {
    r->prof_launch_total += launch_counter() - l0;
    r->prof_steps += 1;
  }
}

void run_one_step(smoothe_run* r) {
  const bool use_graph = r->opt.use_graphs && !r->profiling && !r->debug && !r->graph_failed;
  if (use_graph && !r->graph_exec) {
    cudaGraph_t graph = nullptr;
    const int64_t before = launch_counter();
    bool ok = cudaStreamBeginCapture(r->stream, cudaStreamCaptureModeThreadLocal) == cudaSuccess;
    if (ok) {
      r->in_capture = true;
      try {
        enqueue_step(r);
      } catch (const Failure& f) {
        ok = false;
        if (std::getenv("SMOOTHE_GRAPH_DEBUG")) std::fprintf(stderr, "[graph] %s\n", f.msg.c_str());
      }
      r->in_capture = false;
      cudaError_t e = cudaStreamEndCapture(r->stream, &graph);
      ok = ok && e == cudaSuccess && graph != nullptr;
    }
    if (ok) ok = cudaGraphInstantiate(&r->graph_exec, graph, 0) == cudaSuccess;
    if (graph) cudaGraphDestroy(graph);
    launch_counter() = before;
    if (!ok) {
      if (std::getenv("SMOOTHE_GRAPH_DEBUG"))
        std::fprintf(stderr, "[graph] capture failed: %s\n", cudaGetErrorString(cudaGetLastError()));
      (void)cudaGetLastError();
      r->graph_exec = nullptr;
      r->graph_failed = true;  // fall back to direct launches (still all on the GPU)
      std::fprintf(stderr, "[smoothe] warning: CUDA graph capture of the step failed; "
                   "running direct launches (set SMOOTHE_GRAPH_DEBUG=1 for the reason)\n");
    }
  }
  if (use_graph && r->graph_exec) {
    SM_CUDA(cudaGraphLaunch(r->graph_exec, r->stream));
    r->graph_steps++;
  } else {
    enqueue_step(r);
  }
  if ((size_t)r->steps_run < r->ev_step.size()) {
    SM_CUDA(cudaEventRecord(r->ev_step[r->steps_run], r->stream));
  }
  r->steps_run++;
}

// Version pools.  All (K + 1) M rows per chunk -- the stacks of
// a full recompute -- when that is small; else a fraction of it
// (SMOOTHE_POOL_FRAC, default 0.15 of the K sweeps; measured on C4: a step
// recomputes 7% of (K+1) M class rows early in a run, more later)
// that smoothe_run_steps grows when a step overflows.
int64_t initial_pool_rows(const smoothe_run* r) {
  const Shape& sh = r->sh;
  const int64_t full = ((int64_t)r->K + 1) * sh.M;
  const double bytes = (double)full * sh.Bp * 4.0 * (r->agg.wI != 0.f ? 3 : 2);
  const char* e = std::getenv("SMOOTHE_POOL_FRAC");
  if (!e && bytes <= 4e9) return full;
  const double frac = e ? std::atof(e) : 0.15;
  return std::min<int64_t>(full, sh.M + (int64_t)std::ceil(frac * r->K * sh.M));
}

void alloc_pools(smoothe_run* r, int64_t cap) {
  SweepState& w = r->sw;
  for (void* p : {(void*)w.qpool, (void*)w.pipool, (void*)w.apool})
    if (p) runmem_free(r->owned, p);
  w.qpool = w.pipool = nullptr;
  w.apool = nullptr;
  w.cap = cap;
  const size_t n = (size_t)w.nchunk * cap * w.wc;
  w.qpool = dalloc<float>(r->owned, n);
  if (r->agg.wI != 0.f) w.pipool = dalloc<float>(r->owned, n);
  w.apool = dalloc<int32_t>(r->owned, n);
}

// After steps were enqueued: if any step overflowed a version pool (it was
// aborted: no update, no keep-best), grow the pools to 1.25x the most rows a
// chunk asked for (at least 1.5x), re-initialise version 0, drop the captured
// graph (its pointers changed) and return the number of aborted steps, which
// the caller repeats.  Synchronises the run's stream.
int pool_check_grow(smoothe_run* r) {
  SweepState& w = r->sw;
  int32_t f[4];
  SM_CUDA(cudaMemcpyAsync(f, w.abort_flag, sizeof(f), cudaMemcpyDeviceToHost, r->stream));
  SM_CUDA(cudaStreamSynchronize(r->stream));
  r->pool_high = std::max<int64_t>(r->pool_high, f[2]);
  if (f[1] == 0) return 0;
  const int64_t full = ((int64_t)r->K + 1) * r->sh.M;
  const int64_t want = std::max<int64_t>((int64_t)(1.25 * f[2]) + 1, (int64_t)(1.5 * w.cap));
  if (w.cap >= full) throw Failure{SMOOTHE_E_STATE, "version pool overflow at full capacity"};
  alloc_pools(r, std::min(full, want));
  launch_pool_version0(r->stream, r->sh, r->g->dev, w);
  SM_CUDA(cudaMemsetAsync(w.abort_flag, 0, sizeof(int32_t) * 2, r->stream));
  if (r->graph_exec) {
    SM_CUDA(cudaGraphExecDestroy(r->graph_exec));
    r->graph_exec = nullptr;
  }
  r->pool_grows++;
  return f[1];
}

void alloc_state(smoothe_run* r, const smoothe_cost_model* cost) {
  const Shape& sh = r->sh;
  const HostGraph& hg = r->g->host;
  auto& o = r->owned;
  const size_t NB = (size_t)sh.N * sh.Bp, MB = (size_t)sh.M * sh.Bp;
  r->theta = dalloc<float>(o, NB);
  r->m = dalloc<float>(o, NB);
  r->v = dalloc<float>(o, NB);
  r->cp = dalloc<float>(o, NB + sh.Bp);  // + one zero row: the padding parent of the sweeps
  r->gcp = dalloc<float>(o, NB);
  {
    SweepState& w = r->sw;
    const char* env = std::getenv("SMOOTHE_SWEEP_ALL");
    w.all = env && env[0] == '1';
    const size_t slots = (size_t)r->K + 1;
    if (r->agg.wI != 0.f) w.cur_pi = dalloc<float>(o, MB);
    w.cur_am = dalloc<int32_t>(o, MB);
    w.qbuf[0] = dalloc<float>(o, 2 * MB);
    w.qbuf[1] = w.qbuf[0] + MB;
    w.K = r->K;
    w.num_sms = num_sms(r->device);
    w.wc = std::min(sh.Bp, 128);
    w.nchunk = sh.Bp / w.wc;
    w.lastrow = dalloc<int32_t>(o, (size_t)w.nchunk * sh.M);
    w.list = dalloc<int4>(o, (size_t)w.nchunk * slots * sh.M);
    w.list_n = dalloc<int32_t>(o, (size_t)w.nchunk * (slots + 1));
    w.pool_n = dalloc<int32_t>(o, w.nchunk);
    w.abort_flag = dalloc<int32_t>(o, 4);
    {
      // dead-gradient skipping pays only where the gradient can underflow to
      // zero within the K sweeps (C4, K = 207: from sweep ~76 down); at K < 100
      // it never does and its stamps cost 10-14% (C2, C3; C5 +0.6%), so it is
      // on for K >= 100 (SMOOTHE_GLIVE=1 / 0 forces)
      const char* genv = std::getenv("SMOOTHE_GLIVE");
      if (genv ? genv[0] == '1' : r->K >= 100) {
        w.glive = dalloc<int32_t>(o, slots + 1);
        w.gstamp = dalloc<int32_t>(o, 2 * (size_t)w.nchunk * sh.M);
        SM_CUDA(cudaMemset(w.gstamp, 0xFF, sizeof(int32_t) * 2 * w.nchunk * sh.M));
      }
    }
    {
      auto envi = [](const char* k, int d) {
        const char* e = std::getenv(k);
        return e && e[0] ? std::atoi(e) : d;
      };
      w.fblock = w.all ? 0 : envi("SMOOTHE_FBLOCK", 16);
      w.rblock = std::max(1, envi("SMOOTHE_RBLOCK", 8));
      w.plain_if = envi("SMOOTHE_PLAIN_IF", 0) != 0;
      w.rswitch = envi("SMOOTHE_RSWITCH", 1) != 0;
      // large graphs (>= 100k reverse items) get the gated schedule of the
      // captured step, whose conditional nodes read the forward change flags;
      // SMOOTHE_BIG_SCHED=1 / 0 forces it on / off (tests of the gated
      // schedule on small graphs)
      const int bs = envi("SMOOTHE_BIG_SCHED", -1);
      w.big_sched = bs >= 0 ? bs != 0 : r->g->dev.num_rev_items >= 100000;
      if (!w.all && w.big_sched) w.fchg = dalloc<int32_t>(o, slots + 1);
    }
    alloc_pools(r, initial_pool_rows(r));
    int32_t* stamps = dalloc<int32_t>(o, 4 * (size_t)sh.M);
    for (int b = 0; b < 2; ++b) {  // consecutive: k_sweep_reset fills all four at once
      w.dirty[b] = stamps + (size_t)b * sh.M;
      w.chg[b] = stamps + (size_t)(2 + b) * sh.M;
    }
    // frozen-sweep path: on for K >= 48 (enough sweeps to freeze and pay for
    // the W build and the final pass), SMOOTHE_REV_W=0 / 1 forces it
    if (r->opt.converge) w.lastchg = dalloc<int32_t>(o, sh.Bp);
    const char* wenv = std::getenv("SMOOTHE_REV_W");
    w.converge = r->opt.converge != 0;
    // convergence mode: with the frozen-sweep path the W kernels pass a
    // converged seed's g_q through, without it the reverse kernel does
    w.wmode = (wenv ? wenv[0] == '1' : r->K >= 48) && r->g->dev.num_cedge > 0;
    if (w.wmode) {
      const char* penv = std::getenv("SMOOTHE_WSPMV_PERSIST");
      w.wpersist = penv ? penv[0] == '1' : r->g->dev.num_witems >= 100000;
      w.W = dalloc<float>(o, (size_t)r->g->dev.num_cedge * sh.Bp);
      w.S = dalloc<float>(o, MB);
      w.kq = dalloc<float>(o, MB);
      if (r->agg.wI != 0.f) w.kpi = dalloc<float>(o, MB);
      w.kam = dalloc<int32_t>(o, MB);
      w.wm = dalloc<int32_t>(o, sh.Bp);
      w.wpart = dalloc<float>(o, (size_t)std::max(1, r->g->dev.w_num_slots) * sh.Bp);
      const char* fuse = std::getenv("SMOOTHE_WFUSE");
      if (!(fuse && fuse[0] == '0') && r->g->dev.w_num_slots > 0) {
        const size_t nc = (size_t)r->g->dev.w_num_slots * w.nchunk;
        w.wcnt = dalloc<int32_t>(o, nc);
        SM_CUDA(cudaMemset(w.wcnt, 0, sizeof(int32_t) * nc));
      }
      r->frozen_count = dalloc<int64_t>(o, 4);  // launches, live edges / rows, rows written
      SM_CUDA(cudaMemset(r->frozen_count, 0, 4 * sizeof(int64_t)));
    }
  }
  r->gq[0] = dalloc<float>(o, MB);
  r->gq[1] = dalloc<float>(o, MB);
  const int rows_per_block_min = 256 / 32;  // kBlock / LPR(32): fewest rows per block
  const int nbig = r->g->dev.num_big;
  r->f_rows = (std::max(sh.M, sh.N) + rows_per_block_min - 1) / rows_per_block_min + 1 + nbig;
  {  // rows of partial sums each row-group kernel writes (its grid.x)
    const int per = 256 / (sh.Bp >= 128 ? 32 : sh.Bp / 4);
    r->rows_M = nbig + (sh.M + per - 1) / per;  // class kernels: one block per big class first
    r->rows_N = (sh.N + per - 1) / per;
  }
  r->f_part = dalloc<float>(o, (size_t)r->f_rows * sh.Bp);
  if (r->overlap) r->f_part_d = dalloc<float>(o, (size_t)r->f_rows * sh.Bp);
  r->f = dalloc<double>(o, sh.Bp);
  r->fextra = dalloc<double>(o, sh.Bp);
  r->ftot = dalloc<double>(o, sh.Bp);
  r->h_part = dalloc<double>(o, (size_t)std::max(1, hg.num_scc) * r->ngroups);
  r->h = dalloc<double>(o, r->ngroups);
  r->loss = dalloc<double>(o, 1);
  r->pen = dalloc<float>(o, std::max<size_t>(1, hg.slot_node.size() * (size_t)r->ngroups));
  {
    const size_t bytes = notears_big_scratch(hg, r->ngroups, &r->big_gpb);
    if (bytes) r->big_scratch = dalloc<double>(o, bytes / sizeof(double));
  }
  r->choice = dalloc<int32_t>(o, MB);
  r->sel = dalloc<uint32_t>(o, (size_t)sh.N * sh.W);
  r->reach = dalloc<uint32_t>(o, (size_t)sh.M * sh.W);
  r->settle = dalloc<uint32_t>(o, (size_t)sh.M * sh.W);
  r->flags = dalloc<int32_t>(o, 8);
  r->invalid = dalloc<uint32_t>(o, sh.W);
  r->dcost_rows = decode_cost_rows(sh);
  r->dcost_part = dalloc<double>(o, (size_t)r->dcost_rows * sh.Bp);
  r->dcost = dalloc<double>(o, sh.Bp);
  r->dextra = dalloc<double>(o, sh.Bp);
  r->best = dalloc<double>(o, 6);  // (cost, step, seed, steps since), the step's candidate (cost, seed)
  r->best_flag = dalloc<int32_t>(o, 1);
  r->best_choice = dalloc<int32_t>(o, sh.M);
  r->counter = dalloc<int32_t>(o, 1);
  r->scal = dalloc<double>(o, 3);
  r->trace = dalloc<double>(o, 4 * (size_t)kTraceCap);
  r->red_scratch = dalloc<double>(o, (size_t)128 * sh.Bp);
  if (r->overlap) r->red_scratch_d = dalloc<double>(o, (size_t)128 * sh.Bp);
  r->rev_part = dalloc<float>(o, (size_t)std::max(1, r->g->dev.rev_num_slots) * sh.Bp);
  r->rev_cnt = dalloc<int32_t>(o, (size_t)sh.M * std::max(1, sh.Bp / 32));  // per (class, warp seed slice)
  r->rev_cursor = dalloc<int32_t>(o, (size_t)(r->K + 2) * std::max(1, sh.Bp / 128));
  r->dbg_p = nullptr;

  // cost model
  std::vector<float> uf(sh.N);
  std::vector<double> ud(cost->u, cost->u + sh.N);
  for (int i = 0; i < sh.N; ++i) uf[i] = (float)cost->u[i];
  r->u_f = upload(o, uf);
  r->u_d = upload(o, ud);
  if (r->cost_kind != SMOOTHE_COST_LINEAR) {
    r->p = dalloc<float>(o, NB);
    r->gp = dalloc<float>(o, NB);
    r->sbin = dalloc<float>(o, NB);
  }
  if (r->cost_kind == SMOOTHE_COST_QUADRATIC) {
    // symmetric neighbour lists: pair (i, j, w) appears as j in nbr(i) and i in nbr(j)
    std::vector<int32_t> ptr(sh.N + 1, 0);
    for (int64_t e = 0; e < cost->quad_nnz; ++e) {
      ptr[cost->quad_i[e] + 1]++;
      ptr[cost->quad_j[e] + 1]++;
    }
    for (int i = 0; i < sh.N; ++i) ptr[i + 1] += ptr[i];
    std::vector<int32_t> nbr(ptr[sh.N]), fill(ptr.begin(), ptr.end() - 1);
    std::vector<float> w(ptr[sh.N]);
    for (int64_t e = 0; e < cost->quad_nnz; ++e) {
      const int a = cost->quad_i[e], b = cost->quad_j[e];
      w[fill[a]] = (float)cost->quad_w[e];
      nbr[fill[a]++] = b;
      w[fill[b]] = (float)cost->quad_w[e];
      nbr[fill[b]++] = a;
    }
    r->q_ptr = upload(o, ptr);
    r->q_nbr = upload(o, nbr);
    r->q_w = upload(o, w);
  }
  if (r->cost_kind == SMOOTHE_COST_MLP) {
    const int H1 = r->H1, H2 = r->H2;
    r->W1 = upload(o, std::vector<float>(cost->W1, cost->W1 + (size_t)H1 * sh.N));
    // W1 in the TMA layer-1 kernel's tile order (constant for the run)
    r->W1t = upload(o, mlp_w1_tiles(cost->W1, H1, sh.N));
    r->W1b = upload(o, mlp_w1_back_tiles(cost->W1, H1, sh.N));
    r->b1 = upload(o, std::vector<float>(cost->b1, cost->b1 + H1));
    r->W2 = upload(o, std::vector<float>(cost->W2, cost->W2 + (size_t)H2 * H1));
    r->b2 = upload(o, std::vector<float>(cost->b2, cost->b2 + H2));
    r->W3 = upload(o, std::vector<float>(cost->W3, cost->W3 + H2));
    r->b3 = upload(o, std::vector<float>(cost->b3, cost->b3 + 1));
    r->nsplit = mlp_nsplit(r->device);
    r->z1_part = dalloc<float>(o, (size_t)r->nsplit * 128 * sh.Bp);
    r->z1 = dalloc<float>(o, (size_t)H1 * sh.Bp);
    if (r->overlap) {
      r->z1_part_d = dalloc<float>(o, (size_t)r->nsplit * 128 * sh.Bp);
      r->z1_d = dalloc<float>(o, (size_t)H1 * sh.Bp);
    }
    r->gz1 = dalloc<float>(o, (size_t)H1 * sh.Bp);
  }
}

void init_state(smoothe_run* r) {
  const Shape& sh = r->sh;
  cudaStream_t s = r->stream;
  const size_t MB = (size_t)sh.M * sh.Bp;
  launch_theta_init(s, sh, r->opt.rng_key, r->opt.seed_begin, r->theta, r->m, r->v);
  SM_CUDA(cudaMemsetAsync(r->cp + (size_t)sh.N * sh.Bp, 0, sizeof(float) * sh.Bp, s));
  // version 0 in the pools (never overwritten: sweeps take rows from M on):
  // q^0 = e_root; pi = 1; am = the first parent, -1 for the root, whose rows
  // therefore match no e-node, so padding slots (which point at the root) take
  // no correlated term
  launch_pool_version0(s, sh, r->g->dev, r->sw);
  SM_CUDA(cudaMemsetAsync(r->sw.abort_flag, 0, sizeof(int32_t) * 4, s));
  SM_CUDA(cudaMemsetAsync(r->gq[0], 0, sizeof(float) * MB, s));
  SM_CUDA(cudaMemsetAsync(r->gq[1], 0, sizeof(float) * MB, s));
  SM_CUDA(cudaMemsetAsync(r->pen, 0, sizeof(float), s));
  SM_CUDA(cudaMemsetAsync(r->fextra, 0, sizeof(double) * sh.Bp, s));
  SM_CUDA(cudaMemsetAsync(r->counter, 0, sizeof(int32_t), s));
  SM_CUDA(cudaMemsetAsync(r->rev_cnt, 0, sizeof(int32_t) * sh.M * std::max(1, sh.Bp / 32), s));
  SM_CUDA(cudaMemsetAsync(r->trace, 0xff, sizeof(double) * 4 * kTraceCap, s));  // NaN: not run
  const double init_best[6] = {INFINITY, -1.0, -1.0, 0.0, INFINITY, -1.0};
  SM_CUDA(cudaMemcpyAsync(r->best, init_best, sizeof(init_best), cudaMemcpyHostToDevice, s));
  SM_CUDA(cudaMemsetAsync(r->best_choice, 0xff, sizeof(int32_t) * sh.M, s));
  SM_CUDA(cudaStreamSynchronize(s));
}

void copy_rows_d2h(float* dst, const float* src, int rows, int B, int Bp, cudaStream_t s) {
  if (!dst) return;
  SM_CUDA(cudaMemcpy2DAsync(dst, sizeof(float) * B, src, sizeof(float) * Bp, sizeof(float) * B,
                            rows, cudaMemcpyDeviceToHost, s));
}

void copy_rows_h2d(float* dst, const float* src, int rows, int B, int Bp, cudaStream_t s) {
  SM_CUDA(cudaMemcpy2DAsync(dst, sizeof(float) * Bp, src, sizeof(float) * B, sizeof(float) * B,
                            rows, cudaMemcpyHostToDevice, s));
}

}  // namespace

// ===========================================================================
// C ABI
// ===========================================================================
extern "C" {

const char* smoothe_last_error(void) { return g_last_error.c_str(); }
const char* smoothe_version(void) { return "smoothe-b200 0.1 (sm_100a)"; }

smoothe_status smoothe_load_egraph(int32_t num_classes, int32_t num_nodes, const int32_t* class_ptr,
                                   const int64_t* child_ptr, const int32_t* child_class,
                                   int32_t root_class, int device_ordinal, smoothe_egraph** out) {
  if (!out) {
    set_error("NULL out");
    return SMOOTHE_E_INVALID_ARG;
  }
  *out = nullptr;
  smoothe_egraph* g = nullptr;
  auto owner = new (std::nothrow) smoothe_egraph_dev_owner();
  const bool timing = std::getenv("SMOOTHE_LOAD_TIMING") != nullptr;
  auto t0 = std::chrono::steady_clock::now();
  auto lap = [&](const char* what) {
    if (!timing) return;
    const auto t1 = std::chrono::steady_clock::now();
    std::fprintf(stderr, "[load] %-22s %.4f s\n", what, std::chrono::duration<double>(t1 - t0).count());
    t0 = t1;
  };
  smoothe_status st = guarded(nullptr, [&] {
    g = new smoothe_egraph();
    build_host_graph(num_classes, num_nodes, class_ptr, child_ptr, child_class, root_class, g->host);
    lap("host analysis (total)");
    g->device = device_ordinal;
    if (device_ordinal >= 0) {
      int ndev = 0;
      SM_CUDA(cudaGetDeviceCount(&ndev));
      SM_REQUIRE(device_ordinal < ndev, SMOOTHE_E_INVALID_ARG, "device ordinal out of range");
      SM_CUDA(cudaSetDevice(device_ordinal));
      // (two attribute queries: cudaGetDeviceProperties took ~150 ms of the load)
      int major = 0, minor = 0;
      SM_CUDA(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, device_ordinal));
      SM_CUDA(cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, device_ordinal));
      SM_REQUIRE(major == 10, SMOOTHE_E_CUDA,
                 "libsmoothe is built for sm_100a; device has sm_" + std::to_string(major) +
                     std::to_string(minor));
      lap("device query");
      const HostGraph& h = g->host;
      DevGraph& d = g->dev;
      int64_t& b = d.bytes;
      auto uploads = [&](Arena& o) {
        d.class_ptr = upload(o, h.class_ptr, &b);
        d.child_ptr = upload(o, h.child_ptr, &b);
        {  // padded with the root id so batched kernels may read up to 8 past E
          std::vector<int32_t> padded(h.child_class);
          padded.resize(h.child_class.size() + 8, h.root);
          d.child_class = upload(o, padded, &b);
        }
        d.par_ptr = upload(o, h.par_ptr, &b);
        d.par_node = upload(o, h.par_node, &b);
        d.par_class = upload(o, h.par_class, &b);
        d.scc_class_ptr = upload(o, h.scc_class_ptr, &b);
        d.scc_class = upload(o, h.scc_class, &b);
        d.scc_of_class = upload(o, h.scc_of_class, &b);
        d.ent_ptr = upload(o, h.ent_ptr, &b);
        d.ent_i = upload(o, h.ent_i, &b);
        d.ent_j = upload(o, h.ent_j, &b);
        d.ent_node_ptr = upload(o, h.ent_node_ptr, &b);
        d.ent_node = upload(o, h.ent_node, &b);
        d.slot_ptr = upload(o, h.slot_ptr, &b);
        d.slot_node = upload(o, h.slot_node, &b);
        d.slot_iloc = upload(o, h.slot_iloc, &b);
        d.slot_jptr = upload(o, h.slot_jptr, &b);
        d.slot_jloc = upload(o, h.slot_jloc, &b);
        d.node_slot = upload(o, h.node_slot, &b);
        d.pad_child_ptr = upload(o, h.pad_child_ptr, &b);
        d.pad_child = upload(o, h.pad_child, &b);
        d.pad_par_ptr = upload(o, h.pad_par_ptr, &b);
        d.pad_par = upload(o, h.pad_par, &b);
        d.pad_batch_node = upload(o, h.pad_batch_node, &b);
        d.big_class = upload(o, h.big_class, &b);
        d.dmin = upload(o, h.dmin, &b);
        d.cls_child_ptr = upload(o, h.cls_child_ptr, &b);
        d.cls_child = upload(o, h.cls_child, &b);
        d.pad_cedge = upload(o, h.pad_cedge, &b);
        d.cedge_class = upload(o, h.cedge_class, &b);
        d.cedge_ptr = upload(o, h.cedge_ptr, &b);
        d.cedge_node = upload(o, h.cedge_node, &b);
        d.witem = upload(o, h.witem, &b);
        d.wmulti = upload(o, h.wmulti, &b);
        d.wmulti_ptr = upload(o, h.wmulti_ptr, &b);
        d.num_witems = (int32_t)(h.witem.size() / 4);
        d.num_wmulti = (int32_t)h.wmulti.size();
        d.w_num_slots = h.w_num_slots;
        d.num_cedge = (int64_t)h.cls_child.size();
        d.num_big = (int32_t)h.big_class.size();
        d.rev_item = upload(o, h.rev_item, &b);
        d.rev_class_item_ptr = upload(o, h.rev_class_item_ptr, &b);
        d.num_rev_items = (int32_t)(h.rev_item.size() / 8);
        d.rev_num_slots = h.rev_num_slots;
        d.lvl_cptr = upload(o, h.lvl_cptr, &b);
        d.lvl_class = upload(o, h.lvl_class, &b);
        d.lvl_sptr = upload(o, h.lvl_sptr, &b);
        d.lvl_scc = upload(o, h.lvl_scc, &b);
      };
      Arena measure;
      uploads(measure);
      Arena arena;
      SM_CUDA(cudaMalloc(&arena.base, measure.used));
      owner->owned.push_back(arena.base);
      b = 0;
      uploads(arena);
      lap("device upload");
    }
  });
  if (st != SMOOTHE_OK) {
    if (owner) {
      for (void* p : owner->owned) cudaFree(p);
      delete owner;
    }
    delete g;
    return st;
  }
  g->owned = std::move(owner->owned);  // freed by smoothe_free_egraph
  delete owner;
  *out = g;
  return SMOOTHE_OK;
}

smoothe_status smoothe_egraph_get_info(const smoothe_egraph* g, smoothe_egraph_info* out) {
  if (!g || !out) {
    set_error("NULL argument");
    return SMOOTHE_E_INVALID_ARG;
  }
  const HostGraph& h = g->host;
  out->num_classes = h.M;
  out->num_nodes = h.N;
  out->num_edges = h.E;
  out->root = h.root;
  out->K_auto = h.K_auto;
  out->num_scc = h.num_scc;
  out->scc_classes = h.scc_classes;
  out->scc_max = h.scc_max;
  out->max_class_size = h.max_class_size;
  out->max_in_degree = h.max_in_degree;
  out->device = g->device;
  out->device_bytes = g->dev.bytes;
  return SMOOTHE_OK;
}

smoothe_status smoothe_egraph_get_scc(const smoothe_egraph* g, int32_t* scc_of_class) {
  if (!g || !scc_of_class) {
    set_error("NULL argument");
    return SMOOTHE_E_INVALID_ARG;
  }
  std::memcpy(scc_of_class, g->host.scc_of_class.data(), sizeof(int32_t) * g->host.M);
  return SMOOTHE_OK;
}

smoothe_status smoothe_greedy(smoothe_egraph* g, const double* u, int32_t* choice,
                             double* class_cost, smoothe_greedy_result* out) {
  return guarded(nullptr, [&] {
    SM_REQUIRE(g && u && out, SMOOTHE_E_INVALID_ARG, "NULL argument");
    SM_REQUIRE(g->device >= 0, SMOOTHE_E_STATE, "host-only e-graph (device_ordinal = -1)");
    SM_CUDA(cudaSetDevice(g->device));
    const HostGraph& hg = g->host;
    const int M = hg.M, grid = greedy_grid(g->device);
    std::vector<void*> o;
    struct Free {
      std::vector<void*>& o;
      cudaStream_t s = nullptr;
      ~Free() {
        if (s) cudaStreamDestroy(s);
        for (void* p : o) cudaFree(p);
      }
    } fr{o};
    SM_CUDA(cudaStreamCreateWithFlags(&fr.s, cudaStreamNonBlocking));
    std::vector<double> uh(u, u + hg.N);
    // the worklist's fixpoint needs u >= 0: a negative cost on a cycle would
    // lower a class's key on every pass (Bellman-Ford without termination)
    for (int i = 0; i < hg.N; ++i)
      SM_REQUIRE(std::isfinite(uh[i]) && uh[i] >= 0.0, SMOOTHE_E_INVALID_ARG,
                 "greedy needs finite non-negative costs u");
    double* ud = upload(o, uh);
    double* cost = dalloc<double>(o, M);
    int32_t* ints = dalloc<int32_t>(o, (size_t)6 * M + 3 + grid);
    int32_t *height = ints, *sel = ints + M, *reach = ints + 2 * (size_t)M,
            *frontier = ints + 3 * (size_t)M, *chout = ints + 5 * (size_t)M,
            *counts = ints + 6 * (size_t)M, *npart = counts + 3;
    double* part = dalloc<double>(o, (size_t)grid + 4);
    double* result = part + grid;
    SM_CUDA(cudaMemsetAsync(cost, 0, sizeof(double) * M, fr.s));
    SM_CUDA(cudaMemsetAsync(ints, 0, sizeof(int32_t) * ((size_t)6 * M + 3 + grid), fr.s));
    launch_greedy(fr.s, hg, g->dev, grid, ud, cost, height, sel, reach, frontier, counts, part,
                  npart, chout, result);
    double res[4];
    SM_CUDA(cudaMemcpyAsync(res, result, sizeof(res), cudaMemcpyDeviceToHost, fr.s));
    if (choice)
      SM_CUDA(cudaMemcpyAsync(choice, chout, sizeof(int32_t) * M, cudaMemcpyDeviceToHost, fr.s));
    if (class_cost)
      SM_CUDA(cudaMemcpyAsync(class_cost, cost, sizeof(double) * M, cudaMemcpyDeviceToHost, fr.s));
    SM_CUDA(cudaStreamSynchronize(fr.s));
    if (class_cost)  // classes the root cannot reach are not evaluated
      for (int j = 0; j < M; ++j)
        if (hg.dmin[j] == INT32_MAX) class_cost[j] = INFINITY;
    out->dag_cost = res[0];
    out->root_cost = res[1];
    out->valid = (int32_t)res[2];
    out->selected_classes = (int32_t)res[3];
  });
}

smoothe_status smoothe_run_warm_start(smoothe_run* run, const int32_t* choice, float bias) {
  return guarded(run, [&] {
    check_run(run);
    SM_REQUIRE(choice, SMOOTHE_E_INVALID_ARG, "NULL choice");
    const Shape& sh = run->sh;
    for (int j = 0; j < sh.M; ++j)
      SM_REQUIRE(choice[j] < 0 || (choice[j] >= run->g->host.class_ptr[j] &&
                                   choice[j] < run->g->host.class_ptr[j + 1]),
                 SMOOTHE_E_INVALID_ARG, "choice[j] is not an e-node of class j");
    struct Tmp {
      std::vector<void*> o;
      ~Tmp() {
        for (void* p : o) cudaFree(p);
      }
    } tmp;
    int32_t* d = dalloc<int32_t>(tmp.o, sh.M);
    SM_CUDA(cudaMemcpyAsync(d, choice, sizeof(int32_t) * sh.M, cudaMemcpyHostToDevice,
                            run->stream));
    launch_warm_start(run->stream, sh.M, sh.Bp, d, bias, run->theta);
    SM_CUDA(cudaStreamSynchronize(run->stream));
  });
}

smoothe_status smoothe_options_default(smoothe_options* opt) {
  if (!opt) {
    set_error("NULL options");
    return SMOOTHE_E_INVALID_ARG;
  }
  std::memset(opt, 0, sizeof(*opt));
  opt->assumption = SMOOTHE_AGG_HYBRID;
  opt->prop_iters = -1;
  opt->lambda = 1.0;
  opt->penalty_group = 1;
  opt->lr = 0.1;
  opt->beta1 = 0.9;
  opt->beta2 = 0.999;
  opt->eps = 1e-8;
  opt->optimizer = 0;
  opt->use_graphs = 1;
  return SMOOTHE_OK;
}

smoothe_status smoothe_run_create(smoothe_egraph* g, const smoothe_cost_model* cost,
                                  int32_t num_seeds, const smoothe_options* opt,
                                  smoothe_run** out) {
  if (!out) {
    set_error("NULL out");
    return SMOOTHE_E_INVALID_ARG;
  }
  *out = nullptr;
  smoothe_run* r = new (std::nothrow) smoothe_run();
  if (!r) return SMOOTHE_E_OOM;
  smoothe_status st = guarded(nullptr, [&] {
    SM_REQUIRE(g && cost && opt && cost->u, SMOOTHE_E_INVALID_ARG, "NULL argument");
    SM_REQUIRE(g->device >= 0, SMOOTHE_E_STATE, "host-only e-graph (device_ordinal = -1)");
    SM_REQUIRE(num_seeds > 0, SMOOTHE_E_INVALID_ARG, "num_seeds must be > 0");
    SM_REQUIRE(opt->penalty_group > 0 && num_seeds % opt->penalty_group == 0,
               SMOOTHE_E_INVALID_ARG, "penalty_group must divide num_seeds (S13)");
    SM_REQUIRE(opt->assumption >= 0 && opt->assumption <= 2, SMOOTHE_E_INVALID_ARG, "bad assumption");
    SM_REQUIRE(opt->optimizer == 0 || opt->optimizer == 1, SMOOTHE_E_INVALID_ARG, "bad optimizer");
    SM_REQUIRE(cost->kind >= 0 && cost->kind <= 2, SMOOTHE_E_INVALID_ARG, "bad cost kind");
    r->g = g;
    r->opt = *opt;
    r->device = g->device;
    r->owned.device = g->device;
    SM_CUDA(cudaSetDevice(r->device));
    const HostGraph& hg = g->host;
    Shape& sh = r->sh;
    sh.M = hg.M;
    sh.N = hg.N;
    sh.root = hg.root;
    sh.B = num_seeds;
    sh.Bp = num_seeds <= 32 ? 32 : num_seeds <= 64 ? 64 : ((num_seeds + 127) / 128) * 128;
    sh.W = sh.Bp / 32;
    r->K = opt->prop_iters < 0 ? hg.K_auto : opt->prop_iters;
    r->G = opt->penalty_group;
    r->ngroups = num_seeds / r->G;
    r->agg = opt->assumption == SMOOTHE_AGG_INDEPENDENT   ? Agg{1.f, 0.f}
             : opt->assumption == SMOOTHE_AGG_CORRELATED ? Agg{0.f, 1.f}
                                                          : Agg{0.5f, 0.5f};
    r->cost_kind = cost->kind;
    if (cost->kind == SMOOTHE_COST_QUADRATIC) {
      SM_REQUIRE(cost->quad_nnz >= 0 && (cost->quad_nnz == 0 || (cost->quad_i && cost->quad_j && cost->quad_w)),
                 SMOOTHE_E_INVALID_ARG, "quadratic pairs missing");
      for (int64_t e = 0; e < cost->quad_nnz; ++e)
        SM_REQUIRE(cost->quad_i[e] >= 0 && cost->quad_i[e] < sh.N && cost->quad_j[e] >= 0 &&
                       cost->quad_j[e] < sh.N && cost->quad_i[e] != cost->quad_j[e],
                   SMOOTHE_E_INVALID_ARG, "bad quadratic pair");
    }
    if (cost->kind == SMOOTHE_COST_MLP) {
      SM_REQUIRE(cost->W1 && cost->b1 && cost->W2 && cost->b2 && cost->W3 && cost->b3,
                 SMOOTHE_E_INVALID_ARG, "MLP weights missing");
      SM_REQUIRE(cost->mlp_hidden1 > 0 && cost->mlp_hidden1 <= 64 && cost->mlp_hidden2 > 0 &&
                     cost->mlp_hidden2 <= 16,
                 SMOOTHE_E_INVALID_ARG, "MLP hidden sizes must be <= 64 and <= 16");
      r->H1 = cost->mlp_hidden1;
      r->H2 = cost->mlp_hidden2;
    }
    SM_CUDA(cudaStreamCreateWithFlags(&r->stream, cudaStreamNonBlocking));
    {
      const char* ov = std::getenv("SMOOTHE_DECODE_OVERLAP");
      r->overlap = !(ov && ov[0] == '0');
    }
    SM_CUDA(cudaStreamCreateWithFlags(&r->stream_body, cudaStreamNonBlocking));
    SM_CUDA(cudaStreamCreateWithFlags(&r->stream_body2, cudaStreamNonBlocking));
    if (r->overlap) {
      SM_CUDA(cudaStreamCreateWithFlags(&r->stream2, cudaStreamNonBlocking));
      SM_CUDA(cudaEventCreateWithFlags(&r->ev_fork, cudaEventDisableTiming));
      SM_CUDA(cudaEventCreateWithFlags(&r->ev_join, cudaEventDisableTiming));
      SM_CUDA(cudaEventCreateWithFlags(&r->ev_pen, cudaEventDisableTiming));
    }
    r->coop_grid = decode_grid(r->device);
    alloc_state(r, cost);
    SM_CUDA(cudaEventCreate(&r->ev_start));
    r->ev_step.resize(4096);
    for (auto& e : r->ev_step) SM_CUDA(cudaEventCreate(&e));
    r->t_create = std::chrono::steady_clock::now();
    SM_CUDA(cudaEventRecord(r->ev_start, r->stream));
    init_state(r);
    g->refcount++;
  });
  if (st != SMOOTHE_OK) {
    runmem_recycle(r->owned);
    if (r->stream) cudaStreamDestroy(r->stream);
    delete r;
    return st;
  }
  *out = r;
  return SMOOTHE_OK;
}

smoothe_status smoothe_run_steps(smoothe_run* run, int32_t steps) {
  return guarded(run, [&] {
    check_run(run);
    SM_REQUIRE(steps >= 0, SMOOTHE_E_INVALID_ARG, "steps must be >= 0");
    cudaStream_t user = (cudaStream_t)run->opt.cuda_stream;
    cudaEvent_t join = nullptr;
    if (user) {  // order after the caller's stream
      SM_CUDA(cudaEventCreateWithFlags(&join, cudaEventDisableTiming));
      SM_CUDA(cudaEventRecord(join, user));
      SM_CUDA(cudaStreamWaitEvent(run->stream, join, 0));
    }
    const bool checks = run->opt.patience > 0 || run->opt.time_limit_s > 0;
    const bool growable = run->sw.cap < ((int64_t)run->K + 1) * run->sh.M;
    int32_t left = steps;
    while (left > 0) {
      int32_t done = 0;
      bool stop = false;
      for (; done < left && !stop; ++done) {
        run_one_step(run);
        if (checks && ((done + 1) % 8 == 0 || done + 1 == left)) {
          double best[4];
          SM_CUDA(cudaMemcpyAsync(best, run->best, sizeof(best), cudaMemcpyDeviceToHost, run->stream));
          SM_CUDA(cudaStreamSynchronize(run->stream));
          if (run->opt.patience > 0 && best[3] >= run->opt.patience) stop = true;
          const double el = std::chrono::duration<double>(std::chrono::steady_clock::now() - run->t_create).count();
          if (run->opt.time_limit_s > 0 && el >= run->opt.time_limit_s) stop = true;
        }
      }
      // steps aborted by a full version pool are repeated on grown pools
      const int aborted = growable ? pool_check_grow(run) : 0;
      run->steps_run -= aborted;
      left = stop ? 0 : aborted;
    }
    if (user) {
      SM_CUDA(cudaEventRecord(join, run->stream));
      SM_CUDA(cudaStreamWaitEvent(user, join, 0));
      SM_CUDA(cudaEventDestroy(join));
    }
  });
}

smoothe_status smoothe_run_synchronize(smoothe_run* run) {
  return guarded(run, [&] {
    check_run(run);
    SM_CUDA(cudaStreamSynchronize(run->stream));
  });
}

smoothe_status smoothe_optimize(smoothe_egraph* g, const smoothe_cost_model* cost, int32_t num_seeds,
                                int32_t steps, const smoothe_options* opt, smoothe_run** out) {
  smoothe_status st = smoothe_run_create(g, cost, num_seeds, opt, out);
  if (st != SMOOTHE_OK) return st;
  st = smoothe_run_steps(*out, steps);
  if (st != SMOOTHE_OK) return st;
  return smoothe_run_synchronize(*out);
}

smoothe_status smoothe_extract(smoothe_run* run, int32_t* choice, smoothe_summary* out) {
  bool valid = false;
  smoothe_status st = guarded(run, [&] {
    check_run(run);
    SM_CUDA(cudaStreamSynchronize(run->stream));
    double best[4], loss = 0.0;
    SM_CUDA(cudaMemcpy(best, run->best, sizeof(best), cudaMemcpyDeviceToHost));
    SM_CUDA(cudaMemcpy(&loss, run->loss, sizeof(double), cudaMemcpyDeviceToHost));
    valid = std::isfinite(best[0]);
    if (choice) SM_CUDA(cudaMemcpy(choice, run->best_choice, sizeof(int32_t) * run->sh.M, cudaMemcpyDeviceToHost));
    if (out) {
      std::memset(out, 0, sizeof(*out));
      out->best_cost = best[0];
      out->best_step = (int32_t)best[1];
      out->best_seed = (int64_t)best[2];
      out->valid = valid ? 1 : 0;
      out->steps_run = run->steps_run;
      out->K = run->K;
      out->last_loss = loss;
      out->graph_mode = run->graph_failed ? -1 : (run->graph_steps > 0 ? 1 : 0);
      int32_t f[4];
      SM_CUDA(cudaMemcpy(f, run->sw.abort_flag, sizeof(f), cudaMemcpyDeviceToHost));
      out->pool_rows = run->sw.cap;
      out->pool_peak_rows = std::max<int64_t>(run->pool_high, f[2]);
      out->pool_grows = run->pool_grows;
      float ms = 0.f;
      const int bs = out->best_step;
      if (valid && bs >= 0 && (size_t)bs < run->ev_step.size() && bs < run->steps_run) {
        SM_CUDA(cudaEventElapsedTime(&ms, run->ev_start, run->ev_step[bs]));
        out->time_to_best_s = ms * 1e-3;
      } else {
        out->time_to_best_s = -1.0;
      }
      const int last = std::min<int>(run->steps_run, (int)run->ev_step.size()) - 1;
      if (last >= 0) {
        SM_CUDA(cudaEventElapsedTime(&ms, run->ev_start, run->ev_step[last]));
        out->step_time_s = ms * 1e-3 / (last + 1);
      }
    }
  });
  if (st == SMOOTHE_OK && !valid) {
    set_error("no valid extraction sampled");
    return SMOOTHE_E_NO_VALID;
  }
  return st;
}

smoothe_status smoothe_debug_step(smoothe_run* run, const float* theta_in, const float* m_in,
                                  const float* v_in, int32_t step_index, smoothe_debug_out* dump) {
  return guarded(run, [&] {
    check_run(run);
    SM_REQUIRE(dump != nullptr, SMOOTHE_E_INVALID_ARG, "NULL dump");
    SM_REQUIRE(step_index >= 0, SMOOTHE_E_INVALID_ARG, "step_index must be >= 0");
    const Shape& sh = run->sh;
    cudaStream_t s = run->stream;
    const size_t NB = (size_t)sh.N * sh.Bp;
    if (theta_in) copy_rows_h2d(run->theta, theta_in, sh.N, sh.B, sh.Bp, s);
    if (m_in) copy_rows_h2d(run->m, m_in, sh.N, sh.B, sh.Bp, s);
    else SM_CUDA(cudaMemsetAsync(run->m, 0, sizeof(float) * NB, s));
    if (v_in) copy_rows_h2d(run->v, v_in, sh.N, sh.B, sh.Bp, s);
    else SM_CUDA(cudaMemsetAsync(run->v, 0, sizeof(float) * NB, s));
    SM_CUDA(cudaMemcpyAsync(run->counter, &step_index, sizeof(int32_t), cudaMemcpyHostToDevice, s));
    // debug scratch
    std::vector<void*> scratch;
    run->dbg_p = run->cost_kind == SMOOTHE_COST_LINEAR ? dalloc<float>(scratch, NB) : nullptr;
    run->dbg_gth = dalloc<float>(scratch, NB);
    run->dbg_gcp = dalloc<float>(scratch, NB);
    run->dbg_dcost = dalloc<double>(scratch, sh.Bp);
    run->dbg_valid = dalloc<uint8_t>(scratch, sh.Bp);
    std::vector<float> theta_keep;
    run->debug = true;
    try {
      // the step overwrites theta; keep the input's cp etc. from the step itself
      // (a step aborted by a full version pool left theta, m, v and the step
      // counter as they were: grow the pools and take it again)
      enqueue_step(run);
      while (pool_check_grow(run) > 0) enqueue_step(run);
    } catch (...) {
      run->debug = false;
      for (void* p : scratch) cudaFree(p);
      throw;
    }
    run->debug = false;
    const float* pdev = run->cost_kind == SMOOTHE_COST_LINEAR ? run->dbg_p : run->p;
    copy_rows_d2h(dump->cp, run->cp, sh.N, sh.B, sh.Bp, s);
    copy_rows_d2h(dump->qK, run->sw.qbuf[run->K & 1], sh.M, sh.B, sh.Bp, s);
    copy_rows_d2h(dump->p, pdev, sh.N, sh.B, sh.Bp, s);
    copy_rows_d2h(dump->grad_cp, run->dbg_gcp, sh.N, sh.B, sh.Bp, s);
    copy_rows_d2h(dump->grad_theta, run->dbg_gth, sh.N, sh.B, sh.Bp, s);
    copy_rows_d2h(dump->theta_out, run->theta, sh.N, sh.B, sh.Bp, s);
    copy_rows_d2h(dump->m_out, run->m, sh.N, sh.B, sh.Bp, s);
    copy_rows_d2h(dump->v_out, run->v, sh.N, sh.B, sh.Bp, s);
    // q stack / routes from the version pools: per seed chunk, the row of
    // class j at sweep t is its last version listed up to sweep t (rows
    // [0, M): version 0), rebuilt from the forward's lists on the host
    if (dump->qstack || dump->route) {
      const SweepState& w = run->sw;
      const int K = run->K;
      std::vector<int32_t> ln((size_t)w.nchunk * (K + 2));
      std::vector<int4> lst((size_t)w.nchunk * (K + 1) * sh.M);
      std::vector<float> qp(dump->qstack ? (size_t)w.cap * w.wc : 0);
      std::vector<int32_t> ap(dump->route ? (size_t)w.cap * w.wc : 0);
      SM_CUDA(cudaMemcpyAsync(ln.data(), w.list_n, sizeof(int32_t) * ln.size(), cudaMemcpyDeviceToHost, s));
      SM_CUDA(cudaMemcpyAsync(lst.data(), w.list, sizeof(int4) * lst.size(), cudaMemcpyDeviceToHost, s));
      std::vector<int32_t> row(sh.M);
      for (int c = 0; c < w.nchunk; ++c) {
        if (dump->qstack)
          SM_CUDA(cudaMemcpyAsync(qp.data(), w.qpool + (size_t)c * w.cap * w.wc,
                                  sizeof(float) * qp.size(), cudaMemcpyDeviceToHost, s));
        if (dump->route)
          SM_CUDA(cudaMemcpyAsync(ap.data(), w.apool + (size_t)c * w.cap * w.wc,
                                  sizeof(int32_t) * ap.size(), cudaMemcpyDeviceToHost, s));
        SM_CUDA(cudaStreamSynchronize(s));
        const int b0 = c * w.wc, b1 = std::min(sh.B, b0 + w.wc);
        for (int j = 0; j < sh.M; ++j) row[j] = j;
        for (int t = 0; t <= K; ++t) {
          if (t > 0)
            for (int i = 0; i < ln[(size_t)c * (K + 2) + t]; ++i) {
              const int4 e = lst[((size_t)c * (K + 1) + t) * sh.M + i];
              row[e.x] = e.z;
            }
          for (int j = 0; j < sh.M; ++j) {
            const size_t src = (size_t)row[j] * w.wc;
            if (dump->qstack)
              for (int b = b0; b < b1; ++b)
                dump->qstack[((size_t)t * sh.M + j) * sh.B + b] = qp[src + (b - b0)];
            if (dump->route && t > 0)  // route row t - 1 = sweep t
              for (int b = b0; b < b1; ++b)
                dump->route[((size_t)(t - 1) * sh.M + j) * sh.B + b] = ap[src + (b - b0)];
          }
        }
      }
    }
    if (dump->f) SM_CUDA(cudaMemcpyAsync(dump->f, run->ftot, sizeof(double) * sh.B, cudaMemcpyDeviceToHost, s));
    if (dump->h) {
      if (run->g->host.num_scc > 0)
        SM_CUDA(cudaMemcpyAsync(dump->h, run->h, sizeof(double) * run->ngroups, cudaMemcpyDeviceToHost, s));
      else
        std::memset(dump->h, 0, sizeof(double) * run->ngroups);
    }
    if (dump->loss) SM_CUDA(cudaMemcpyAsync(dump->loss, run->loss, sizeof(double), cudaMemcpyDeviceToHost, s));
    if (dump->choice)
      SM_CUDA(cudaMemcpy2DAsync(dump->choice, sizeof(int32_t) * sh.B, run->choice, sizeof(int32_t) * sh.Bp,
                                sizeof(int32_t) * sh.B, sh.M, cudaMemcpyDeviceToHost, s));
    if (dump->valid) SM_CUDA(cudaMemcpyAsync(dump->valid, run->dbg_valid, sh.B, cudaMemcpyDeviceToHost, s));
    if (dump->disc_cost)
      SM_CUDA(cudaMemcpyAsync(dump->disc_cost, run->dbg_dcost, sizeof(double) * sh.B, cudaMemcpyDeviceToHost, s));
    if (dump->sweeps) {
      std::vector<int32_t> lc(sh.Bp, run->K - 1);
      if (run->sw.converge) {
        SM_CUDA(cudaMemcpyAsync(lc.data(), run->sw.lastchg, sizeof(int32_t) * sh.Bp,
                                cudaMemcpyDeviceToHost, s));
        SM_CUDA(cudaStreamSynchronize(s));
      }
      for (int b = 0; b < sh.B; ++b) dump->sweeps[b] = std::min(run->K, lc[b] + 1);
    }
    std::vector<uint32_t> rbits;
    if (dump->reached) {
      rbits.resize((size_t)sh.M * sh.W);
      SM_CUDA(cudaMemcpyAsync(rbits.data(), run->reach, sizeof(uint32_t) * rbits.size(), cudaMemcpyDeviceToHost, s));
    }
    SM_CUDA(cudaStreamSynchronize(s));
    if (dump->reached)
      for (int j = 0; j < sh.M; ++j)
        for (int b = 0; b < sh.B; ++b)
          dump->reached[(size_t)j * sh.B + b] = (rbits[(size_t)j * sh.W + (b >> 5)] >> (b & 31)) & 1u;
    if ((size_t)run->steps_run < run->ev_step.size())
      SM_CUDA(cudaEventRecord(run->ev_step[run->steps_run], s));
    for (void* p : scratch) SM_CUDA(cudaFree(p));
    run->dbg_p = run->dbg_gth = run->dbg_gcp = nullptr;
    run->dbg_dcost = nullptr;
    run->dbg_valid = nullptr;
    run->steps_run++;
  });
}

smoothe_status smoothe_get_theta(smoothe_run* run, float* theta) {
  return guarded(run, [&] {
    check_run(run);
    SM_REQUIRE(theta, SMOOTHE_E_INVALID_ARG, "NULL theta");
    copy_rows_d2h(theta, run->theta, run->sh.N, run->sh.B, run->sh.Bp, run->stream);
    SM_CUDA(cudaStreamSynchronize(run->stream));
  });
}

smoothe_status smoothe_run_get_trace(smoothe_run* run, double* out, int32_t max_steps,
                                     int32_t* n_out) {
  return guarded(run, [&] {
    check_run(run);
    SM_REQUIRE(out && n_out && max_steps >= 0, SMOOTHE_E_INVALID_ARG, "bad trace arguments");
    SM_CUDA(cudaStreamSynchronize(run->stream));
    const int n = std::min({run->steps_run, kTraceCap, (int)max_steps});
    if (n > 0) SM_CUDA(cudaMemcpy(out, run->trace, sizeof(double) * 4 * n, cudaMemcpyDeviceToHost));
    *n_out = n;
  });
}

smoothe_status smoothe_get_state(smoothe_run* run, float* theta, float* m, float* v,
                                 int32_t* steps_run) {
  return guarded(run, [&] {
    check_run(run);
    if (theta) copy_rows_d2h(theta, run->theta, run->sh.N, run->sh.B, run->sh.Bp, run->stream);
    if (m) copy_rows_d2h(m, run->m, run->sh.N, run->sh.B, run->sh.Bp, run->stream);
    if (v) copy_rows_d2h(v, run->v, run->sh.N, run->sh.B, run->sh.Bp, run->stream);
    SM_CUDA(cudaStreamSynchronize(run->stream));
    if (steps_run) *steps_run = run->steps_run;
  });
}

smoothe_status smoothe_run_profile(smoothe_run* run, int32_t enable) {
  return guarded(run, [&] {
    check_run(run);
    SM_CUDA(cudaStreamSynchronize(run->stream));
    run->profiling = enable != 0;
    run->prof_ev.clear();
    for (auto& v : run->prof_kev) v.clear();
    if (run->frozen_count)
      SM_CUDA(cudaMemsetAsync(run->frozen_count, 0, 4 * sizeof(int64_t), run->stream));
    run->prof_pool_used = 0;
    std::memset(run->prof_launch, 0, sizeof(run->prof_launch));
    run->prof_launch_total = 0;
    run->prof_steps = 0;
  });
}

smoothe_status smoothe_run_get_profile(smoothe_run* run, smoothe_profile* out) {
  return guarded(run, [&] {
    check_run(run);
    SM_REQUIRE(out, SMOOTHE_E_INVALID_ARG, "NULL out");
    SM_CUDA(cudaStreamSynchronize(run->stream));
    std::memset(out, 0, sizeof(*out));
    for (const auto& ev : run->prof_ev) {
      for (int ph = 0; ph < SMOOTHE_NUM_PHASES; ++ph) {
        float ms = 0.f;
        SM_CUDA(cudaEventElapsedTime(&ms, ev[ph], ev[ph + 1]));
        out->phase_ms[ph] += ms;
      }
    }
    for (int ph = 0; ph < SMOOTHE_NUM_PHASES; ++ph) out->phase_launches[ph] = run->prof_launch[ph];
    if (run->frozen_count)
      SM_CUDA(cudaMemcpy(&out->frozen_sweeps, run->frozen_count, 4 * sizeof(int64_t),
                         cudaMemcpyDeviceToHost));
    for (int w = 0; w < 3; ++w) {
      for (const auto& ev : run->prof_kev[w]) {
        float ms = 0.f;
        SM_CUDA(cudaEventElapsedTime(&ms, ev[0], ev[1]));
        out->sweep_kernel_ms[w] += ms;
      }
      out->sweep_kernel_launches[w] = (int64_t)run->prof_kev[w].size();
    }
    out->steps = run->prof_steps;
    out->launches = run->prof_launch_total;
    out->num_seeds_padded = run->sh.Bp;
  });
}

void smoothe_release_cached_memory(int device_ordinal) { cache_release(device_ordinal); }

void smoothe_free_run(smoothe_run* run) {
  if (!run) return;
  cudaSetDevice(run->device);
  cudaStreamSynchronize(run->stream);
  if (run->graph_exec) cudaGraphExecDestroy(run->graph_exec);
  runmem_recycle(run->owned);
  for (auto e : run->ev_step) cudaEventDestroy(e);
  for (auto e : run->prof_pool) cudaEventDestroy(e);
  if (run->ev_start) cudaEventDestroy(run->ev_start);
  if (run->stream) cudaStreamDestroy(run->stream);
  if (run->stream2) cudaStreamDestroy(run->stream2);
  if (run->stream_body) cudaStreamDestroy(run->stream_body);
  if (run->stream_body2) cudaStreamDestroy(run->stream_body2);
  if (run->ev_fork) cudaEventDestroy(run->ev_fork);
  if (run->ev_join) cudaEventDestroy(run->ev_join);
  if (run->ev_pen) cudaEventDestroy(run->ev_pen);
  if (run->g) {
    run->g->refcount--;
    if (run->g->freed && run->g->refcount == 0) smoothe_free_egraph(run->g);
  }
  delete run;
}

void smoothe_free_egraph(smoothe_egraph* g) {
  if (!g) return;
  g->freed = true;
  if (g->refcount > 1) {  // runs still alive: freed when the last one goes
    g->refcount--;
    return;
  }
  if (g->device >= 0) {  // the arena holding every device array
    cudaSetDevice(g->device);
    for (void* p : g->owned) cudaFree(p);
  }
  delete g;
}

}  // extern "C"
