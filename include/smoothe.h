/* smoothe.h -- C ABI of libsmoothe.so, the B200 (sm_100a) implementation of
 * SmoothE's seed-parallel gradient step (Cai et al., ASPLOS'25).
 *
 * Citations "P<n>" are lines of the paper text /root/reference/PAPER.md;
 * readings "S<n>" of silent or garbled passages are listed in DESIGN.md.
 *
 * Conventions
 *  - Every call returns smoothe_status; no exception or longjmp crosses the ABI.
 *    On failure smoothe_last_error() describes the cause (thread-local string,
 *    valid until the next call on the same thread).
 *  - Input pointers are HOST pointers owned by the caller and copied before the
 *    call returns: the caller may free them immediately.
 *  - Handles (smoothe_egraph, smoothe_run) are owned by the library and freed
 *    with smoothe_free_egraph / smoothe_free_run.  A run keeps a reference to
 *    its e-graph: free runs first.
 *  - Output buffers are caller-allocated host memory of the sizes stated.
 *  - Per-seed arrays use the layout [row][B] (seed innermost), B = num_seeds.
 *  - Any CUDA failure returns SMOOTHE_E_CUDA and poisons the run: every later
 *    call on it returns SMOOTHE_E_STATE.
 *  - There is no CPU fallback: without a usable sm_100 device, load with
 *    device_ordinal >= 0 and every compute call fail with SMOOTHE_E_CUDA.
 */
#ifndef SMOOTHE_H
#define SMOOTHE_H

#include <stdint.h>

#if defined(__GNUC__)
#define SMOOTHE_API __attribute__((visibility("default")))
#else
#define SMOOTHE_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  SMOOTHE_OK = 0,
  SMOOTHE_E_INVALID_ARG = 1, /* NULL pointer, size out of range, bad option value       */
  SMOOTHE_E_BAD_GRAPH = 2,   /* empty class, child/root id out of range, ptr not monotone */
  SMOOTHE_E_OOM = 3,         /* host or device allocation failed                          */
  SMOOTHE_E_CUDA = 4,        /* CUDA runtime error (no device, launch failure, ...)       */
  SMOOTHE_E_NO_VALID = 5,    /* no valid (acyclic, complete) extraction sampled yet       */
  SMOOTHE_E_STATE = 6        /* call not allowed in this state (poisoned run, host-only graph) */
} smoothe_status;

typedef struct smoothe_egraph smoothe_egraph; /* opaque: host analysis + device copy      */
typedef struct smoothe_run smoothe_run;       /* opaque: per-run device state (theta, ...) */

/* ---------------------------------------------------------------------------
 * smoothe_load_egraph -- the e-graph of the extraction problem (P91-101).
 *
 * E-classes m_0..m_{M-1}; e-nodes n_0..n_{N-1}.  Class j owns the contiguous
 * e-nodes class_ptr[j] .. class_ptr[j+1]-1 (this defines ec(i), P98).
 * child_ptr/child_class give ch_i, the child e-classes of e-node i (P96), as
 * CSR; duplicates are removed (ch_i is a set, reading S5).  pa_j (P97) is
 * derived.  root_class is the root e-class (index 0 in the paper, P94).
 *
 *   class_ptr   [M+1]  int32, class_ptr[0] = 0, class_ptr[M] = N, strictly increasing
 *   child_ptr   [N+1]  int64, child_ptr[0] = 0, non-decreasing
 *   child_class [child_ptr[N]] int32 in [0, M)
 *
 * Builds (host): CSR children, CSC parents sorted by e-node id, strongly
 * connected components of the e-class graph (P318), and K_auto (reading S1).
 * device_ordinal >= 0 uploads everything to that GPU; device_ordinal = -1 keeps
 * a host-only handle usable with smoothe_egraph_get_info / _get_scc only.
 * Errors: SMOOTHE_E_BAD_GRAPH (empty class S28, out-of-range id, non-monotone
 * pointers), SMOOTHE_E_INVALID_ARG (NULL, M or N <= 0, N >= 2^29, more than
 * 2^31-1 edges), SMOOTHE_E_CUDA, SMOOTHE_E_OOM.
 * ------------------------------------------------------------------------- */
SMOOTHE_API smoothe_status smoothe_load_egraph(int32_t num_classes, int32_t num_nodes,
                                   const int32_t *class_ptr, const int64_t *child_ptr,
                                   const int32_t *child_class, int32_t root_class,
                                   int device_ordinal, smoothe_egraph **out);

typedef struct {
  int32_t num_classes, num_nodes; /* M, N                                                */
  int64_t num_edges;              /* E = sum_i |ch_i| after de-duplication               */
  int32_t root;
  int32_t K_auto;                 /* longest root path after DFS back-edge removal (S1)  */
  int32_t num_scc;                /* non-trivial SCCs (size > 1 or a self-loop)          */
  int32_t scc_classes;            /* classes inside them                                 */
  int32_t scc_max;                /* largest non-trivial SCC                             */
  int32_t max_class_size;
  int32_t max_in_degree;          /* max |pa_j|                                          */
  int32_t device;                 /* device ordinal, -1 for a host-only handle           */
  int64_t device_bytes;           /* device memory held by the graph                     */
} smoothe_egraph_info;

SMOOTHE_API smoothe_status smoothe_egraph_get_info(const smoothe_egraph *g, smoothe_egraph_info *out);

/* scc_of_class [M]: index of the non-trivial SCC containing class j, numbered
 * in order of first appearance by class id; -1 for classes on no cycle. */
SMOOTHE_API smoothe_status smoothe_egraph_get_scc(const smoothe_egraph *g, int32_t *scc_of_class);

/* ---------------------------------------------------------------------------
 * Cost model f (P101, P156, P409, P425; readings S22-S25).
 *   LINEAR:    f(p) = u^T p
 *   QUADRATIC: f(p) = u^T p + sum_e w_e p_{i_e} p_{j_e}     (reading S24; i_e != j_e)
 *   MLP:       f(p) = u^T p + W3 relu(W2 relu(W1 p + b1) + b2) + b3   (P409, P425)
 * u is always present.  MLP weights are row-major [out][in] float32 with
 * W1 [H1][N], W2 [H2][H1], W3 [1][H2].  All arrays are copied.
 * ------------------------------------------------------------------------- */
typedef enum { SMOOTHE_COST_LINEAR = 0, SMOOTHE_COST_QUADRATIC = 1, SMOOTHE_COST_MLP = 2 } smoothe_cost_kind;

typedef struct {
  smoothe_cost_kind kind;
  const double *u;                 /* [N]; integer-valued u makes decoded costs exact (S19) */
  int64_t quad_nnz;
  const int32_t *quad_i, *quad_j;  /* [quad_nnz] */
  const double *quad_w;            /* [quad_nnz] */
  int32_t mlp_hidden1, mlp_hidden2;/* H1 <= 64, H2 <= 16 (paper: 64, 8) */
  const float *W1, *b1, *W2, *b2, *W3, *b3;
} smoothe_cost_model;

typedef enum {
  SMOOTHE_AGG_INDEPENDENT = 0, /* Eq. 6b, P207-210 */
  SMOOTHE_AGG_CORRELATED = 1,  /* Eq. 7,  P219-221 */
  SMOOTHE_AGG_HYBRID = 2       /* mean of the two, P223 (default, P277) */
} smoothe_assumption;

typedef struct {
  smoothe_assumption assumption;
  int32_t prop_iters;      /* K propagation sweeps (P215); < 0 => K_auto (reading S1)       */
  double lambda;           /* NOTEARS weight (Eq. 10a, P264)                               */
  int32_t penalty_group;   /* G seeds share one Eq.-11 matrix; must divide num_seeds (S13) */
  double lr, beta1, beta2, eps;
  int32_t optimizer;       /* 0 = Adam (default), 1 = SGD (reading S10)                    */
  int32_t patience;        /* stop after this many steps without a better best; 0 = off (P279) */
  double time_limit_s;     /* stop after this wall time; 0 = off (P279)                    */
  uint64_t rng_key;        /* Philox key of the theta initialisation (S9)                  */
  int64_t seed_begin;      /* global index of this rank's first seed (multi-GPU sharding)  */
  void *cuda_stream;       /* cudaStream_t to launch on, or NULL for a private stream      */
  int32_t use_graphs;      /* 1 = replay each step as a captured CUDA graph                */
  int32_t converge;        /* 1 = "repeat until convergence" (P215, reading S1b): each     */
                           /* seed's sweeps stop at the first one that changes none of its */
                           /* q rows (fp32, bitwise), at most K; the reverse mode runs the */
                           /* sweeps performed.  0 = exactly K sweeps (default)            */
} smoothe_options;

/* Defaults: HYBRID, K_auto, lambda 1, G = 1, Adam(lr 0.1, 0.9, 0.999, 1e-8),
 * no patience / time limit, rng_key 0, seed_begin 0, NULL stream, graphs on. */
SMOOTHE_API smoothe_status smoothe_options_default(smoothe_options *opt);

/* ---------------------------------------------------------------------------
 * Runs.  A run holds B = num_seeds independent logits theta (P291-297), their
 * Adam state, the propagation stacks and the best extraction so far.
 *
 * smoothe_run_create   allocates and initialises theta from Philox (S9).
 * smoothe_run_steps    enqueues `steps` optimisation steps on the run's
 *                      stream.  Each step: softmax (Eq. 3b) -> K sweeps of
 *                      Eqs. 5-7 -> f(p) + lambda*h(A_t) (Eq. 10) -> reverse
 *                      mode -> Adam -> decode of the step's theta (P279) ->
 *                      keep the best (cost, step, global seed) (S20).
 *                      Returns without waiting unless patience or a time
 *                      limit needs a host check.
 * smoothe_optimize     = create + steps + synchronize (north-star entry point).
 * ------------------------------------------------------------------------- */
SMOOTHE_API smoothe_status smoothe_run_create(smoothe_egraph *g, const smoothe_cost_model *cost,
                                  int32_t num_seeds, const smoothe_options *opt,
                                  smoothe_run **out);
SMOOTHE_API smoothe_status smoothe_run_steps(smoothe_run *run, int32_t steps);
SMOOTHE_API smoothe_status smoothe_run_synchronize(smoothe_run *run);
SMOOTHE_API smoothe_status smoothe_optimize(smoothe_egraph *g, const smoothe_cost_model *cost,
                                int32_t num_seeds, int32_t steps, const smoothe_options *opt,
                                smoothe_run **out);

typedef struct {
  double best_cost;        /* f_b(s) of the best valid extraction; +inf if none            */
  int64_t best_seed;       /* global seed index                                            */
  int32_t best_step;       /* step that first produced it                                  */
  int32_t valid;           /* 1 if any valid extraction was sampled                        */
  int32_t steps_run;
  int32_t K;               /* sweeps per step actually used                                */
  double time_to_best_s;   /* run creation -> end of best_step, CUDA events                */
  double step_time_s;      /* mean device time per step                                    */
  double last_loss;        /* L of the last step = sum_b f_b + lambda * sum_g G h_g (S12) */
  int64_t pool_rows;       /* version-pool rows per seed chunk: capacity     */
  int64_t pool_peak_rows;  /* most rows a chunk's forward took in one step so far          */
  int32_t pool_grows;      /* times the pools grew (the overflowing steps were repeated)    */
  int32_t graph_mode;      /* how the steps ran: 1 = replayed from the captured CUDA graph, */
                           /* 0 = direct launches (use_graphs = 0, profiling or debug),     */
                           /* -1 = capture failed, fell back to direct launches (warned on  */
                           /* stderr; results identical, timing not the graph path's)       */
} smoothe_summary;

/* Copies the best extraction: choice[M] = chosen e-node of each selected class,
 * -1 for classes not in the extracted term.  choice may be NULL (summary only).
 * Returns SMOOTHE_E_NO_VALID (choice all -1, summary->valid = 0) if none. */
SMOOTHE_API smoothe_status smoothe_extract(smoothe_run *run, int32_t *choice, smoothe_summary *out);

/* ---------------------------------------------------------------------------
 * Parity hook.  Overwrites the run's theta (and m, v; NULL = zeros) with the
 * given host arrays [N][B], runs ONE step with Adam step number step_index + 1,
 * and copies the step's intermediates into caller-owned host buffers (any
 * pointer may be NULL).  Used by tests to compare with the fp64 oracle.
 * ------------------------------------------------------------------------- */
typedef struct {
  float *cp;           /* [N][B]  softmax of theta_in                          */
  float *qK;           /* [M][B]  q^K                                          */
  float *p;            /* [N][B]  p = cp * q^K[ec]                             */
  float *grad_cp;      /* [N][B]  dL/dcp including the penalty term            */
  float *grad_theta;   /* [N][B]  dL/dtheta                                    */
  float *theta_out;    /* [N][B]  updated theta                                */
  float *m_out, *v_out;/* [N][B]                                               */
  double *f;           /* [B]     f(p_b)                                       */
  double *h;           /* [B/G]   NOTEARS h per penalty group                  */
  double *loss;        /* [1]                                                  */
  int32_t *choice;     /* [M][B]  argmax_{k in m_j} theta_in_k (lowest id)     */
  uint8_t *reached;    /* [M][B]  class selected by the decode                 */
  uint8_t *valid;      /* [B]                                                  */
  double *disc_cost;   /* [B]     f_b(s), +inf when invalid                    */
  float *qstack;       /* [(K+1)][M][B] or NULL                                */
  int32_t *route;      /* [K][M][B] e-node the max of sweep t routed to: the  */
                       /* champion of the ascending-id scan with takeover at */
                       /* p > p_champion (1 + 2^-10), fp32 (reading S7');    */
                       /* -1 for classes without parents; NULL = skip         */
  int32_t *sweeps;     /* [B]     sweeps the seed's step performed (K, or its */
                       /* convergence sweep with converge = 1); NULL = skip  */
} smoothe_debug_out;

SMOOTHE_API smoothe_status smoothe_debug_step(smoothe_run *run, const float *theta_in, const float *m_in,
                                  const float *v_in, int32_t step_index, smoothe_debug_out *dump);

/* ---------------------------------------------------------------------------
 * Greedy worklist extraction, the paper's "heuristic method" (PAPER.md:133,
 * Sec. 2), on the e-graph's device: e-class costs start
 * at infinity; an e-node's aggregated cost is u_i plus the costs of its child
 * e-classes; an e-class takes the best aggregated cost of its e-nodes; the
 * extraction is read top-down from the root.  Ties (reading G1):
 * (cost, height, e-node id) lexicographically, height = 1 + max child height
 * (0 for a leaf), so the selection is acyclic and independent of the order of
 * evaluation.  Linear cost only (the heuristic's own model).
 *   u           [N] e-node costs (copied)
 *   choice      [M] caller-owned or NULL: selected e-node of every class in the
 *               extraction, -1 elsewhere
 *   class_cost  [M] caller-owned or NULL: the heuristic's class cost (its tree
 *               estimate, shared subterms counted once per use); +inf for
 *               classes without a finite derivation or unreachable from the root
 * Errors: E_INVALID_ARG (NULL g / u / out, or a negative or non-finite u: the
 * worklist's fixpoint needs u >= 0), E_STATE (host-only e-graph), E_CUDA.
 * ------------------------------------------------------------------------- */
typedef struct {
  double dag_cost;          /* f_b(s) of the extraction: sum of u over the selected
                               e-node of each reached class, once (P100, S19); +inf if none */
  double root_cost;         /* the heuristic's estimate for the root (tree cost)          */
  int32_t valid;            /* 1 iff the root has a finite derivation                     */
  int32_t selected_classes; /* classes in the extraction                                  */
} smoothe_greedy_result;

SMOOTHE_API smoothe_status smoothe_greedy(smoothe_egraph *g, const double *u, int32_t *choice,
                              double *class_cost, smoothe_greedy_result *out);

/* Warm start: theta_k += bias for k = choice[j] (every class j with choice[j] >= 0,
 * every seed of the run), e.g. from smoothe_greedy.  Call after smoothe_run_create,
 * before the first step.  choice [M] host, copied; E_INVALID_ARG if choice[j] is
 * not an e-node of class j. */
SMOOTHE_API smoothe_status smoothe_run_warm_start(smoothe_run *run, const int32_t *choice, float bias);

/* theta [N][B] of the run as it stands (host copy). */
SMOOTHE_API smoothe_status smoothe_get_theta(smoothe_run *run, float *theta);

/* Per-step record of the run (PAPER.md:459-461 compare the
 * relaxed loss with the sampled solutions along the optimisation): out[n][4]
 * host, caller-owned, for steps 0 .. n-1 (n = min(steps run, 4096, max_steps)):
 *   [0] min over the run's seeds of the relaxed cost f(p_b) at that step,
 *   [1] its mean over the seeds,
 *   [2] min over the seeds of the sampled (decoded) cost f_b(s) of that step
 *       (+inf if no sample was valid),
 *   [3] number of valid samples.
 * Relaxed values are the step's loss terms (before the update); sampled ones
 * decode the same theta (reading S17). */
SMOOTHE_API smoothe_status smoothe_run_get_trace(smoothe_run *run, double *out, int32_t max_steps,
                                                 int32_t *n_out);

/* The optimiser state as it stands, host copies [N][B] (any pointer may be
 * NULL), and the number of steps run: a debug step from this state with
 * step_index = *steps_run continues the run exactly (tests: parity after
 * steps replayed from the CUDA graph). */
SMOOTHE_API smoothe_status smoothe_get_state(smoothe_run *run, float *theta, float *m, float *v,
                                             int32_t *steps_run);

/* ---------------------------------------------------------------------------
 * Measurement.  With profiling on, every phase of every step is bracketed by
 * CUDA events on the run's stream; smoothe_run_get_profile synchronises and
 * returns the accumulated device time per phase and the number of kernel
 * launches since profiling was (re)enabled.
 * ------------------------------------------------------------------------- */
enum {
  SMOOTHE_PHASE_SOFTMAX = 0,  /* softmax + argmax + decode selection masks    */
  SMOOTHE_PHASE_FORWARD = 1,  /* K forward sweeps                             */
  SMOOTHE_PHASE_COST = 2,     /* f(p), dL/dp, backward initialisation         */
  SMOOTHE_PHASE_PENALTY = 3,  /* NOTEARS                                      */
  SMOOTHE_PHASE_REVERSE = 4,  /* K reverse sweeps                             */
  SMOOTHE_PHASE_UPDATE = 5,   /* softmax backward + Adam                      */
  SMOOTHE_PHASE_DECODE = 6,   /* reach, settle, discrete cost                 */
  SMOOTHE_PHASE_BEST = 7,     /* keep-best                                    */
  SMOOTHE_NUM_PHASES = 8
};

typedef struct {
  double phase_ms[SMOOTHE_NUM_PHASES];
  int64_t phase_launches[SMOOTHE_NUM_PHASES];
  int64_t steps;
  int64_t launches;          /* kernels launched by the library in the window   */
  int32_t num_seeds_padded;  /* seeds rounded up to the kernels' row width      */
  /* the sweep kernels alone (CUDA events around each launch on the run's
     stream): [0] k_sweep_forward, [1] k_sweep_reverse, [2] k_wspmv (frozen
     reverse sweeps)                                    */
  double sweep_kernel_ms[3];
  int64_t sweep_kernel_launches[3];
  int64_t frozen_sweeps;     /* k_wspmv launches with at least one frozen seed
                                and a live input (g_q^t not all zero)           */
  /* units (row or class edge x seed chunk of min(Bp, 128) seeds) those
     launches move, summed over them (dead-gradient skipping):
     class edges whose W row is loaded (child's g_q^t live), rows whose
     g_q^t / S are read and S written, rows whose g_q^{t-1} is written      */
  int64_t frozen_live_edges;
  int64_t frozen_live_rows;
  int64_t frozen_rows_written;
} smoothe_profile;

SMOOTHE_API smoothe_status smoothe_run_profile(smoothe_run *run, int32_t enable);
SMOOTHE_API smoothe_status smoothe_run_get_profile(smoothe_run *run, smoothe_profile *out);

SMOOTHE_API const char *smoothe_last_error(void);
SMOOTHE_API const char *smoothe_version(void);
SMOOTHE_API void smoothe_free_run(smoothe_run *run);
/* smoothe_free_run keeps the freed run's device blocks (per device, the last
 * freed run's only) for the next run of the same shape; this returns them to
 * the driver.  device_ordinal -1: every device.  (Allocation failures release
 * the cache of the device by themselves.) */
SMOOTHE_API void smoothe_release_cached_memory(int device_ordinal);
SMOOTHE_API void smoothe_free_egraph(smoothe_egraph *g);

#ifdef __cplusplus
}
#endif
#endif /* SMOOTHE_H */
