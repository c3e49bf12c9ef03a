/*
 * mp.h -- C-ABI of libmp, the B200 (sm_100a) implementation of MultiPrio's
 * data-parallel scoring and queue-build path (Tayeb, Bramas, Faverge,
 * Guermouche, "Dynamic Tasks Scheduling with Multiple Priorities on
 * Heterogeneous Computing Systems", IPDPS'24, hal-04498634).
 *
 * Citations "P:l.N" refer to /root/reference/PAPER.md line N; readings cN
 * refer to DESIGN.md §2 (= SURVEY.md §8(c)).
 *
 * Conventions (all entry points):
 *  - d_* are DEVICE pointers on the current CUDA device, h_* HOST pointers.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *    stream).  Every call is asynchronous on `stream` unless stated; inputs
 *    are never modified; every output buffer is caller-owned except the
 *    handle's internal arrays (exposed read-only by mp_dag_get_info).
 *  - Argument errors are detected on the host and returned before any
 *    launch.  Errors the device detects (MP_ERR_DOMAIN for durations) are
 *    raised into a per-handle device flag and reported by mp_check(), which
 *    synchronises `stream`; only mp_build_dag synchronises by itself.
 *  - No C++ exception crosses the ABI.  mp_last_error() returns a thread-local
 *    detail string for the last failing call.
 *  - One handle is used by one stream at a time: its per-handle scratch is
 *    reused by every call.  A caller may switch streams between calls; when
 *    the scratch grows the library synchronises the device first, so no
 *    kernel of an earlier call on another stream still uses the old buffer.
 *  - CSR offsets (d_row_ptr) are int32: the limit E < 2^31 below makes them
 *    fit (SURVEY §8(b) proposed int64; DESIGN.md §1 lists the deviation).
 *  - Layouts: per-task-per-arch arrays are row-major [n][A] (task-major).
 *  - Limits: 1 <= A <= 8, 0 <= n < 2^30, unique edges E < 2^31.
 *  - Durations delta(t,a) are binary32 milliseconds in {+inf} U {0} U
 *    [2^-41, 2^20); +inf = "t has no implementation on a" (can_exec false,
 *    P:l.91, l.135); -0 is read as +0; anything else (NaN, negative, nonzero
 *    below 2^-41, finite >= 2^20) or a task with no enabled arch is
 *    MP_ERR_DOMAIN (reading c20).  An arch a is enabled iff h_workers[a] > 0
 *    (get_worker_count(a) > 0, Alg. 1 P:l.135).
 *  - All float results are bit-exact with the CPU oracle: every binary32 op
 *    is an explicit round-to-nearest-even op, no FMA contraction, sums are
 *    exact integers.
 */
#ifndef MP_H
#define MP_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct mp_dag mp_dag; /* opaque; owns the CSR, levels and workspaces */

typedef enum {
    MP_OK = 0,
    MP_ERR_ARG = 1,    /* bad argument / id out of range / self-loop        */
    MP_ERR_CYCLE = 2,  /* the edge set is not a DAG                         */
    MP_ERR_DOMAIN = 3, /* duration outside the domain above                 */
    MP_ERR_CUDA = 4,   /* a CUDA runtime error (detail in mp_last_error)     */
    MP_ERR_NOMEM = 5   /* device allocation failed                          */
} mp_status;

typedef enum {
    MP_CRIT_BOTTOM_LEVEL = 0, /* bl(t) / CP, arch-independent (north_star)    */
    MP_CRIT_NOD = 1           /* NOD_a(t) / max_t NOD_a, eq. 2 P:l.193         */
} mp_crit;

/* Read-only views of the handle's device arrays (valid until mp_free). */
typedef struct {
    int32_t n_tasks;
    int64_t n_edges;         /* unique edges                                  */
    int32_t n_levels;        /* L = 1 + max level (0 when n = 0)              */
    int32_t max_width;       /* max tasks in one level                        */
    const int32_t* d_row_ptr;     /* [n+1] successor CSR offsets              */
    const int32_t* d_col;         /* [E]   successor ids, ascending per row   */
    const int32_t* d_indeg;       /* [n]   |lambda^-(t)|                       */
    const int32_t* d_level;       /* [n]   0 if no predecessor else 1+max     */
    const int32_t* d_level_ptr;   /* [L+1] offsets of each level in order     */
    const int32_t* d_level_order; /* [n]   ids sorted by (level, id)          */
} mp_dag_info;

/* One priority queue's counters (Alg. 1, P:l.135). */
typedef struct {
    int32_t count;   /* ready_tasks_count: entries in the queue              */
    int32_t head;    /* task id at the root of the heap (queue[0]) or -1     */
    uint64_t brw_lo; /* best_remaining_work = sum of delta(t,a) over entries */
    int64_t brw_hi;  /*   with delta(t,a) == min_a' delta(t,a'), as the exact */
                     /*   128-bit integer hi:lo in units of 2^-64 ms          */
    double brw;      /* that exact value rounded once to binary64            */
} mp_queue_summary;  /* 32 bytes */

/*
 * a1 + a2: DAG ingest and topological levels.
 * Builds G = (V, E) from n_edges (src -> dst) pairs: "for each edge
 * (t_i, t_j), t_j cannot start before the completion of t_i" (P:l.89);
 * lambda^+/- are sets (Table I, P:l.83-84) so duplicate pairs collapse
 * (reading c19).  Levels: level(t) = 0 if lambda^-(t) is empty else
 * 1 + max level(p), p in lambda^-(t); level_order lists ids by (level, id).
 * d_src/d_dst: device int32[n_edges]; may be NULL when n_edges = 0.
 * Errors: MP_ERR_ARG for n < 0, id outside [0, n) or a self-loop;
 * MP_ERR_CYCLE when the pairs contain a cycle.  Synchronises `stream` once.
 * On success *out owns its device buffers (release with mp_free).
 */
mp_status mp_build_dag(int32_t n_tasks, int64_t n_edges, const int32_t* d_src,
                       const int32_t* d_dst, void* stream, mp_dag** out);

/*
 * Same as mp_build_dag, into an existing handle: the previous DAG is replaced
 * and the handle's device buffers are reused (grow-only), so re-ingesting a
 * DAG no larger than an earlier one performs no device allocation.  On error
 * the handle holds an empty DAG (n = 0) and stays valid for mp_free.
 */
mp_status mp_dag_rebuild(mp_dag* dag, int32_t n_tasks, int64_t n_edges, const int32_t* d_src,
                         const int32_t* d_dst, void* stream);

mp_status mp_dag_get_info(const mp_dag* dag, mp_dag_info* out);

/*
 * a3 + a4 (+ a5): bottom-level criticality (north_star) and, optionally, the
 * paper's NOD criticality (eq. 2, P:l.191-193).
 *   w(t)  = min over enabled a of delta(t,a)            (reading c2, P:l.265)
 *   bl(t) = w(t) + max_{s in lambda^+(t)} bl(s), or w(t) without successors
 *   *d_cp = CP = max_t bl(t)
 *   NOD_a(t) = sum_{s in lambda^+(t), s enabled on a} 1/|{p in lambda^-(s) :
 *             p enabled on a}| for (t,a) enabled, else 0 (reading c10); each
 *             term is floor(2^32/k), the sum an exact 64-bit integer, converted
 *             once to binary32 and scaled by 2^-32 (reading c11).
 * d_dur: float[n][A]; h_workers: int32[A]; d_bl: float[n]; d_cp: float[1];
 * d_nod: float[n][A] or NULL.  Domain errors -> device flag (mp_check).
 */
mp_status mp_bottom_level(mp_dag* dag, int32_t n_arch, const float* d_dur,
                          const int32_t* h_workers, float* d_bl, float* d_cp,
                          float* d_nod, void* stream);

/*
 * a6: gain heuristic, eq. 1 (P:l.172), hd(a) (P:l.176), Table II (P:l.180-187).
 *   ref(t,a) = min over enabled a' != a of delta(t,a')   (reading c6)
 *   d(t,a)   = ref - delta(t,a)
 *   hd(a)    = max |d(t,a)| over tasks with >= 2 enabled archs incl. a (c4, c5)
 *   gain     = 1 if t has one enabled arch (P:l.170, c7); 0.5 if hd(a) = 0 (c8);
 *              else (d + hd) / (hd + hd); 0 where (t,a) is not enabled.
 * d_gain: float[n][A]; d_hd: float[A];
 * d_flags: uint8[n][A], bit0 = enabled(t,a), bit1 = delta(t,a) == w(t)
 *   ("normalized_speedup(t,a) == 1", Alg. 1, reading c15).
 */
mp_status mp_affinity(mp_dag* dag, int32_t n_arch, const float* d_dur,
                      const int32_t* h_workers, float* d_gain, float* d_hd,
                      uint8_t* d_flags, void* stream);

/*
 * a7: normalised criticality and the combined key.  "All values are
 * normalized between 0 and 1" (P:l.166): crit_n = crit / max crit (reading
 * c9; 0 when the max is 0).  Tasks are ordered by gain first, criticality on
 * equal gain (P:l.138, l.322):
 *   key(t,a) = ((0x3F800000 - bits(gain)) << 32) | (0x3F800000 - bits(crit_n))
 * so ascending key = (gain desc, crit_n desc); UINT64_MAX where not enabled.
 * kind = MP_CRIT_BOTTOM_LEVEL: d_crit = bl float[n], d_crit_norm float[n];
 * kind = MP_CRIT_NOD: d_crit = nod float[n][A], normalised per arch over
 *   enabled tasks, d_crit_norm float[n][A].   d_key: uint64[n][A].
 */
mp_status mp_score(mp_dag* dag, int32_t n_arch, mp_crit kind, const float* d_crit,
                   const float* d_gain, const uint8_t* d_flags, float* d_crit_norm,
                   uint64_t* d_key, void* stream);

/*
 * a8 + a9: one priority queue per architecture type (the heaps h_m of
 * P:l.97-106, l.130; memory nodes of one arch share a queue, reading c13).
 * Queue a holds {t : enabled(t,a) and (d_done == NULL or ready(t))},
 * ready(t) = !done(t) and all predecessors done (P:l.91, reading c18),
 * sorted by (key ascending, id ascending) (reading c12); a sorted array is a
 * valid binary max-heap.  d_qptr: int64[A+1] offsets into d_qtask (capacity
 * n*A int32); d_sum: mp_queue_summary[A] (count, head, best_remaining_work
 * over entries with flags bit1).  d_dur supplies delta for the brw sums.
 */
mp_status mp_build_queues(mp_dag* dag, int32_t n_arch, const uint64_t* d_key,
                          const uint8_t* d_flags, const float* d_dur,
                          const uint8_t* d_done, int64_t* d_qptr, int32_t* d_qtask,
                          mp_queue_summary* d_sum, void* stream);

/*
 * a10: batched replicas.  For r in [r0, r0+R):
 *   delta_r(t,a) = delta(t,a) * (1 + sigma * (2u - 1)), u = (splitmix64(seed
 *   + c * 0x9E3779B97F4A7C15) >> 40) * 2^-24 with counter
 *   c = (r*n + t)*A + a + 1, each float op RN binary32 (north_star
 *   "duration-perturbed instances of one DAG"); then a3-a9 with
 *   MP_CRIT_BOTTOM_LEVEL in ALL mode.  Replica results depend only on the
 *   global replica id r (world-size invariant).
 * d_base_dur: float[n][A]; d_cp: float[R]; d_sum: mp_queue_summary[R][A];
 * d_qtask: int32[R][n*A] (queue a of replica r at offset r*n*A + qoff_a, where
 *   qoff_a = sum of that replica's counts of archs < a) or NULL.
 */
mp_status mp_replicas_run(mp_dag* dag, int32_t n_arch, const float* d_base_dur,
                          const int32_t* h_workers, uint64_t seed, float sigma,
                          int64_t r0, int32_t R, float* d_cp, mp_queue_summary* d_sum,
                          int32_t* d_qtask, void* stream);

/*
 * incremental READY-mode PUSH (the paper's dynamic setting,
 * P:l.91 "a ready task is a task for which all dependencies are released",
 * Alg. 1 PUSH at batch granularity).
 * mp_ready_init: d_rem[t] = |lambda^-(t)| (predecessors not completed yet).
 * mp_queues_push: given the current queues (d_qptr_in/d_qtask_in, e.g. from
 * mp_build_queues with d_done = all-zero, i.e. the sources) and a batch of
 * m completed tasks (d_batch, int32[m]; each was ready and is completed once),
 *   - removes the batch's tasks from every queue (they were popped, Alg. 2),
 *   - decrements d_rem of their successors; successors reaching 0 are newly
 *     ready and join every queue whose arch can run them (P:l.104),
 *   - writes the merged queues to d_qptr_out/d_qtask_out (capacity n*A; must
 *     not alias the input), still sorted by (key asc, id asc), and summaries.
 * Invariant (tested): after pushing batches B1..Bk the queues equal
 * mp_build_queues in READY mode with done = B1 U .. U Bk.  d_key/d_flags/d_dur
 * are the whole-DAG scores of mp_score/mp_affinity (reading c18).
 * The batch is validated before any state changes: an id outside [0,n), a
 * task that is not ready (a predecessor not completed), a task completed in
 * an earlier batch or listed twice in this one raises MP_ERR_ARG (mp_check)
 * and leaves d_rem and the output queues' inputs untouched (the outputs then
 * hold the unchanged queues).  A completed task's d_rem entry becomes -1.
 */
mp_status mp_ready_init(mp_dag* dag, int32_t* d_rem, void* stream);
mp_status mp_queues_push(mp_dag* dag, int32_t n_arch, const uint64_t* d_key, const uint8_t* d_flags,
                         const float* d_dur, const int32_t* d_batch, int32_t m, int32_t* d_rem,
                         const int64_t* d_qptr_in, const int32_t* d_qtask_in, int64_t* d_qptr_out,
                         int32_t* d_qtask_out, mp_queue_summary* d_sum, void* stream);

/*
 * N1, static-order variant.  Because the scores are whole-DAG (reading c18),
 * every READY-mode queue is the ALL-mode queue restricted to the ready tasks,
 * in the same order.  The caller keeps the ALL-mode queues (d_qptr_all,
 * d_qtask_all from mp_build_queues with d_done = NULL), d_rem (mp_ready_init)
 * and a done mask d_done (uint8[n], zeroed by the caller before the first
 * push); a push marks the batch done, releases successors and compacts the
 * ALL-mode queues into d_qptr_out / d_qtask_out (capacity n*A) with the
 * summaries -- the same queues mp_queues_push produces, with no sort or merge.
 * Pushing the empty batch (m = 0) yields the sources' queues.  A batch task
 * that is not ready, completed before, listed twice, or outside [0,n) raises
 * MP_ERR_ARG (mp_check); the batch is validated before any state changes, so
 * d_rem and d_done are then unchanged.  A completed task's d_rem becomes -1.
 */
mp_status mp_queues_push_all(mp_dag* dag, int32_t n_arch, const int64_t* d_qptr_all, const int32_t* d_qtask_all,
                             const uint8_t* d_flags, const float* d_dur, const int32_t* d_batch, int32_t m,
                             int32_t* d_rem, uint8_t* d_done, int64_t* d_qptr_out, int32_t* d_qtask_out,
                             mp_queue_summary* d_sum, void* stream);

/*
 * discrete-event simulation of MultiPrio on a platform of
 * h_workers[a] workers of each architecture type a: PUSH (Alg. 1,
 * P:l.133-136) of every task that becomes ready (P:l.91), POP (Alg. 2,
 * P:l.140-160) by every idle worker with the eviction mechanism
 * (pop_condition, §V-D, P:l.214-220; eviction = 0 disables it, Fig. 4 top)
 * and MAX_TRIES = max_tries, and lazy removal of processed duplicates
 * (P:l.130).  Readings s1-s9: times are binary64 ms, a task
 * runs delta_r(t,a) (the scored duration of its arch); workers are numbered
 * arch-major and pop in id order at each event time after the completions
 * at that time have released their successors; get_most_local_prio_task is
 * the heap root (no data model); pop_condition(t, a) = eviction off, or a is
 * a best arch of t, or best_remaining_work[b] > delta(t,a) for every best
 * arch b; a pop removes t from every heap's counters at once.
 * Instance r in [r0, r0+R) uses delta_r of mp_replicas_run (sigma = 0: the
 * base durations) and the ALL-mode queues that give the heap orders:
 * d_qtask [R][n*A] and d_sum [R][A] exactly as mp_replicas_run writes them,
 * or, for one DAG (R = 1, r0 = 0, sigma = 0), mp_build_queues' ALL-mode
 * d_qtask / d_sum (any criticality kind).
 * Outputs: d_stats [R]; d_start double[R][n] and d_worker int32[R][n] (the
 * schedule; either may be NULL).  Limits: 1 <= sum of workers <= 256.
 * A queue entry outside [0, n), a task missing from its arch's queue or a
 * schedule that cannot complete raise MP_ERR_ARG through mp_check.
 */
typedef struct {
    double makespan;   /* completion time of the last task (ms)              */
    int64_t pops;      /* successful POPs (= n)                              */
    int64_t evictions; /* heaps_evict_task calls                             */
    int64_t dups;      /* duplicates a pop leaves in the other heaps (P:l.130) */
    int64_t rounds;    /* POP calls that ended on MAX_TRIES                  */
    int64_t moved;     /* bytes of accessed data not resident at task starts */
    double busy[8];    /* sum of delta_r(t,a) over tasks run on arch a, exact */
                       /*   sum rounded once to binary64                     */
    int32_t ran[8];    /* tasks run on arch a                                */
} mp_sim_stats;        /* 144 bytes */

mp_status mp_simulate(mp_dag* dag, int32_t n_arch, const float* d_base_dur, const int32_t* h_workers,
                      uint64_t seed, float sigma, int64_t r0, int32_t R, const int32_t* d_qtask,
                      const mp_queue_summary* d_sum, int32_t max_tries, int32_t eviction,
                      mp_sim_stats* d_stats, double* d_start, int32_t* d_worker, void* stream);

/*
 * the same simulation with POP's data-locality pick,
 * get_most_local_prio_task (§V-C, P:l.205-212): among the first top_n heap
 * entries (priority order) whose gain is within eps of the root's
 * (gain(root) - gain(t) <= eps, one binary32 subtraction; reading l1), the
 * task with the largest LS_SDH^2(m, t) (eq. 3, P:l.209) on the popping
 * worker's memory node m, ties to the higher priority (l3):
 *   LS_SDH^2(m,t) = sum over t's accesses of data resident on m of
 *                   size (mode R) or size^2 (mode W or RW, l2), exact uint64.
 * Data model: d_acc_ptr int64[n+1], d_acc_handle int32[], d_acc_mode uint8[]
 * (1 = R, 2 = W, 3 = RW) per task, d_size uint64[n_handles] bytes (< 2^28).
 * Every handle starts resident on node 0 only; a task started on node m
 * makes its data resident on m, and a write leaves m the only copy (l4).
 * Memory nodes: h_worker_node[W] (NULL: arch-0 workers share node 0, every
 * other worker has its own node 1, 2, ...; l5).  A task runs
 * delta_r(t,a) (+) missing bytes x xfer_ms_per_byte (l6).
 * top_n <= 1 and d_acc_ptr = NULL give mp_simulate; top_n <= 32; eps >= 0.
 * The P:l.238 setting is top_n = 10, eps = 0.8.
 */
typedef struct {
    int32_t max_tries;           /* MAX_TRIES (>= 1)                          */
    int32_t eviction;            /* pop_condition on (1) / off (0)            */
    int32_t top_n;               /* n of §V-C (<= 1: the heap root)           */
    float eps;                   /* epsilon of §V-C                           */
    int32_t n_handles;           /* data handles                              */
    int32_t n_nodes;             /* memory nodes (0: from h_worker_node)      */
    const int64_t* d_acc_ptr;    /* [n+1], or NULL: no data model             */
    const int32_t* d_acc_handle; /* [acc]                                     */
    const uint8_t* d_acc_mode;   /* [acc]                                     */
    const uint64_t* d_size;      /* [n_handles]                               */
    const int32_t* h_worker_node;/* [W] host, or NULL                         */
    double xfer_ms_per_byte;     /* >= 0                                      */
} mp_sim_config;

mp_status mp_simulate_cfg(mp_dag* dag, int32_t n_arch, const float* d_base_dur, const int32_t* h_workers,
                          uint64_t seed, float sigma, int64_t r0, int32_t R, const int32_t* d_qtask,
                          const mp_queue_summary* d_sum, const mp_sim_config* cfg, mp_sim_stats* d_stats,
                          double* d_start, int32_t* d_worker, void* stream);

/*
 * variants (ablations of readings c2, c4, c10).
 *
 * mp_bottom_level_w: bottom-level (a4) with a choice of node weight:
 *   MP_WEIGHT_MIN  = min over enabled archs (reading c2, = mp_bottom_level);
 *   MP_WEIGHT_MEAN = HEFT's mean cost over the platform's processors
 *     (reading v1): w(t) = (sum over enabled a, in arch order, of
 *     h_workers[a] * delta(t,a)) / sum of h_workers[a], each op one RN
 *     binary64 op, rounded once to binary32.
 *
 * mp_affinity_prefix: eq. 1 gains with hd(a) read as "the highest execution
 *   time difference recorded SO FAR" (P:l.176, reading v2): tasks are pushed
 *   in the order d_order (int32[n], a permutation of [0,n); NULL = id order)
 *   and task t's gains use the running max of |d(u,a)| over the tasks u
 *   pushed up to and including t.  d_hd receives the final max (= mp_affinity's
 *   hd); d_flags as mp_affinity.  An id outside [0,n) raises MP_ERR_ARG via
 *   mp_check.
 *
 * mp_nod_remaining: NOD (eq. 2) on the remaining graph (reading v3): tasks
 *   with d_done[t] != 0 are removed from lambda^- and lambda^+; done tasks
 *   score 0.  d_done = all-zero gives mp_bottom_level's d_nod.
 */
typedef enum { MP_WEIGHT_MIN = 0, MP_WEIGHT_MEAN = 1 } mp_weight;

mp_status mp_bottom_level_w(mp_dag* dag, int32_t n_arch, const float* d_dur, const int32_t* h_workers,
                            mp_weight kind, float* d_bl, float* d_cp, void* stream);
mp_status mp_affinity_prefix(mp_dag* dag, int32_t n_arch, const float* d_dur, const int32_t* h_workers,
                             const int32_t* d_order, float* d_gain, float* d_hd, uint8_t* d_flags, void* stream);
mp_status mp_nod_remaining(mp_dag* dag, int32_t n_arch, const float* d_dur, const int32_t* h_workers,
                           const uint8_t* d_done, float* d_nod, void* stream);

/* Synchronise `stream`, then return (and clear) the handle's device error
 * flag: MP_OK or MP_ERR_DOMAIN; MP_ERR_CUDA on a pending CUDA error. */
mp_status mp_check(mp_dag* dag, void* stream);

/* NULL-safe.  Synchronises the device before releasing the buffers. */
void mp_free(mp_dag* dag);

const char* mp_status_str(mp_status s);
const char* mp_last_error(void);

/* Library introspection for tests: "sm_100a", version string. */
const char* mp_build_info(void);

/*
 * Per-level latency microbenchmarks (SURVEY §8(d) two-term roofline): a level-
 * synchronous pass over a depth-L DAG costs at least L x t_level.  Launches one
 * microkernel on `stream` that performs L level boundaries of the given kind and
 * nothing else (the caller times it):
 *   MP_MB_SYNC     one CTA of 1024 threads, L __syncthreads
 *   MP_MB_CLUSTER  one cluster of `arg` (2..8) CTAs, L cluster barriers
 *   MP_MB_GRID     one CTA per SM (cooperative launch), L grid barriers
 *   MP_MB_CHAIN    one thread, L dependent L2 loads p = d_next[p] (d_next: a
 *                  permutation cycle of uint32 indices, device, caller-owned)
 * d_sink: one uint32 of device scratch (keeps the work observable).
 */
enum { MP_MB_SYNC = 0, MP_MB_CLUSTER = 1, MP_MB_GRID = 2, MP_MB_CHAIN = 3 };
mp_status mp_microbench(int32_t kind, int32_t L, int32_t arg, const uint32_t* d_next, uint32_t* d_sink,
                        void* stream);

/* Diagnostics.  mp_launch_count: kernels libmp has launched in this process.
 * mp_prof_enable(1): bracket every launch with CUDA events on its stream;
 * mp_prof_query synchronises on those events and returns the summed device
 * time (ms) and launch count of kernel `name` (e.g. "k_sort_pass") since the
 * last mp_prof_reset.  Host-side bookkeeping only; results are unaffected. */
uint64_t mp_launch_count(void);
void mp_prof_enable(int on);
void mp_prof_reset(void);
mp_status mp_prof_query(const char* name, double* total_ms, int64_t* launches);
/* Comma-separated names of every kernel timed since the last mp_prof_reset;
 * returns the length needed (excluding the NUL); writes at most len bytes. */
int64_t mp_prof_names(char* buf, int64_t len);

#ifdef __cplusplus
}
#endif

#endif /* MP_H */
