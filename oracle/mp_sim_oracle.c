/*
 * mp_sim_oracle.c -- plain, slow, single-threaded CPU oracle for SURVEY.md
 * §8(f) row N2: a discrete-event simulation of MultiPrio's PUSH (Alg. 1,
 * P:l.133-136) and POP (Alg. 2, P:l.140-160) with the eviction mechanism
 * (pop_condition, §V-D, P:l.214-220) and lazy removal of duplicates
 * (P:l.130) over a whole task DAG, on a platform of h_workers[a] workers of
 * each architecture type a.
 *
 * TEST INFRASTRUCTURE ONLY (same rules as mp_oracle.c): only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
 * may load it.  It shares no code with the CUDA library.  Its data structure
 * is the paper's own: one binary max-heap per memory node (P:l.130), ordered
 * by the combined score (gain first, criticality on equal gain, P:l.138),
 * i.e. by the a7 key ascending, ties by task id (reading c12); the CUDA path
 * uses rank bitmaps instead.
 *
 * Row N3 is the data-locality pick of POP: get_most_local_
 * prio_task (§V-C, P:l.205-212) scores the first n heap entries whose score
 * is within epsilon of the root's with LS_SDH^2 (eq. 3, P:l.209) on the
 * worker's memory node, given per-task data accesses, handle sizes and a
 * residency state that task starts update (readings l1-l6).
 *
 * Readings (s1-s9, l1-l6) are cited inline as "sN" / "lN".
 *
 * Pins (tests/test_oracle_pins.py, "sim" tests): hand-worked schedules of
 * Table II's tasks (P:l.180-187) with and without eviction, the closed forms
 * makespan = CP with unbounded workers and = sum of durations with one
 * worker, the list-scheduling bounds max(CP, W^-1 sum w) <= makespan <=
 * W^-1 sum w + (1 - 1/W) CP (one arch), and trace invariants (precedence,
 * no overlap, exactly-once, greedy / highest-priority-first without
 * eviction), plus Fig. 4's direction (eviction lowers GPU idle time).
 * `stale` (lazy removals, P:l.130) is pinned by the hand-worked counts in
 * tests/golden/sim_worked.json; `dups` (duplicates a pop leaves) equals
 * (enabled archs - 1) per task without eviction, and stale == dups at
 * completion.  N3 (top_n, any n >= 1; the paper puts no cap on n, P:l.207):
 * hand-worked locality schedules and an independent replay
 * (test_locality_replay, top_n up to 64).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

enum { SO_OK = 0, SO_ERR_ARG = 1, SO_ERR_NOMEM = 5, SO_ERR_STUCK = 6 };

typedef unsigned __int128 u128;

typedef struct {             /* per simulated instance                         */
    double makespan;         /* completion time of the last task (ms)          */
    int64_t pops;            /* successful POPs (= n)                          */
    int64_t evictions;       /* heaps_evict_task calls (Alg. 2)                */
    int64_t dups;            /* duplicates a pop leaves in other heaps (P:l.130) */
    int64_t rounds;          /* POP calls that ended on MAX_TRIES              */
    int64_t moved;           /* bytes of accessed data not resident at start   */
    double busy[8];          /* sum of delta(t,a) over tasks run on arch a     */
    int32_t ran[8];          /* tasks run on arch a                            */
    int64_t stale;           /* processed duplicates met at a heap root and     */
                             /* dropped there ("lazily removed", P:l.130)      */
} so_stats;

/* delta as an exact integer count of 2^-64 ms (domain: 0 or [2^-41, 2^20)) */
static u128 fx(float d) {
    if (d == 0.0f) return 0;
    int e;
    float f = frexpf(d, &e);
    uint64_t mant = (uint64_t)ldexpf(f, 24);
    return (u128)mant << (e - 24 + 64);
}

/* ---------------- one binary max-heap per memory node (P:l.130) ---------- */
typedef struct {
    int32_t* v;              /* task ids                                       */
    int32_t size;
    const uint64_t* key;     /* key[t*A + a] of this heap's arch               */
    int32_t A, a;
} heap;

/* "higher" = higher priority = smaller (key, id) */
static int higher(const heap* h, int32_t x, int32_t y) {
    uint64_t kx = h->key[(int64_t)x * h->A + h->a], ky = h->key[(int64_t)y * h->A + h->a];
    if (kx != ky) return kx < ky;
    return x < y;
}

static void heap_insert(heap* h, int32_t t) {
    int32_t i = h->size++;
    h->v[i] = t;
    while (i > 0) {
        int32_t p = (i - 1) / 2;
        if (!higher(h, h->v[i], h->v[p])) break;
        int32_t tmp = h->v[i]; h->v[i] = h->v[p]; h->v[p] = tmp;
        i = p;
    }
}

static void heap_pop_root(heap* h) {
    h->v[0] = h->v[--h->size];
    int32_t i = 0;
    for (;;) {
        int32_t l = 2 * i + 1, r = l + 1, b = i;
        if (l < h->size && higher(h, h->v[l], h->v[b])) b = l;
        if (r < h->size && higher(h, h->v[r], h->v[b])) b = r;
        if (b == i) break;
        int32_t tmp = h->v[i]; h->v[i] = h->v[b]; h->v[b] = tmp;
        i = b;
    }
}

/* ---------------- scheduler state ---------------------------------------- */
typedef struct {
    int32_t n, A, W;
    const int32_t* row_ptr;
    const int32_t* col;
    const float* dur;        /* canonical delta(t,a), +inf = cannot execute    */
    const int32_t* workers;
    heap h[8];
    uint8_t* counted;        /* [n][A]: t counted in ready_tasks_count[a]      */
    uint8_t* started;        /* [n]                                            */
    int32_t* rem;            /* [n] predecessors not completed                 */
    int64_t count[8];        /* ready_tasks_count (Alg. 1)                     */
    u128 brw[8];             /* best_remaining_work (Alg. 1), exact            */
    int max_tries, eviction;
    /* N3 data locality (eq. 3) */
    const float* gain;       /* [n][A] eq. 1 gains (the heaps' first score)    */
    int top_n;               /* n of P:l.238 (<= 1: the root)                  */
    float eps;               /* epsilon of P:l.238                             */
    const int64_t* acc_ptr;  /* [n+1] data accesses of each task, or NULL      */
    const int32_t* acc_h;    /* handle                                         */
    const uint8_t* acc_mode; /* bit0 read, bit1 write (R = 1, W = 2, RW = 3)   */
    const uint64_t* size;    /* [H] bytes                                      */
    int32_t H, M;            /* handles, memory nodes                          */
    uint8_t* resident;       /* [M][H]                                         */
    int32_t* cand;           /* [max(top_n, 1)] candidates of one POP          */
} sched;

static int en(const sched* s, int32_t t, int32_t a) {
    return !isinf(s->dur[(int64_t)t * s->A + a]) && s->workers[a] > 0;
}

/* normalized_speedup(t,a) == 1 <=> delta(t,a) is the minimum over enabled
 * archs (reading c15) */
static int best(const sched* s, int32_t t, int32_t a) {
    if (!en(s, t, a)) return 0;
    float d = s->dur[(int64_t)t * s->A + a];
    for (int32_t b = 0; b < s->A; b++)
        if (en(s, t, b) && s->dur[(int64_t)t * s->A + b] < d) return 0;
    return 1;
}

/* Alg. 1 PUSH: t joins every heap whose arch can run it (P:l.104). */
static void push(sched* s, int32_t t) {
    for (int32_t a = 0; a < s->A; a++) {
        if (!en(s, t, a)) continue;
        heap_insert(&s->h[a], t);
        s->counted[(int64_t)t * s->A + a] = 1;
        s->count[a] += 1;
        if (best(s, t, a)) s->brw[a] += fx(s->dur[(int64_t)t * s->A + a]);
    }
}

/* §V-D: the best worker always takes the task; another worker takes it when
 * best_remaining_work of the best arch exceeds delta(t, w_a) (s4). */
static int pop_condition(const sched* s, int32_t t, int32_t a) {
    if (!s->eviction) return 1;
    if (best(s, t, a)) return 1;
    u128 mine = fx(s->dur[(int64_t)t * s->A + a]);
    for (int32_t b = 0; b < s->A; b++)
        if (best(s, t, b) && !(s->brw[b] > mine)) return 0;
    return 1;
}

/* remove t from the counters of every heap that still counts it (s5) */
static void uncount(sched* s, int32_t t) {
    for (int32_t b = 0; b < s->A; b++) {
        int64_t i = (int64_t)t * s->A + b;
        if (!s->counted[i]) continue;
        s->counted[i] = 0;
        s->count[b] -= 1;
        if (best(s, t, b)) s->brw[b] -= fx(s->dur[i]);
    }
}

/* eq. 3 (P:l.209): LS_SDH^2(m,t) = sum of the sizes of t's data resident on
 * m accessed in read mode + sum of the squared sizes of those accessed in
 * write mode (a RW access counts as write, l2). */
static uint64_t ls_sdh2(const sched* s, int32_t m, int32_t t) {
    uint64_t v = 0;
    if (!s->acc_ptr) return 0;
    for (int64_t i = s->acc_ptr[t]; i < s->acc_ptr[t + 1]; i++) {
        int32_t hd = s->acc_h[i];
        if (!s->resident[(int64_t)m * s->H + hd]) continue;
        uint64_t z = s->size[hd];
        v += (s->acc_mode[i] & 2) ? z * z : z;
    }
    return v;
}

/* get_most_local_prio_task (§V-C, P:l.205-212): among the first top_n live
 * entries of heap a in priority order whose gain is within eps of the
 * root's (l1), the one with the largest LS_SDH^2 on memory node m, ties to
 * the higher priority (l3).  On the binary heap: pop the candidates, put
 * back the ones not chosen.  Processed duplicates met on the way are dropped
 * (s5).  Returns the chosen task, already removed from the heap, or -1. */
static int32_t take_most_local(sched* s, int32_t a, int32_t m, so_stats* st) {
    heap* h = &s->h[a];
    int32_t* cand = s->cand;
    int k = 0, kmax = s->top_n > 1 ? s->top_n : 1;
    float g0 = 0.0f;
    while (k < kmax && h->size > 0) {
        int32_t t = h->v[0];
        heap_pop_root(h);
        if (s->started[t]) { st->stale += 1; continue; }    /* lazy removal (P:l.130) */
        float g = s->gain ? s->gain[(int64_t)t * s->A + a] : 0.0f;
        if (k == 0) g0 = g;
        else {
            float diff = g0 - g;                   /* one RN binary32 op */
            if (!(diff <= s->eps)) { heap_insert(h, t); break; }
        }
        cand[k++] = t;
    }
    if (k == 0) return -1;
    int b = 0;
    if (k > 1) {
        uint64_t bv = ls_sdh2(s, m, cand[0]);
        for (int i = 1; i < k; i++) {
            uint64_t v = ls_sdh2(s, m, cand[i]);
            if (v > bv) { bv = v; b = i; }
        }
    }
    for (int i = 0; i < k; i++)
        if (i != b) heap_insert(h, cand[i]);
    return cand[b];
}

/* Alg. 2 POP for a worker of arch a on memory node m (heaps per arch,
 * reading c13).  Returns the task, or -1; *hit_max = 1 when MAX_TRIES ended
 * it. */
static int32_t pop(sched* s, int32_t a, int32_t m, so_stats* st, int* hit_max) {
    int tries = 0;
    *hit_max = 0;
    while (tries < s->max_tries) {
        int32_t t = take_most_local(s, a, m, st);  /* already off heap a */
        if (t < 0) return -1;
        if (pop_condition(s, t, a)) {              /* heaps_pop_and_update      */
            for (int32_t b = 0; b < s->A; b++)     /* "any duplicate tasks in   */
                if (b != a && s->counted[(int64_t)t * s->A + b])   /* other     */
                    st->dups += 1;                 /* queues will remain there" */
            uncount(s, t);
            s->started[t] = 1;
            st->pops += 1;
            return t;
        }
        s->counted[(int64_t)t * s->A + a] = 0;    /* heaps_evict_task          */
        s->count[a] -= 1;                          /* t is not best on a        */
        st->evictions += 1;
        tries += 1;
    }
    *hit_max = 1;
    return -1;
}

typedef struct {               /* simulation options                            */
    int32_t max_tries;         /* MAX_TRIES (s7), >= 1                           */
    int32_t eviction;          /* pop_condition on (1) / off (0)                 */
    int32_t top_n;             /* N3 candidates n (P:l.238: 10); <= 1 = root     */
    float eps;                 /* N3 epsilon (P:l.238: 0.8)                      */
    int32_t n_handles;         /* H                                              */
    int32_t n_nodes;           /* M (0 = default, l5)                            */
    const int64_t* acc_ptr;    /* [n+1] or NULL = no data model                  */
    const int32_t* acc_h;      /* [acc]                                          */
    const uint8_t* acc_mode;   /* [acc] 1 = R, 2 = W, 3 = RW                     */
    const uint64_t* size;      /* [H] bytes, < 2^28                              */
    const int32_t* worker_node;/* [W] or NULL = default (l5)                     */
    double xfer_ms_per_byte;   /* transfer time of non-resident data (l6)        */
} so_config;

/*
 * Inputs: the DAG (successor CSR, indeg), canonical durations dur[n][A]
 * (already perturbed for a replica), workers[A], the a7 keys key[n][A], the
 * eq. 1 gains gain[n][A] (used by the N3 epsilon filter; may be NULL when
 * top_n <= 1), options *cfg.  Workers are numbered arch-major (workers[0]
 * workers of arch 0 first, ...) (s2).  Outputs: *st, and if not NULL
 * start[n] (ms) and worker[n].
 */
int or_simulate(int32_t n, int32_t A, const int32_t* row_ptr, const int32_t* col, const int32_t* indeg,
                const float* dur, const int32_t* workers, const uint64_t* key, const float* gain,
                const so_config* cfg, so_stats* st, double* start, int32_t* worker) {
    if (n < 0 || A < 1 || A > 8 || !cfg || cfg->max_tries < 1) return SO_ERR_ARG;
    if (cfg->top_n > 1 && !gain) return SO_ERR_ARG;
    int32_t W = 0;
    for (int32_t a = 0; a < A; a++) W += workers[a] > 0 ? workers[a] : 0;
    if (W < 1) return SO_ERR_ARG;
    memset(st, 0, sizeof(*st));
    sched s;
    memset(&s, 0, sizeof(s));
    s.n = n; s.A = A; s.W = W; s.row_ptr = row_ptr; s.col = col; s.dur = dur; s.workers = workers;
    s.max_tries = cfg->max_tries; s.eviction = cfg->eviction;
    s.gain = gain; s.top_n = cfg->top_n; s.eps = cfg->eps;
    s.acc_ptr = cfg->acc_ptr; s.acc_h = cfg->acc_h; s.acc_mode = cfg->acc_mode; s.size = cfg->size;
    s.H = cfg->acc_ptr ? cfg->n_handles : 0;
    size_t nn = (size_t)n + 1;
    s.counted = (uint8_t*)calloc(nn * (size_t)A, 1);
    s.cand = (int32_t*)malloc((size_t)(s.top_n > 1 ? s.top_n : 1) * sizeof(int32_t));
    s.started = (uint8_t*)calloc(nn, 1);
    s.rem = (int32_t*)malloc(nn * sizeof(int32_t));
    int32_t* warch = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    int32_t* wtask = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    double* wend = (double*)malloc((size_t)W * sizeof(double));
    uint8_t* again = (uint8_t*)malloc((size_t)W);
    int32_t* wnode = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    u128 busy[8] = {0};
    int rc = SO_ERR_NOMEM;
    for (int32_t a = 0; a < A; a++) {
        s.h[a].v = (int32_t*)malloc(nn * sizeof(int32_t));
        s.h[a].key = key; s.h[a].A = A; s.h[a].a = a;
        if (!s.h[a].v) goto out;
    }
    if (!s.counted || !s.cand || !s.started || !s.rem || !warch || !wtask || !wend || !again || !wnode) goto out;
    for (int32_t a = 0, w = 0; a < A; a++)
        for (int32_t k = 0; k < workers[a]; k++, w++) { warch[w] = a; wtask[w] = -1; wend[w] = 0.0; }
    /* memory nodes (l5): given, or arch-0 workers share node 0 and every
     * other worker has its own node */
    s.M = 0;
    for (int32_t w = 0; w < W; w++) {
        wnode[w] = cfg->worker_node ? cfg->worker_node[w] : (warch[w] == 0 ? 0 : 1 + w - workers[0]);
        if (wnode[w] < 0) { rc = SO_ERR_ARG; goto out; }
        if (wnode[w] + 1 > s.M) s.M = wnode[w] + 1;
    }
    if (cfg->n_nodes > s.M) s.M = cfg->n_nodes;
    /* every handle starts in main memory, node 0 (l4) */
    s.resident = (uint8_t*)calloc((size_t)s.M * (size_t)(s.H > 0 ? s.H : 1), 1);
    if (!s.resident) goto out;
    for (int32_t hd = 0; hd < s.H; hd++) s.resident[hd] = 1;

    /* time 0: every task without predecessors is ready (P:l.91) */
    for (int32_t t = 0; t < n; t++) {
        s.rem[t] = indeg[t];
        if (indeg[t] == 0) push(&s, t);
    }
    int32_t done = 0;
    double T = 0.0;
    rc = SO_OK;
    for (;;) {
        /* dispatch (s2, s7): idle workers call POP in id order; workers whose
         * POP ended on MAX_TRIES call it again, round-robin, at the same T */
        for (int32_t w = 0; w < W; w++) again[w] = wtask[w] < 0;
        for (int any = 1; any;) {
            any = 0;
            for (int32_t w = 0; w < W; w++) {
                if (!again[w]) continue;
                int hit;
                int32_t t = pop(&s, warch[w], wnode[w], st, &hit);
                again[w] = (uint8_t)hit;
                any |= hit;
                if (hit) st->rounds += 1;
                if (t >= 0) {
                    int32_t a = warch[w], m = wnode[w];
                    float d = dur[(int64_t)t * A + a];
                    /* data of t moves to node m; a write leaves m the only copy (l4) */
                    uint64_t miss = 0;
                    if (s.acc_ptr) {
                        for (int64_t i = s.acc_ptr[t]; i < s.acc_ptr[t + 1]; i++)
                            if (!s.resident[(int64_t)m * s.H + s.acc_h[i]]) miss += s.size[s.acc_h[i]];
                        for (int64_t i = s.acc_ptr[t]; i < s.acc_ptr[t + 1]; i++) {
                            int32_t hd = s.acc_h[i];
                            if (s.acc_mode[i] & 2)
                                for (int32_t m2 = 0; m2 < s.M; m2++) s.resident[(int64_t)m2 * s.H + hd] = 0;
                            s.resident[(int64_t)m * s.H + hd] = 1;
                        }
                    }
                    st->moved += (int64_t)miss;
                    double x = (double)miss * cfg->xfer_ms_per_byte;    /* l6 */
                    wtask[w] = t;
                    wend[w] = T + ((double)d + x);          /* s1 */
                    if (start) start[t] = T;
                    if (worker) worker[t] = w;
                    busy[a] += fx(d);
                    st->ran[a] += 1;
                }
            }
        }
        /* next event: earliest completion (s2) */
        int32_t nb = 0;
        double Tn = INFINITY;
        for (int32_t w = 0; w < W; w++)
            if (wtask[w] >= 0) { nb++; if (wend[w] < Tn) Tn = wend[w]; }
        if (nb == 0) break;
        T = Tn;
        /* completions at T in worker id order release successors (P:l.91) */
        for (int32_t w = 0; w < W; w++) {
            if (wtask[w] < 0 || wend[w] != T) continue;
            int32_t t = wtask[w];
            wtask[w] = -1;
            done++;
            for (int32_t e = row_ptr[t]; e < row_ptr[t + 1]; e++)
                if (--s.rem[col[e]] == 0) push(&s, col[e]);
        }
    }
    if (done != n) rc = SO_ERR_STUCK;
    st->makespan = T;
    for (int32_t a = 0; a < A; a++) st->busy[a] = ldexp((double)busy[a], -64);
out:
    for (int32_t a = 0; a < A; a++) free(s.h[a].v);
    free(s.counted); free(s.started); free(s.rem); free(warch); free(wtask); free(wend); free(again);
    free(wnode); free(s.resident); free(s.cand);
    return rc;
}
