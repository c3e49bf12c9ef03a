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
 * Readings (s1-s9) are cited inline as "sN".
 *
 * Pins (tests/test_oracle_pins.py, "sim" tests): hand-worked schedules of
 * Table II's tasks (P:l.180-187) with and without eviction, the closed forms
 * makespan = CP with unbounded workers and = sum of durations with one
 * worker, the list-scheduling bounds max(CP, W^-1 sum w) <= makespan <=
 * W^-1 sum w + (1 - 1/W) CP (one arch), and trace invariants (precedence,
 * no overlap, exactly-once, greedy / highest-priority-first without
 * eviction), plus Fig. 4's direction (eviction lowers GPU idle time).
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
    double busy[8];          /* sum of delta(t,a) over tasks run on arch a     */
    int32_t ran[8];          /* tasks run on arch a                            */
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

/* Alg. 2 POP for a worker of arch a (memory node w_m of type a, reading
 * c13).  Returns the task, or -1; *hit_max = 1 when MAX_TRIES ended it. */
static int32_t pop(sched* s, int32_t a, so_stats* st, int* hit_max) {
    heap* h = &s->h[a];
    int tries = 0;
    *hit_max = 0;
    while (tries < s->max_tries) {
        if (h->size == 0) return -1;
        int32_t t = h->v[0];                       /* get_most_local_prio_task: */
        if (s->started[t]) {                       /* the heap root (s6)        */
            heap_pop_root(h);                      /* processed duplicate:      */
            continue;                              /* removed, not a try (s5)   */
        }
        if (pop_condition(s, t, a)) {
            heap_pop_root(h);                      /* heaps_pop_and_update      */
            for (int32_t b = 0; b < s->A; b++)     /* "any duplicate tasks in   */
                if (b != a && s->counted[(int64_t)t * s->A + b])   /* other     */
                    st->dups += 1;                 /* queues will remain there" */
            uncount(s, t);
            s->started[t] = 1;
            st->pops += 1;
            return t;
        }
        heap_pop_root(h);                          /* heaps_evict_task          */
        s->counted[(int64_t)t * s->A + a] = 0;
        s->count[a] -= 1;                          /* t is not best on a        */
        st->evictions += 1;
        tries += 1;
    }
    *hit_max = 1;
    return -1;
}

/*
 * Inputs: the DAG (successor CSR, indeg), canonical durations dur[n][A]
 * (already perturbed for a replica), workers[A], the a7 keys key[n][A],
 * max_tries >= 1, eviction in {0,1}.  Workers are numbered arch-major
 * (workers[0] workers of arch 0 first, ...) (s2).  Outputs: *st, and if not
 * NULL start[n] (ms) and worker[n].
 */
int or_simulate(int32_t n, int32_t A, const int32_t* row_ptr, const int32_t* col, const int32_t* indeg,
                const float* dur, const int32_t* workers, const uint64_t* key, int32_t max_tries,
                int32_t eviction, so_stats* st, double* start, int32_t* worker) {
    if (n < 0 || A < 1 || A > 8 || max_tries < 1) return SO_ERR_ARG;
    int32_t W = 0;
    for (int32_t a = 0; a < A; a++) W += workers[a] > 0 ? workers[a] : 0;
    if (W < 1) return SO_ERR_ARG;
    memset(st, 0, sizeof(*st));
    sched s;
    memset(&s, 0, sizeof(s));
    s.n = n; s.A = A; s.W = W; s.row_ptr = row_ptr; s.col = col; s.dur = dur; s.workers = workers;
    s.max_tries = max_tries; s.eviction = eviction;
    size_t nn = (size_t)n + 1;
    s.counted = (uint8_t*)calloc(nn * (size_t)A, 1);
    s.started = (uint8_t*)calloc(nn, 1);
    s.rem = (int32_t*)malloc(nn * sizeof(int32_t));
    int32_t* warch = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    int32_t* wtask = (int32_t*)malloc((size_t)W * sizeof(int32_t));
    double* wend = (double*)malloc((size_t)W * sizeof(double));
    uint8_t* again = (uint8_t*)malloc((size_t)W);
    u128 busy[8] = {0};
    int rc = SO_ERR_NOMEM;
    for (int32_t a = 0; a < A; a++) {
        s.h[a].v = (int32_t*)malloc(nn * sizeof(int32_t));
        s.h[a].key = key; s.h[a].A = A; s.h[a].a = a;
        if (!s.h[a].v) goto out;
    }
    if (!s.counted || !s.started || !s.rem || !warch || !wtask || !wend || !again) goto out;
    for (int32_t a = 0, w = 0; a < A; a++)
        for (int32_t k = 0; k < workers[a]; k++, w++) { warch[w] = a; wtask[w] = -1; wend[w] = 0.0; }

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
                int32_t t = pop(&s, warch[w], st, &hit);
                again[w] = (uint8_t)hit;
                any |= hit;
                if (hit) st->rounds += 1;
                if (t >= 0) {
                    int32_t a = warch[w];
                    float d = dur[(int64_t)t * A + a];
                    wtask[w] = t;
                    wend[w] = T + (double)d;              /* s1 */
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
    return rc;
}
