/*
 * mp_oracle.c -- plain, slow, single-threaded CPU oracle for the MultiPrio
 * scoring / queue-build hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant generator with the CUDA
 * library (paper_conf_ipps_tayebbfg24_b200/csrc); neither includes the other.
 *
 * Build: gcc -O2 -ffp-contract=off -fno-fast-math -shared -fPIC
 * Every binary32 quantity is a C `float`; on x86-64 (SSE, FLT_EVAL_METHOD 0)
 * each +, -, *, / below is one IEEE-754 binary32 round-to-nearest-even op,
 * which is the precision the path is defined in (reading c14).
 *
 * Citations: "P:l.N" = /root/reference/PAPER.md line N.
 *
 * Pins, function by function (tests/test_oracle_pins.py unless noted; each
 * pins the function against something other than itself):
 *   or_build_dag        networkx topological_generations (levels), Cholesky /
 *                       QR closed forms n, E, depth, dedup and
 *                       id/self-loop errors (test_levels_equal_networkx_*,
 *                       test_cholesky_closed_forms, test_qr_closed_forms,
 *                       test_error_paths)
 *   or_check_durations  domain edges 2^-41 / 2^20, NaN, -0, no enabled arch
 *                       (test_error_paths, test_best_remaining_work_exact)
 *   or_bottom_level     brute-force path enumeration on dyadic DAGs, networkx
 *                       longest path, chain/star, Cholesky CP closed form
 *   or_bottom_level_w   Fractions (mean-weight longest path) (test_n4_oracle)
 *   or_nod              Fig. 3's printed 2.5 / 1 (P:l.198), Fractions within
 *                       the c11 bound, in-tree 1/indeg
 *   or_nod_remaining    Fig. 3's dynamic scenario, Fractions (test_n4_oracle)
 *   or_affinity         Table II's six printed gains and hd = 19 (P:l.180-187),
 *                       the rule as worded in P:l.170-172, brute-force hd,
 *                       two-arch symmetry, hd = 0, workers = 0
 *   or_affinity_prefix  Table II in the paper's push order, a hand-worked
 *                       other order (test_n4_oracle)
 *   or_score  (BL)      Appendix-A crit_n (bl / CP), key order vs Python tuple
 *                       order on float32 values (test_score_key_packing_order)
 *   or_score  (NOD)     per-arch normalisation (P:l.166, reading c9) against
 *                       hand-worked Fig. 3 values with a masked arch and exact
 *                       Fractions on 3-arch masked DAGs
 *                       (test_nod_crit_norm_*)
 *   or_build_queues     Python sorted() on (-gain, -crit_n, id), membership and
 *                       duplication (P:l.104), READY membership, Appendix-A
 *                       queues, brw exact vs Fractions
 *   or_perturb          splitmix64 published reference vector, sigma range and
 *                       sigma = 0 identity
 *   or_replica          equals the stepwise path; sigma = 0 equals c2
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

enum { OR_OK = 0, OR_ERR_ARG = 1, OR_ERR_CYCLE = 2, OR_ERR_DOMAIN = 3, OR_ERR_NOMEM = 5 };

typedef struct {           /* one queue summary, Alg. 1 counters (P:l.135) */
    int32_t count;         /* ready_tasks_count[m]                          */
    int32_t head;          /* root of the heap h_m (first queue entry) or -1 */
    uint64_t brw_lo;       /* best_remaining_work[m] as an exact integer     */
    int64_t brw_hi;        /*   in units of 2^-64 ms (128-bit, hi:lo)        */
    double brw;            /* that integer x 2^-64, rounded once to double   */
} or_summary;

/* --------------------------------------------------------------------- */
/* a1 + a2: DAG ingest and topological levels                             */
/* G=(V,E), lambda^-(t), lambda^+(t) are sets (P:l.83-84 Table I, l.89).  */
/* --------------------------------------------------------------------- */

static int cmp_u64(const void* a, const void* b) {
    uint64_t x = *(const uint64_t*)a, y = *(const uint64_t*)b;
    return (x > y) - (x < y);
}

/* Outputs: row_ptr[n+1], col[cap m] (successor ids, ascending per row),
 * indeg[n], level[n], level_ptr[n+1], level_order[n]; *out_E, *out_L.
 * level(v) = 0 if v has no predecessor, else 1 + max level(pred) (Kahn,
 * FIFO); level_order = ids stably sorted by level. */
int or_build_dag(int32_t n, int64_t m, const int32_t* src, const int32_t* dst,
                 int32_t* row_ptr, int32_t* col, int32_t* indeg, int32_t* level,
                 int32_t* level_ptr, int32_t* level_order, int64_t* out_E, int32_t* out_L) {
    if (n < 0 || m < 0) return OR_ERR_ARG;
    for (int64_t i = 0; i < m; i++) {
        if (src[i] < 0 || src[i] >= n || dst[i] < 0 || dst[i] >= n) return OR_ERR_ARG;
        if (src[i] == dst[i]) return OR_ERR_ARG;               /* self-loop */
    }
    uint64_t* pr = (uint64_t*)malloc((size_t)(m > 0 ? m : 1) * sizeof(uint64_t));
    int32_t* rem = (int32_t*)malloc((size_t)(n > 0 ? n : 1) * sizeof(int32_t));
    int32_t* fifo = (int32_t*)malloc((size_t)(n > 0 ? n : 1) * sizeof(int32_t));
    int32_t* cnt = (int32_t*)calloc((size_t)n + 1, sizeof(int32_t));
    if (!pr || !rem || !fifo || !cnt) { free(pr); free(rem); free(fifo); free(cnt); return OR_ERR_NOMEM; }
    for (int64_t i = 0; i < m; i++) pr[i] = ((uint64_t)(uint32_t)src[i] << 32) | (uint32_t)dst[i];
    qsort(pr, (size_t)m, sizeof(uint64_t), cmp_u64);
    int64_t E = 0;                                            /* set semantics: dedup */
    for (int64_t i = 0; i < m; i++)
        if (i == 0 || pr[i] != pr[i - 1]) pr[E++] = pr[i];
    for (int32_t v = 0; v <= n; v++) row_ptr[v] = 0;
    for (int32_t v = 0; v < n; v++) indeg[v] = 0;
    for (int64_t i = 0; i < E; i++) {
        int32_t u = (int32_t)(pr[i] >> 32), v = (int32_t)(pr[i] & 0xffffffffu);
        row_ptr[u + 1]++;
        indeg[v]++;
        col[i] = v;
    }
    for (int32_t v = 0; v < n; v++) row_ptr[v + 1] += row_ptr[v];

    /* Kahn with a FIFO; a task is ready when all predecessors are done (P:l.91) */
    int32_t head = 0, tail = 0;
    for (int32_t v = 0; v < n; v++) {
        rem[v] = indeg[v];
        level[v] = 0;
        if (rem[v] == 0) fifo[tail++] = v;
    }
    while (head < tail) {
        int32_t u = fifo[head++];
        for (int32_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) {
            int32_t v = col[e];
            if (level[u] + 1 > level[v]) level[v] = level[u] + 1;
            if (--rem[v] == 0) fifo[tail++] = v;
        }
    }
    int rc = OR_OK;
    int32_t L = 0;
    if (tail < n) {
        rc = OR_ERR_CYCLE;
    } else {
        for (int32_t v = 0; v < n; v++)
            if (level[v] + 1 > L) L = level[v] + 1;
        for (int32_t v = 0; v < n; v++) cnt[level[v] + 1]++;  /* stable counting sort */
        for (int32_t l = 0; l < L; l++) cnt[l + 1] += cnt[l];
        for (int32_t l = 0; l <= L; l++) level_ptr[l] = cnt[l];
        for (int32_t v = 0; v < n; v++) level_order[cnt[level[v]]++] = v;
    }
    *out_E = E;
    *out_L = L;
    free(pr); free(rem); free(fifo); free(cnt);
    return rc;
}

/* --------------------------------------------------------------------- */
/* a3: enabled mask, node weight, domain                                   */
/* Alg. 1 (P:l.135): can_exec(t,a) and get_worker_count(a) > 0.            */
/* --------------------------------------------------------------------- */

static const float OR_DMIN = 0x1p-41f;   /* reading c20 */
static const float OR_DMAX = 0x1p20f;

/* Canonicalise -0 -> +0 into `out`; OR_ERR_DOMAIN on NaN, negative values,
 * nonzero |d| < 2^-41, finite d >= 2^20, or a task with no enabled arch. */
int or_check_durations(int32_t n, int32_t A, const float* dur, const int32_t* workers, float* out) {
    if (n < 0 || A < 1 || A > 8) return OR_ERR_ARG;
    for (int64_t i = 0; i < (int64_t)n * A; i++) {
        float d = dur[i];
        if (d == 0.0f) d = 0.0f;
        if (isnan(d) || d < 0.0f) return OR_ERR_DOMAIN;
        if (!isinf(d) && d != 0.0f && (d < OR_DMIN || d >= OR_DMAX)) return OR_ERR_DOMAIN;
        out[i] = d;
    }
    for (int32_t t = 0; t < n; t++) {
        int k = 0;
        for (int32_t a = 0; a < A; a++) k += (!isinf(out[(int64_t)t * A + a]) && workers[a] > 0);
        if (k == 0) return OR_ERR_DOMAIN;
    }
    return OR_OK;
}

static int enabled(const float* dur, const int32_t* workers, int32_t A, int32_t t, int32_t a) {
    return !isinf(dur[(int64_t)t * A + a]) && workers[a] > 0;
}

/* w(t) = min over enabled archs of delta(t,a) (reading c2, "critical path
 * with infinite resources", P:l.265). */
static float weight(const float* dur, const int32_t* workers, int32_t A, int32_t t) {
    float w = INFINITY;
    for (int32_t a = 0; a < A; a++)
        if (enabled(dur, workers, A, t, a) && dur[(int64_t)t * A + a] < w) w = dur[(int64_t)t * A + a];
    return w;
}

/* --------------------------------------------------------------------- */
/* a4: bottom-level (north_star): bl(v) = w(v) + max_{s in succ(v)} bl(s),  */
/* bl(v) = w(v) when v has no successor; CP = max_v bl(v).                 */
/* --------------------------------------------------------------------- */
/* N4: HEFT-style mean cost as the node weight (reading v1):
 * w(t) = (sum over enabled a, in arch order, of W_a * delta(t,a)) / sum of
 * W_a, each op one RN binary64 op, rounded once to binary32. */
static float weight_mean(const float* dur, const int32_t* workers, int32_t A, int32_t t) {
    double num = 0.0;
    int64_t den = 0;
    for (int32_t a = 0; a < A; a++)
        if (enabled(dur, workers, A, t, a)) {
            num = num + (double)workers[a] * (double)dur[(int64_t)t * A + a];
            den += workers[a];
        }
    return (float)(num / (double)den);
}

static int bottom_level_kind(int32_t n, int32_t A, const int32_t* row_ptr, const int32_t* col,
                             const int32_t* level_order, const float* dur_in, const int32_t* workers,
                             int32_t wkind, float* bl, float* cp);

int or_bottom_level(int32_t n, int32_t A, const int32_t* row_ptr, const int32_t* col,
                    const int32_t* level_order, const float* dur_in, const int32_t* workers,
                    float* bl, float* cp) {
    return bottom_level_kind(n, A, row_ptr, col, level_order, dur_in, workers, 0, bl, cp);
}

/* wkind 0: w = min over enabled archs (c2); 1: mean cost (v1) */
int or_bottom_level_w(int32_t n, int32_t A, const int32_t* row_ptr, const int32_t* col,
                      const int32_t* level_order, const float* dur_in, const int32_t* workers,
                      int32_t wkind, float* bl, float* cp) {
    if (wkind < 0 || wkind > 1) return OR_ERR_ARG;
    return bottom_level_kind(n, A, row_ptr, col, level_order, dur_in, workers, wkind, bl, cp);
}

static int bottom_level_kind(int32_t n, int32_t A, const int32_t* row_ptr, const int32_t* col,
                             const int32_t* level_order, const float* dur_in, const int32_t* workers,
                             int32_t wkind, float* bl, float* cp) {
    float* dur = (float*)malloc((size_t)((int64_t)n * A + 1) * sizeof(float));
    if (!dur) return OR_ERR_NOMEM;
    int rc = or_check_durations(n, A, dur_in, workers, dur);
    if (rc) { free(dur); return rc; }
    float best = 0.0f;
    for (int32_t i = n - 1; i >= 0; i--) {                /* reverse topological order */
        int32_t v = level_order[i];
        float w = wkind ? weight_mean(dur, workers, A, v) : weight(dur, workers, A, v);
        if (row_ptr[v] == row_ptr[v + 1]) {
            bl[v] = w;
        } else {
            float mx = -INFINITY;
            for (int32_t e = row_ptr[v]; e < row_ptr[v + 1]; e++)
                if (bl[col[e]] > mx) mx = bl[col[e]];
            bl[v] = w + mx;
        }
        if (bl[v] > best) best = bl[v];
    }
    *cp = best;
    free(dur);
    return OR_OK;
}

/* --------------------------------------------------------------------- */
/* a5: NOD (eq. 2, P:l.193):                                               */
/*   NOD(t) = sum_{s in lambda+(t, P_m)} 1 / |lambda-(s, P_m)|             */
/* with lambda+/- filtered by can-execute on arch a (reading c10) and each */
/* term taken as floor(2^32 / |lambda-|) in a 64-bit integer (reading c11) */
/* converted once to binary32 and scaled by 2^-32.  nod = 0 when (t,a) is  */
/* not enabled.                                                            */
/* --------------------------------------------------------------------- */
static int nod_done(int32_t n, int32_t A, const int32_t* row_ptr, const int32_t* col,
                    const float* dur_in, const int32_t* workers, const uint8_t* done, float* nod);

int or_nod(int32_t n, int32_t A, const int32_t* row_ptr, const int32_t* col,
           const float* dur_in, const int32_t* workers, float* nod) {
    return nod_done(n, A, row_ptr, col, dur_in, workers, NULL, nod);
}

/* N4: NOD against the REMAINING graph (reading v3): completed tasks (done)
 * leave lambda-; successors that are done and done tasks themselves score 0.
 * With done = all-zero this is or_nod. */
int or_nod_remaining(int32_t n, int32_t A, const int32_t* row_ptr, const int32_t* col,
                     const float* dur_in, const int32_t* workers, const uint8_t* done, float* nod) {
    return nod_done(n, A, row_ptr, col, dur_in, workers, done, nod);
}

static int nod_done(int32_t n, int32_t A, const int32_t* row_ptr, const int32_t* col,
                    const float* dur_in, const int32_t* workers, const uint8_t* done, float* nod) {
    float* dur = (float*)malloc((size_t)((int64_t)n * A + 1) * sizeof(float));
    int32_t* ind = (int32_t*)calloc((size_t)n + 1, sizeof(int32_t));
    if (!dur || !ind) { free(dur); free(ind); return OR_ERR_NOMEM; }
    int rc = or_check_durations(n, A, dur_in, workers, dur);
    if (rc) { free(dur); free(ind); return rc; }
    for (int32_t a = 0; a < A; a++) {
        for (int32_t s = 0; s < n; s++) ind[s] = 0;
        for (int32_t p = 0; p < n; p++)                        /* |lambda-(s, P_a)| */
            if (enabled(dur, workers, A, p, a) && !(done && done[p]))
                for (int32_t e = row_ptr[p]; e < row_ptr[p + 1]; e++) ind[col[e]]++;
        for (int32_t t = 0; t < n; t++) {
            float v = 0.0f;
            if (enabled(dur, workers, A, t, a) && !(done && done[t])) {
                uint64_t acc = 0;
                for (int32_t e = row_ptr[t]; e < row_ptr[t + 1]; e++) {
                    int32_t s = col[e];
                    if (enabled(dur, workers, A, s, a) && !(done && done[s]))
                        acc += (uint64_t)(4294967296ull / (uint64_t)ind[s]);
                }
                v = (float)acc * 0x1p-32f;
            }
            nod[(int64_t)t * A + a] = v;
        }
    }
    free(dur); free(ind);
    return OR_OK;
}

/* --------------------------------------------------------------------- */
/* a6: gain heuristic (eq. 1, P:l.172; hd(a) P:l.176; Table II l.180-187). */
/*   gain = 1 if only one arch type can perform t (P:l.170, reading c7);   */
/*   otherwise ((ref - delta(t,a)) + hd(a)) / (2 hd(a)), where ref is the  */
/*   second-fastest time if a is the fastest, else the fastest, i.e.       */
/*   ref = min over the other enabled archs (reading c6); hd(a) = max |d|  */
/*   over the scored set (readings c4, c5); 0.5 when hd(a) = 0 (c8).       */
/* flags bit0 = enabled(t,a); bit1 = "normalized_speedup(t,a) == 1"       */
/*   (delta(t,a) == w(t), Alg. 1 P:l.135, reading c15).                    */
/* --------------------------------------------------------------------- */
int or_affinity(int32_t n, int32_t A, const float* dur_in, const int32_t* workers,
                float* gain, float* hd, uint8_t* flags) {
    float* dur = (float*)malloc((size_t)((int64_t)n * A + 1) * sizeof(float));
    float* dd = (float*)malloc((size_t)((int64_t)n * A + 1) * sizeof(float));
    if (!dur || !dd) { free(dur); free(dd); return OR_ERR_NOMEM; }
    int rc = or_check_durations(n, A, dur_in, workers, dur);
    if (rc) { free(dur); free(dd); return rc; }
    for (int32_t a = 0; a < A; a++) hd[a] = 0.0f;
    for (int32_t t = 0; t < n; t++) {
        int k = 0;
        for (int32_t a = 0; a < A; a++) k += enabled(dur, workers, A, t, a);
        float w = weight(dur, workers, A, t);
        for (int32_t a = 0; a < A; a++) {
            int64_t i = (int64_t)t * A + a;
            flags[i] = 0;
            dd[i] = 0.0f;
            if (!enabled(dur, workers, A, t, a)) continue;
            flags[i] = 1 | (dur[i] == w ? 2 : 0);
            if (k < 2) continue;
            float ref = INFINITY;
            for (int32_t b = 0; b < A; b++)
                if (b != a && enabled(dur, workers, A, t, b) && dur[(int64_t)t * A + b] < ref)
                    ref = dur[(int64_t)t * A + b];
            dd[i] = ref - dur[i];
            if (fabsf(dd[i]) > hd[a]) hd[a] = fabsf(dd[i]);
        }
    }
    for (int32_t t = 0; t < n; t++) {
        int k = 0;
        for (int32_t a = 0; a < A; a++) k += enabled(dur, workers, A, t, a);
        for (int32_t a = 0; a < A; a++) {
            int64_t i = (int64_t)t * A + a;
            if (!(flags[i] & 1)) gain[i] = 0.0f;
            else if (k == 1) gain[i] = 1.0f;
            else if (hd[a] == 0.0f) gain[i] = 0.5f;
            else gain[i] = (dd[i] + hd[a]) / (hd[a] + hd[a]);
        }
    }
    free(dur); free(dd);
    return OR_OK;
}

/* --------------------------------------------------------------------- */
/* a7: normalised criticality and the combined key.                        */
/* "All values are normalized between 0 and 1" (P:l.166): crit_n = crit / */
/* max crit (reading c9).  Tasks are sorted first by gain, then by         */
/* criticality (P:l.138, l.322): key = ((0x3F800000 - bits(gain)) << 32)  */
/*   | (0x3F800000 - bits(crit_n)); ascending key = (gain desc, crit desc). */
/* kind 0: crit = bl[n] (crit_norm[n]); kind 1: crit = nod[n][A]           */
/* normalised per arch over enabled tasks (crit_norm[n][A]).               */
/* --------------------------------------------------------------------- */
/* --------------------------------------------------------------------- */
/* N4: hd(a) "recorded so far" read literally (P:l.176, reading v2): tasks  */
/* are pushed in the given order (NULL = id order) and each task's gain     */
/* uses the running max of |d| over the tasks pushed up to and including   */
/* it; hd[] returns the final max (= or_affinity's hd).                     */
/* --------------------------------------------------------------------- */
int or_affinity_prefix(int32_t n, int32_t A, const float* dur_in, const int32_t* workers,
                       const int32_t* order, float* gain, float* hd, uint8_t* flags) {
    float* dur = (float*)malloc((size_t)((int64_t)n * A + 1) * sizeof(float));
    if (!dur) return OR_ERR_NOMEM;
    int rc = or_check_durations(n, A, dur_in, workers, dur);
    if (rc) { free(dur); return rc; }
    float run[8] = {0};
    for (int32_t i = 0; i < n; i++) {
        int32_t t = order ? order[i] : i;
        if (t < 0 || t >= n) { free(dur); return OR_ERR_ARG; }
        int k = 0;
        for (int32_t a = 0; a < A; a++) k += enabled(dur, workers, A, t, a);
        float w = weight(dur, workers, A, t);
        float dd[8];
        for (int32_t a = 0; a < A; a++) {
            dd[a] = 0.0f;
            if (!enabled(dur, workers, A, t, a)) continue;
            float ref = INFINITY;
            for (int32_t b = 0; b < A; b++)
                if (b != a && enabled(dur, workers, A, t, b) && dur[(int64_t)t * A + b] < ref)
                    ref = dur[(int64_t)t * A + b];
            if (k >= 2) {
                dd[a] = ref - dur[(int64_t)t * A + a];
                if (fabsf(dd[a]) > run[a]) run[a] = fabsf(dd[a]);      /* pushed: recorded */
            }
        }
        for (int32_t a = 0; a < A; a++) {
            int64_t j = (int64_t)t * A + a;
            float g = 0.0f;
            uint8_t f = 0;
            if (enabled(dur, workers, A, t, a)) {
                f = 1 | (dur[j] == w ? 2 : 0);
                if (k == 1) g = 1.0f;
                else if (run[a] == 0.0f) g = 0.5f;
                else g = (dd[a] + run[a]) / (run[a] + run[a]);
            }
            gain[j] = g;
            flags[j] = f;
        }
    }
    for (int32_t a = 0; a < A; a++) hd[a] = run[a];
    free(dur);
    return OR_OK;
}

static uint32_t f2u(float x) { uint32_t u; memcpy(&u, &x, 4); return u; }

int or_score(int32_t n, int32_t A, int32_t kind, const float* crit, const float* gain,
             const uint8_t* flags, float* crit_norm, uint64_t* key) {
    if (n < 0 || A < 1 || A > 8 || (kind != 0 && kind != 1)) return OR_ERR_ARG;
    if (kind == 0) {
        float mx = 0.0f;
        for (int32_t t = 0; t < n; t++) if (crit[t] > mx) mx = crit[t];
        for (int32_t t = 0; t < n; t++) crit_norm[t] = mx > 0.0f ? crit[t] / mx : 0.0f;
    } else {
        for (int32_t a = 0; a < A; a++) {
            float mx = 0.0f;
            for (int32_t t = 0; t < n; t++)
                if ((flags[(int64_t)t * A + a] & 1) && crit[(int64_t)t * A + a] > mx) mx = crit[(int64_t)t * A + a];
            for (int32_t t = 0; t < n; t++) {
                int64_t i = (int64_t)t * A + a;
                crit_norm[i] = ((flags[i] & 1) && mx > 0.0f) ? crit[i] / mx : 0.0f;
            }
        }
    }
    for (int32_t t = 0; t < n; t++)
        for (int32_t a = 0; a < A; a++) {
            int64_t i = (int64_t)t * A + a;
            if (!(flags[i] & 1)) { key[i] = UINT64_MAX; continue; }
            float c = kind == 0 ? crit_norm[t] : crit_norm[i];
            key[i] = ((uint64_t)(0x3F800000u - f2u(gain[i])) << 32) | (uint64_t)(0x3F800000u - f2u(c));
        }
    return OR_OK;
}

/* --------------------------------------------------------------------- */
/* a8 + a9: one queue per architecture type (heaps h_m, P:l.97, l.104,     */
/* l.130; reading c13), entries sorted by (key asc, id asc) (reading c12); */
/* summaries = Alg. 1 counters.  READY mode (done != NULL): only tasks     */
/* t with !done(t) and all predecessors done (P:l.91, reading c18).        */
/* --------------------------------------------------------------------- */
static _Thread_local const uint64_t* g_sort_key;   /* qsort context, per thread (tests and the
                                                    cpu baseline call the oracle from threads) */
static int cmp_entry(const void* pa, const void* pb) {
    int32_t a = *(const int32_t*)pa, b = *(const int32_t*)pb;
    uint64_t ka = g_sort_key[a], kb = g_sort_key[b];
    if (ka != kb) return ka < kb ? -1 : 1;
    return (a > b) - (a < b);
}

typedef unsigned __int128 u128;

/* delta (ms, binary32, 0 or in [2^-41, 2^20)) as an integer number of 2^-64 ms */
static u128 fixed64(float d) {
    if (d == 0.0f) return 0;
    int e;
    float f = frexpf(d, &e);                  /* d = f * 2^e, f in [0.5, 1) */
    uint64_t mant = (uint64_t)ldexpf(f, 24);  /* exact 24-bit integer */
    return (u128)mant << (e - 24 + 64);
}

int or_build_queues(int32_t n, int32_t A, const int32_t* row_ptr, const int32_t* col,
                    const uint64_t* key, const uint8_t* flags, const float* dur,
                    const uint8_t* done, int64_t* qptr, int32_t* qtask, or_summary* sum) {
    if (n < 0 || A < 1 || A > 8) return OR_ERR_ARG;
    uint8_t* blocked = (uint8_t*)calloc((size_t)n + 1, 1);
    int32_t* tmp = (int32_t*)malloc(((size_t)n + 1) * sizeof(int32_t));
    uint64_t* ka = (uint64_t*)malloc(((size_t)n + 1) * sizeof(uint64_t));
    if (!blocked || !tmp || !ka) { free(blocked); free(tmp); free(ka); return OR_ERR_NOMEM; }
    if (done)
        for (int32_t u = 0; u < n; u++)
            if (!done[u])
                for (int32_t e = row_ptr[u]; e < row_ptr[u + 1]; e++) blocked[col[e]] = 1;
    qptr[0] = 0;
    for (int32_t a = 0; a < A; a++) {
        int32_t m = 0;
        for (int32_t t = 0; t < n; t++) {
            int ok = flags[(int64_t)t * A + a] & 1;
            if (done) ok = ok && !done[t] && !blocked[t];
            if (ok) tmp[m++] = t;
            ka[t] = key[(int64_t)t * A + a];
        }
        g_sort_key = ka;
        qsort(tmp, (size_t)m, sizeof(int32_t), cmp_entry);
        u128 acc = 0;
        for (int32_t i = 0; i < m; i++) {
            int32_t t = tmp[i];
            qtask[qptr[a] + i] = t;
            if (flags[(int64_t)t * A + a] & 2) {
                float d = dur[(int64_t)t * A + a];
                acc += fixed64(d == 0.0f ? 0.0f : d);
            }
        }
        qptr[a + 1] = qptr[a] + m;
        sum[a].count = m;
        sum[a].head = m > 0 ? tmp[0] : -1;
        sum[a].brw_lo = (uint64_t)acc;
        sum[a].brw_hi = (int64_t)(uint64_t)(acc >> 64);
        sum[a].brw = ldexp((double)acc, -64);
    }
    free(blocked); free(tmp); free(ka);
    return OR_OK;
}

/* --------------------------------------------------------------------- */
/* a10: one duration-perturbed replica (north_star "batched-replica mode"). */
/* delta_r(t,a) = delta(t,a) * (1 + sigma * (2u - 1)), u = top 24 bits of  */
/* splitmix64 at counter c = ((r * n + t) * A + a + 1) * 2^-24 (SURVEY     */
/* §8(a) a10).  Each float op is RN binary32; +inf and 0 are preserved.    */
/* --------------------------------------------------------------------- */
static uint64_t splitmix64(uint64_t seed, uint64_t c) {
    uint64_t x = seed + c * 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

void or_perturb(int32_t n, int32_t A, const float* base, uint64_t seed, float sigma, int64_t r, float* out) {
    for (int32_t t = 0; t < n; t++)
        for (int32_t a = 0; a < A; a++) {
            uint64_t c = ((uint64_t)r * (uint64_t)n + (uint64_t)t) * (uint64_t)A + (uint64_t)a + 1u;
            float u = (float)(splitmix64(seed, c) >> 40) * 0x1p-24f;
            float twou = 2.0f * u;
            float s = twou - 1.0f;
            float sc = sigma * s;
            float f = 1.0f + sc;
            float d = base[(int64_t)t * A + a];
            out[(int64_t)t * A + a] = d * f;
        }
}

/* Full path for replica r: perturb, w, bl, CP, gain, crit_n = bl / CP, key,
 * queues (ALL mode) and summaries.  qtask may be NULL (summaries only). */
int or_replica(int32_t n, int32_t A, const int32_t* row_ptr, const int32_t* col,
               const int32_t* level_order, const float* base, const int32_t* workers,
               uint64_t seed, float sigma, int64_t r, float* cp, or_summary* sum,
               int32_t* qtask, int64_t* qptr) {
    size_t nA = (size_t)n * (size_t)A + 1;
    float* d = (float*)malloc(nA * sizeof(float));
    float* dc = (float*)malloc(nA * sizeof(float));
    float* bl = (float*)malloc(((size_t)n + 1) * sizeof(float));
    float* gain = (float*)malloc(nA * sizeof(float));
    float* critn = (float*)malloc(((size_t)n + 1) * sizeof(float));
    uint64_t* key = (uint64_t*)malloc(nA * sizeof(uint64_t));
    uint8_t* flags = (uint8_t*)malloc(nA);
    int32_t* q = qtask ? qtask : (int32_t*)malloc(nA * sizeof(int32_t));
    int64_t qp[9];
    float hd[8];
    int rc = OR_ERR_NOMEM;
    if (!d || !dc || !bl || !gain || !critn || !key || !flags || !q) goto done;
    or_perturb(n, A, base, seed, sigma, r, d);
    rc = or_check_durations(n, A, d, workers, dc);
    if (rc) goto done;
    rc = or_bottom_level(n, A, row_ptr, col, level_order, dc, workers, bl, cp);
    if (rc) goto done;
    rc = or_affinity(n, A, dc, workers, gain, hd, flags);
    if (rc) goto done;
    rc = or_score(n, A, 0, bl, gain, flags, critn, key);
    if (rc) goto done;
    rc = or_build_queues(n, A, row_ptr, col, key, flags, dc, NULL, qptr ? qptr : qp, q, sum);
done:
    free(d); free(dc); free(bl); free(gain); free(critn); free(key); free(flags);
    if (!qtask) free(q);
    return rc;
}
