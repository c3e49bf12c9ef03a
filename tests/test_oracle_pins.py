"""Pins of the CPU oracle against things other than itself (-m "not gpu").

Each test names the PAPER.md passage (P:l.N) or mathematical fact it pins.
A plausible mistake anywhere in the oracle (dropped term, wrong sign or index,
transposed operand, wrong tie-break, wrong rounding) fails at least one test.
"""
from __future__ import annotations

import itertools
import json
import math
import os
from fractions import Fraction

import networkx as nx
import numpy as np
import pytest

import oracle
import workloads
from workloads import dense, random_dags

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def load(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def f32(x):
    return float(np.float32(x))


# ----------------------------------------------------------------------------
# a6 gain: Table II (P:l.180-187), eq. 1 (P:l.172), hd (P:l.176)
# ----------------------------------------------------------------------------

def test_table2_gain_values_and_hd():
    g = load("table2_gain.json")
    dur = np.array(g["dur_ms"], np.float32)
    gain, hd, flags = oracle.affinity(dur, np.ones(2, np.int32))
    assert hd.tolist() == g["hd"]
    printed = np.array(g["gain_printed"])
    # the paper prints 3 decimals, truncated (0.6316 -> 0.631)
    assert np.all(np.abs(gain - printed) < 1e-3)
    assert np.all(np.floor(gain.astype(np.float64) * 1000 + 1e-9) / 1000 == printed)
    assert gain[0, 0] == 1.0 and gain[0, 1] == 0.0      # d = +-hd  ->  exactly 1 / 0
    assert np.all(flags & 1)
    # is_best (normalized_speedup == 1, Alg. 1 P:l.135): a1 for tA, tB; a2 for tC
    assert ((flags >> 1) & 1).tolist() == [[1, 0], [1, 0], [0, 1]]


def test_table2_heap_orders():
    """P:l.178: a1 heap tA > tB > tC; a2 heap tC > tB > tA."""
    g = load("table2_gain.json")
    dur = np.array(g["dur_ms"], np.float32)
    dag = oracle.build_dag(3, [], [])
    r = oracle.score_and_queue(dag, dur, np.ones(2, np.int32))
    names = g["tasks"]
    q = r["qtask"]
    assert [names[i] for i in q[:3]] == g["heap_order_a1"]
    assert [names[i] for i in q[3:]] == g["heap_order_a2"]


def _gain_literal_rule(dur_row, workers, a, hd):
    """P:l.170-172 as worded: 1 if one type can perform t; if a is the fastest use
    the second fastest, else the fastest (written from the text, not the oracle)."""
    en = [b for b in range(len(dur_row)) if math.isfinite(dur_row[b]) and workers[b] > 0]
    if len(en) == 1:
        return 1.0
    order = sorted(en, key=lambda b: (dur_row[b], b))
    first, second = order[0], order[1]
    ref = dur_row[second] if a == first else dur_row[first]
    if hd == 0:
        return 0.5
    d = np.float32(np.float32(ref) - np.float32(dur_row[a]))
    return float(np.float32(np.float32(d + np.float32(hd)) / np.float32(np.float32(hd) + np.float32(hd))))


@pytest.mark.parametrize("A,seed", [(2, 1), (3, 2), (3, 3), (4, 4)])
def test_gain_matches_worded_rule_and_ranges(A, seed):
    dur = random_dags.dyadic_durations(300, A, seed, p_inf=0.3)
    workers = np.ones(A, np.int32)
    gain, hd, flags = oracle.affinity(dur, workers)
    for t in range(300):
        en = np.isfinite(dur[t])
        for a in range(A):
            if not en[a]:
                assert flags[t, a] == 0
                continue
            assert gain[t, a] == _gain_literal_rule(dur[t].tolist(), workers, a, hd[a])
            assert 0.0 <= gain[t, a] <= 1.0                      # P:l.166
            if en.sum() == 1:
                assert gain[t, a] == 1.0                          # P:l.170
    # hd(a) = max |d| over multi-arch tasks enabled on a: brute force
    for a in range(A):
        best = 0.0
        for t in range(300):
            en = [b for b in range(A) if np.isfinite(dur[t, b])]
            if a in en and len(en) > 1:
                ref = min(dur[t, b] for b in en if b != a)
                best = max(best, abs(float(ref) - float(dur[t, a])))
        assert hd[a] == np.float32(best)


def test_gain_two_arch_symmetry():
    """With 2 archs hd(a1) = hd(a2) and eq. 1 gives gain(a1) + gain(a2) = 1 in the reals."""
    dur = random_dags.dyadic_durations(2000, 2, 9)
    gain, hd, _ = oracle.affinity(dur, np.ones(2, np.int32))
    assert hd[0] == hd[1]
    s = gain[:, 0].astype(np.float64) + gain[:, 1]
    assert np.all(np.abs(s - 1.0) <= 2.0 ** -23)


def test_gain_hd_zero_and_workers_disable():
    dur = np.array([[2.0, 2.0], [3.0, 3.0]], np.float32)
    gain, hd, flags = oracle.affinity(dur, np.ones(2, np.int32))
    assert hd.tolist() == [0.0, 0.0] and np.all(gain == 0.5)     # reading c8
    assert np.all(flags == 3)                                     # ties are best on both (c15)
    gain, hd, flags = oracle.affinity(dur, np.array([1, 0], np.int32))
    assert np.all(gain[:, 0] == 1.0) and np.all(flags[:, 1] == 0)  # get_worker_count(a) = 0


# ----------------------------------------------------------------------------
# a5 NOD: eq. 2 (P:l.193), Fig. 3 values (P:l.198)
# ----------------------------------------------------------------------------

def test_fig3_nod_values():
    g = load("fig3_nod.json")
    idx = {t: i for i, t in enumerate(g["tasks"])}
    src = [idx[u] for u, v in g["edges"]]
    dst = [idx[v] for u, v in g["edges"]]
    dag = oracle.build_dag(len(idx), src, dst)
    nod = oracle.nod(dag, np.ones((len(idx), 1), np.float32), np.ones(1, np.int32))
    for t, v in g["nod_printed"].items():
        assert nod[idx[t], 0] == v
    assert nod[idx["T2"], 0] > nod[idx["T3"], 0]     # "Task 2 has a higher priority"


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_nod_against_fractions(seed):
    n = 400
    src, dst = random_dags.random_dag(n, 3.0, seed, dup=0.2)
    dur = random_dags.dyadic_durations(n, 3, seed, p_inf=0.3)
    dag = oracle.build_dag(n, src, dst)
    nod = oracle.nod(dag, dur, np.ones(3, np.int32))
    succ = {u: set() for u in range(n)}
    pred = {u: set() for u in range(n)}
    for u, v in zip(src.tolist(), dst.tolist()):
        succ[u].add(v)
        pred[v].add(u)
    for a in range(3):
        en = np.isfinite(dur[:, a])
        for t in range(n):
            if not en[t]:
                assert nod[t, a] == 0
                continue
            exact = sum((Fraction(1, sum(1 for p in pred[s] if en[p])) for s in succ[t] if en[s]), Fraction(0))
            tol = len(succ[t]) * 2.0 ** -32 + float(exact) * 2.0 ** -24
            assert abs(float(nod[t, a]) - float(exact)) <= tol


def test_nod_in_tree_is_reciprocal_indegree():
    # in-tree: every node has one successor, NOD(t) = 1/indeg(succ(t))
    rng = np.random.default_rng(5)
    n = 500
    parent = np.array([rng.integers(i + 1, n) for i in range(n - 1)])
    dag = oracle.build_dag(n, np.arange(n - 1), parent)
    nod = oracle.nod(dag, np.ones((n, 1), np.float32), np.ones(1, np.int32))
    indeg = np.bincount(parent, minlength=n)
    for t in range(n - 1):
        want = np.float32(1.0) / np.float32(indeg[parent[t]])
        assert abs(nod[t, 0] - want) <= np.spacing(want)
    assert nod[n - 1, 0] == 0


def _rn32(q: Fraction) -> np.float32:
    """Correctly rounded binary32 of an exact rational (ties to even)."""
    f = np.float32(float(q))
    cands = [np.nextafter(f, np.float32(-np.inf)), f, np.nextafter(f, np.float32(np.inf))]
    best = min(cands, key=lambda c: (abs(Fraction(float(c)) - q), int(np.float32(c).view(np.uint32)) & 1))
    return np.float32(best)


def test_nod_crit_norm_fig3_two_archs_hand_worked():
    """a7 with MP_CRIT_NOD: "All values are normalized between 0 and 1" (P:l.166)
    applied to eq. 2 (P:l.193), reading c9 = divide NOD_a by its max over the
    tasks enabled on a -- per arch, not one global max.  Fig. 3's DAG with T3
    unable to run on arch 1; values worked by hand from eq. 2 with the c10
    filter:
      arch 0 (all enabled): NOD = T1 2, T2 2.5, T3 1, T5 1/2 (T7's preds T3, T5),
        others 0; max 2.5  -> crit_n 0.8, 1, 0.4, 0, 0.2, 0, 0
      arch 1 (T3 off): T1 -> {T2} (indeg_1 1) = 1; T2 -> T4, T5, T6 (T6's
        arch-1 preds {T2}) = 3; T5 -> T7 (arch-1 preds {T5}) = 1; max 3
        -> crit_n 1/3, 1, 0, 0, 1/3, 0, 0
    A global max (3) would give T2 on arch 0 2.5/3, not 1."""
    g = load("fig3_nod.json")
    idx = {t: i for i, t in enumerate(g["tasks"])}
    src = [idx[u] for u, v in g["edges"]]
    dst = [idx[v] for u, v in g["edges"]]
    dag = oracle.build_dag(len(idx), src, dst)
    dur = np.ones((7, 2), np.float32)
    dur[idx["T3"], 1] = np.inf
    w = np.ones(2, np.int32)
    nod = oracle.nod(dag, dur, w)
    want_nod = [[2, 2.5, 1, 0, 0.5, 0, 0], [1, 3, 0, 0, 1, 0, 0]]
    assert nod.T.tolist() == want_nod
    _, _, flags = oracle.affinity(dur, w)
    gain = np.full((7, 2), 0.5, np.float32)
    cn, key = oracle.score(oracle.CRIT_NOD, nod, gain, flags)
    want = [[Fraction(4, 5), 1, Fraction(2, 5), 0, Fraction(1, 5), 0, 0],
            [Fraction(1, 3), 1, 0, 0, Fraction(1, 3), 0, 0]]
    for a in range(2):
        assert [float(x) for x in cn[:, a]] == [float(_rn32(Fraction(q))) for q in want[a]]
    assert key[idx["T3"], 1] == np.iinfo(np.uint64).max      # not enabled: no queue entry


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_nod_crit_norm_three_archs_masked_against_fractions(seed):
    """crit_n(t,a) = NOD_a(t) / max over enabled t' of NOD_a(t') (P:l.166,
    P:l.193, reading c9), checked against exact Fractions computed here from
    the edge list (not the oracle's NOD): 3 archs, arch 2 enabled on a small
    subset so the per-arch maxima differ and any other normaliser (global max,
    max over all tasks, sum) fails."""
    n = 300
    rng = np.random.default_rng(40 + seed)
    src, dst = random_dags.random_dag(n, 3.0, 40 + seed, dup=0.1)
    dur = random_dags.dyadic_durations(n, 3, 40 + seed, p_inf=0.0)
    dur[rng.random(n) < 0.3, 1] = np.inf
    dur[rng.random(n) < 0.8, 2] = np.inf
    w = np.ones(3, np.int32)
    dag = oracle.build_dag(n, src, dst)
    succ = {u: set() for u in range(n)}
    pred = {u: set() for u in range(n)}
    for u, v in zip(src.tolist(), dst.tolist()):
        succ[u].add(v)
        pred[v].add(u)
    nod = oracle.nod(dag, dur, w)
    _, _, flags = oracle.affinity(dur, w)
    gain = np.full((n, 3), 0.5, np.float32)
    cn, _ = oracle.score(oracle.CRIT_NOD, nod, gain, flags)
    maxima = []
    for a in range(3):
        en = np.isfinite(dur[:, a])
        exact = {t: sum((Fraction(1, sum(1 for p in pred[s] if en[p])) for s in succ[t] if en[s]), Fraction(0))
                 for t in range(n) if en[t]}
        mx = max(exact.values())
        maxima.append(mx)
        assert mx > 0
        for t in range(n):
            if not en[t]:
                assert cn[t, a] == 0
                continue
            q = exact[t] / mx
            # NOD_a is within outdeg 2^-32 + 2^-24 rel of exact (c11), then one RN division
            tol = float(q) * 2.0 ** -21 + len(succ[t]) * 2.0 ** -32 / float(mx)
            assert abs(float(cn[t, a]) - float(q)) <= tol, (t, a)
        # the maximisers get exactly 1
        arg = [t for t in exact if exact[t] == mx]
        assert all(cn[t, a] == 1.0 for t in arg)
        assert 0.0 <= cn[:, a].min() and cn[:, a].max() == 1.0
    assert len(set(maxima)) == 3             # per-arch maxima differ: the normaliser is visible


# ----------------------------------------------------------------------------
# a1/a2 DAG + levels: networkx, closed forms, invariants
# ----------------------------------------------------------------------------

def _nx_graph(n, src, dst):
    G = nx.DiGraph()
    G.add_nodes_from(range(n))
    G.add_edges_from(zip(np.asarray(src).tolist(), np.asarray(dst).tolist()))
    return G


@pytest.mark.parametrize("seed", range(4))
def test_levels_equal_networkx_generations(seed):
    n = 300
    src, dst = random_dags.random_dag(n, 2.5, seed, dup=0.3, max_span=20)
    dag = oracle.build_dag(n, src, dst)
    G = _nx_graph(n, src, dst)
    gens = [sorted(g) for g in nx.topological_generations(G)]
    assert dag.n_levels == len(gens)
    for l, g in enumerate(gens):
        assert dag.level_order[dag.level_ptr[l]:dag.level_ptr[l + 1]].tolist() == g
    assert dag.n_edges == G.number_of_edges()
    # CSR = deduplicated successor sets, ascending
    for u in range(n):
        assert dag.col[dag.row_ptr[u]:dag.row_ptr[u + 1]].tolist() == sorted(G.successors(u))
        assert dag.indeg[u] == G.in_degree(u)
    # every edge goes to a strictly higher level
    assert np.all(dag.level[src] < dag.level[dst])


def test_cholesky_closed_forms():
    for N in range(1, 13):
        w = workloads.cholesky(N)
        dag = oracle.build_dag(w.n, w.src, w.dst)
        assert w.n == N + N * (N - 1) + math.comb(N, 3)
        assert dag.n_edges == (N - 1) * N * (N + 1) // 2
        assert dag.n_levels == 3 * N - 2
    w = workloads.cholesky(64)
    dag = oracle.build_dag(w.n, w.src, w.dst)
    assert (w.n, dag.n_edges, dag.n_levels) == (45760, 131040, 190)
    assert np.diff(dag.level_ptr).max() == math.comb(64, 2)


def test_qr_closed_forms():
    for N in (2, 3, 5, 8, 13):
        w = workloads.qr(N, split_diag=True)
        dag = oracle.build_dag(w.n, w.src, w.dst)
        assert w.n == N * (N + 1) * (2 * N + 1) // 6
        assert dag.n_edges == N * (N - 1) * (2 * N + 1) // 2
        assert dag.n_levels == 3 * N - 2
        s = dense.qr(N, split_diag=False)
        src, dst = s.edges()
        d2 = oracle.build_dag(s.n, src, dst)
        assert d2.n_edges == (N - 1) * N * (N + 1)
        assert d2.n_levels == 4 * N - 3
        assert d2.indeg.max() == N


# ----------------------------------------------------------------------------
# a4 bottom-level: brute-force path enumeration, networkx, closed forms
# ----------------------------------------------------------------------------

def _brute_bl(n, succ, w):
    """Longest path by exhaustive DFS over every path (tiny DAGs only)."""
    def paths_from(v):
        if not succ[v]:
            yield [v]
        for s in succ[v]:
            for p in paths_from(s):
                yield [v] + p
    return [max(sum(Fraction(w[x]) for x in p) for p in paths_from(v)) for v in range(n)]


@pytest.mark.parametrize("seed", range(30))
def test_bl_brute_force_tiny(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 13))
    src, dst = random_dags.random_dag(n, float(rng.uniform(0.5, 2.5)), seed, dup=0.2)
    A = int(rng.integers(1, 4))
    dur = random_dags.dyadic_durations(n, A, seed, p_inf=0.3 if A > 1 else 0.0)
    if seed % 5 == 0:
        dur[rng.random((n, A)) < 0.2] = 0.0
        dur[np.all(~np.isfinite(dur), 1)] = 1.0
    dag = oracle.build_dag(n, src, dst)
    bl, cp = oracle.bottom_level(dag, dur, np.ones(A, np.int32))
    w = [min(float(x) for x in dur[t] if np.isfinite(x)) for t in range(n)]
    succ = {u: sorted(set(dst[src == u].tolist())) for u in range(n)}
    want = _brute_bl(n, succ, w)
    assert [Fraction(float(x)) for x in bl] == want        # dyadic => exact, bit-exact
    assert Fraction(float(cp)) == max(want)


@pytest.mark.parametrize("seed", range(3))
def test_cp_equals_networkx_longest_path(seed):
    n = 2000
    src, dst = random_dags.random_dag(n, 3.0, seed, max_span=50)
    dur = random_dags.dyadic_durations(n, 2, seed)
    dag = oracle.build_dag(n, src, dst)
    bl, cp = oracle.bottom_level(dag, dur, np.ones(2, np.int32))
    w = dur.min(1).astype(np.float64)
    G = nx.DiGraph()
    for v in range(n):
        G.add_edge(("i", v), ("o", v), weight=w[v])
    for u, v in zip(src.tolist(), dst.tolist()):
        G.add_edge(("o", u), ("i", v), weight=0.0)
    assert nx.dag_longest_path_length(G) == float(cp)


def test_bl_chain_and_star():
    n = 50
    dur = random_dags.dyadic_durations(n, 1, 3)
    dag = oracle.build_dag(n, *random_dags.chain(n))
    bl, cp = oracle.bottom_level(dag, dur, np.ones(1, np.int32))
    w = dur[:, 0].astype(np.float64)
    assert [float(x) for x in bl] == [float(w[i:].sum()) for i in range(n)]
    dag = oracle.build_dag(n, *random_dags.star(n))
    bl, cp = oracle.bottom_level(dag, dur, np.ones(1, np.int32))
    assert cp == np.float32(w[0] + w[1:].max())


def _chol_cp_closed_form(N, p, t, s, g):
    if N == 1:
        return p
    return p + (N - 1) * t + (N - 2) * max(g, s + p) + s + p


def test_cholesky_cp_closed_form():
    rng = np.random.default_rng(11)
    for trial in range(60):
        N = int(rng.integers(1, 11))
        k = rng.integers(1, 256, 4) / 16.0   # dyadic
        p, t, s, g = (float(x) for x in k)
        w = workloads.cholesky(N)
        tab = np.array([p, t, s, g], np.float32)
        dur = tab[w.kind][:, None]
        dag = oracle.build_dag(w.n, w.src, w.dst)
        _, cp = oracle.bottom_level(dag, dur, np.ones(1, np.int32))
        assert float(cp) == _chol_cp_closed_form(N, p, t, s, g)
    # unit weights: 3N-2; the C1 / C2 models: 17.25 and 302.25
    for N, want in ((4, 17.25), (64, 302.25)):
        w = workloads.cholesky(N)
        dag = oracle.build_dag(w.n, w.src, w.dst)
        _, cp = oracle.bottom_level(dag, w.dur, w.workers)
        assert cp == want


# ----------------------------------------------------------------------------
# a7/a8/a9 score, queues, summaries
# ----------------------------------------------------------------------------

def test_c1_appendix_a_golden():
    g = load("c1_appendix_a.json")
    w = workloads.config("c1")
    dag = oracle.build_dag(w.n, w.src, w.dst)
    assert dag.level.tolist() == g["level"]
    for u, ss in g["successors"].items():
        assert dag.col[dag.row_ptr[int(u)]:dag.row_ptr[int(u) + 1]].tolist() == ss
    r = oracle.score_and_queue(dag, w.dur, w.workers)
    assert r["bl"].tolist() == g["bl"] and r["cp"] == g["cp"]
    assert np.all(np.abs(r["crit_norm"] - np.array(g["crit_n"])) < 5e-9)
    assert np.all(np.abs(r["gain"][:, 0] - np.array(g["gain_cpu"])) < 1e-7)
    assert np.all(np.abs(r["gain"][:, 1] - np.array(g["gain_gpu"])) < 1e-7)
    assert r["hd"].tolist() == g["hd"]
    nod = oracle.nod(dag, w.dur, w.workers)
    assert np.all(np.abs(nod[:, 0] - np.array(g["nod"])) < 1e-3)
    lab = g["labels"]
    q = r["qtask"].tolist()
    assert [lab[i] for i in q[:20]] == g["queue_cpu"]
    assert [lab[i] for i in q[20:]] == g["queue_gpu"]
    s = r["summary"]
    assert s["brw"].tolist() == g["best_remaining_work"]
    assert s["count"].tolist() == g["count"]
    assert [lab[i] for i in s["head"]] == g["head"]


def _check_queue(qtask, qptr, gain, critn, flags, kind, ready=None):
    n, A = gain.shape
    for a in range(A):
        q = qtask[qptr[a]:qptr[a + 1]].tolist()
        members = [t for t in range(n) if flags[t, a] & 1 and (ready is None or ready[t])]
        c = critn if kind == oracle.CRIT_BL else critn[:, a]
        # lexicographic (gain desc, crit desc) with id ascending (P:l.138, reading c12),
        # computed by Python's sort on the float32 values -- independent of the key packing
        want = sorted(members, key=lambda t: (-float(gain[t, a]), -float(c[t]), t))
        assert q == want
        # a non-increasing array is a valid binary max-heap
        for i in range(len(q)):
            for ch in (2 * i + 1, 2 * i + 2):
                if ch < len(q):
                    assert (gain[q[i], a], c[q[i]]) >= (gain[q[ch], a], c[q[ch]])


@pytest.mark.parametrize("A,kind,seed", [(1, 0, 0), (2, 0, 1), (3, 0, 2), (2, 1, 3), (3, 1, 4), (2, 0, 5)])
def test_queues_sorted_membership_and_duplication(A, kind, seed):
    n = 600
    src, dst = random_dags.random_dag(n, 2.0, seed, dup=0.1, max_span=40)
    dur = random_dags.dyadic_durations(n, A, seed, p_inf=0.25, tiny_set=(seed % 2 == 1))
    dag = oracle.build_dag(n, src, dst)
    r = oracle.score_and_queue(dag, dur, np.ones(A, np.int32), kind=kind)
    _check_queue(r["qtask"], r["qptr"], r["gain"], r["crit_norm"], r["flags"], kind)
    # a task is duplicated into every queue whose arch can run it (P:l.104)
    for t in range(n):
        cnt = sum(int(t in r["qtask"][r["qptr"][a]:r["qptr"][a + 1]]) for a in range(A))
        assert cnt == int(np.isfinite(dur[t]).sum())
    if A == 1:  # pure critical-path list (HLFET): lexsort by (-crit_n, id)
        assert r["qtask"].tolist() == np.lexsort((np.arange(n), -r["crit_norm"].astype(np.float64))).tolist()
    if kind == 0:
        assert r["crit_norm"].max() == 1.0 and r["crit_norm"][np.argmax(r["bl"])] == 1.0


def test_ready_mode_membership():
    n = 500
    src, dst = random_dags.random_dag(n, 2.0, 7, max_span=30)
    dur = random_dags.dyadic_durations(n, 2, 7)
    dag = oracle.build_dag(n, src, dst)
    r = oracle.score_and_queue(dag, dur, np.ones(2, np.int32))
    rng = np.random.default_rng(7)
    # done = a down-closed set: the first k tasks of a topological order
    done = np.zeros(n, np.uint8)
    done[dag.level_order[: n // 3]] = 1
    done[rng.integers(0, n, 5)] = 1          # plus some arbitrary ones
    qptr, qtask, summ = oracle.build_queues(dag, r["key"], r["flags"], dur, done)
    ready = np.array([not done[t] and all(done[u] for u in src[dst == t]) for t in range(n)])
    _check_queue(qtask, qptr, r["gain"], r["crit_norm"], r["flags"], 0, ready=ready)
    assert summ["count"].tolist() == [int(ready.sum())] * 2


def test_best_remaining_work_exact():
    n = 3000
    rng = np.random.default_rng(3)
    # arbitrary binary32 durations over many binades, incl. the domain edges
    dur = (2.0 ** rng.uniform(-41, 19.9, (n, 2))).astype(np.float32)
    dur[0, 0] = np.float32(2.0 ** -41)
    dur[1, 1] = np.nextafter(np.float32(2.0 ** 20), np.float32(0))
    dur[2] = 0.0
    dag = oracle.build_dag(n, [], [])
    r = oracle.score_and_queue(dag, dur, np.ones(2, np.int32))
    for a in range(2):
        best = (r["flags"][:, a] & 2) > 0
        exact = sum((Fraction(float(x)) for x in dur[best, a]), Fraction(0))
        iv = exact * 2 ** 64
        assert iv.denominator == 1
        iv = iv.numerator
        s = r["summary"][a]
        assert int(s["brw_lo"]) == iv & (2 ** 64 - 1) and int(s["brw_hi"]) == iv >> 64
        assert float(s["brw"]) == float(exact)       # exact sum rounded once (float(Fraction) is RN)


def test_score_key_packing_order():
    """key ascending <=> (gain desc, crit desc) on every pair of random float32 values in [0,1]."""
    rng = np.random.default_rng(0)
    g = np.concatenate([rng.random(200), [0.0, 1.0, 0.5]]).astype(np.float32)
    c = np.concatenate([rng.random(200), [0.0, 1.0, 1.0]]).astype(np.float32)
    n = len(g)
    flags = np.ones((n, 1), np.uint8)
    cn, key = oracle.score(oracle.CRIT_BL, c, g[:, None], flags)
    assert np.all(cn == c / c.max())
    for i, j in itertools.combinations(range(n), 2):
        lt = (-g[i], -cn[i]) < (-g[j], -cn[j])
        gt = (-g[i], -cn[i]) > (-g[j], -cn[j])
        assert (key[i, 0] < key[j, 0]) == lt and (key[i, 0] > key[j, 0]) == gt


# ----------------------------------------------------------------------------
# a10 replicas
# ----------------------------------------------------------------------------

def test_splitmix64_reference_vector():
    # splitmix64 with state 0: first output 0xE220A8397B1DCDAF (Vigna's reference
    # sequence); or_perturb(r=0,t=0,a=0) uses counter 1 = that first output.
    u24 = 0xE220A8397B1DCDAF >> 40
    u = u24 * 2.0 ** -24
    f = np.float32(1) + np.float32(0.125) * (np.float32(2 * u) - np.float32(1))
    out = oracle.perturb(np.array([[8.0]], np.float32), 0, 0.125, 0)
    assert out[0, 0] == np.float32(8.0) * f


def test_perturb_range_and_sigma_zero_identity():
    w = workloads.config("c1")
    base = w.dur
    p = oracle.perturb(base, 123, 0.125, 7)
    ratio = p / base
    assert np.all((ratio >= 0.875 - 1e-6) & (ratio <= 1.125 + 1e-6))
    assert not np.all(p == base)
    dag = oracle.build_dag(w.n, w.src, w.dst)
    cp, summ, q, qptr = oracle.replica(dag, base, w.workers, 5, 0.0, 3)
    r = oracle.score_and_queue(dag, base, w.workers)
    assert cp == r["cp"] and q.tolist() == r["qtask"].tolist()
    assert summ.tobytes() == r["summary"].tobytes()


def test_replica_equals_stepwise_path():
    w = workloads.config("c1")
    dag = oracle.build_dag(w.n, w.src, w.dst)
    for r_id in (0, 1, 4095):
        d = oracle.perturb(w.dur, workloads.C5_SEED, workloads.C5_SIGMA, r_id)
        r = oracle.score_and_queue(dag, d, w.workers)
        cp, summ, q, _ = oracle.replica(dag, w.dur, w.workers, workloads.C5_SEED, workloads.C5_SIGMA, r_id)
        assert cp == r["cp"] and q.tolist() == r["qtask"].tolist()
        assert summ.tobytes() == r["summary"].tobytes()


# ----------------------------------------------------------------------------
# error paths (reading c20)
# ----------------------------------------------------------------------------

def test_error_paths():
    with pytest.raises(oracle.OracleError) as e:
        oracle.build_dag(3, [0], [0])
    assert e.value.code == oracle.ERR_ARG
    with pytest.raises(oracle.OracleError) as e:
        oracle.build_dag(3, [0], [3])
    assert e.value.code == oracle.ERR_ARG
    with pytest.raises(oracle.OracleError) as e:
        oracle.build_dag(3, [0, 1, 2], [1, 2, 0])
    assert e.value.code == oracle.ERR_CYCLE
    dag = oracle.build_dag(2, [0], [1])
    for bad in ([np.nan, 1], [-1, 1], [2.0 ** -42, 1], [2.0 ** 20, 1], [np.inf, np.inf], [-np.inf, 1]):
        dur = np.array([bad, [1, 1]], np.float32)
        with pytest.raises(oracle.OracleError) as e:
            oracle.bottom_level(dag, dur, np.ones(2, np.int32))
        assert e.value.code == oracle.ERR_DOMAIN
    # -0 is canonicalised to +0 and accepted
    bl, cp = oracle.bottom_level(dag, np.array([[-0.0, np.inf], [1, 1]], np.float32), np.ones(2, np.int32))
    assert bl.tolist() == [1.0, 1.0] and np.signbit(bl).sum() == 0
    # n = 0, E = 0
    d0 = oracle.build_dag(0, [], [])
    assert d0.n_levels == 0 and d0.n_edges == 0
    d1 = oracle.build_dag(5, [], [])
    assert d1.n_levels == 1


def test_oracle_replicas_thread_safe():
    """The GPU parity test and the cpu baseline run oracle.replica from threads: the
    results must equal the sequential ones (no shared mutable state in the oracle)."""
    from concurrent.futures import ThreadPoolExecutor
    w = workloads.config("c2")
    od = oracle.build_dag(w.n, w.src, w.dst)
    args = (workloads.C5_SEED, workloads.C5_SIGMA)
    seq = [oracle.replica(od, w.dur, w.workers, *args, r) for r in range(16)]
    with ThreadPoolExecutor(8) as ex:
        par = list(ex.map(lambda r: oracle.replica(od, w.dur, w.workers, *args, r), range(16)))
    for a, b in zip(seq, par):
        assert a[0] == b[0] and a[1].tobytes() == b[1].tobytes() and np.array_equal(a[2], b[2])
