"""Pins of the N4 variant oracles against things other than
themselves (-m "not gpu"):

* v1 mean-cost node weight (HEFT's average over processors): exact Fraction
  longest paths on dyadic durations, the one-arch special case (= min).
* v2 hd(a) "recorded so far" (P:l.176) as a running max along the push order:
  Table II's printed gains in the paper's order tA, tB, tC (P:l.180-187), a
  hand-worked other order, final hd = whole-set hd, max-first orders = the
  static gains.
* v3 NOD on the remaining graph: Fig. 3's dynamic scenario (T1 completed, T2
  and T3 ready, P:l.195-198), Fractions on random DAGs with completed
  prefixes, done = nothing -> the static NOD.
"""
from __future__ import annotations

import json
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
from workloads import random_dags

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def load(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def _sets(n, src, dst):
    succ = {u: set() for u in range(n)}
    pred = {u: set() for u in range(n)}
    for u, v in zip(np.asarray(src).tolist(), np.asarray(dst).tolist()):
        succ[u].add(v)
        pred[v].add(u)
    return succ, pred


# ---------------------------------------------------------------- v1 mean cost

@pytest.mark.parametrize("seed", range(5))
def test_mean_weight_exact_longest_path(seed):
    n = 60
    A = 2
    src, dst = random_dags.random_dag(n, 2.0, seed)
    dag = oracle.build_dag(n, src, dst)
    dur = random_dags.dyadic_durations(n, A, seed, denom=8, hi=32)
    # worker totals 2, 4 or 8: every mean is dyadic, so every w and bl is exact
    workers = np.array([(1, 1), (1, 3), (3, 1), (2, 2), (3, 5)][seed], np.int32)
    bl, cp = oracle.bottom_level_w(dag, dur, workers, oracle.WEIGHT_MEAN)
    succ, _ = _sets(n, src, dst)
    w = []
    for t in range(n):
        num = sum(Fraction(int(workers[a])) * Fraction(float(dur[t, a])) for a in range(A) if np.isfinite(dur[t, a]))
        den = sum(int(workers[a]) for a in range(A) if np.isfinite(dur[t, a]))
        w.append(num / den)
    memo = {}

    def exact_bl(v):
        if v not in memo:
            memo[v] = w[v] + max((exact_bl(s) for s in succ[v]), default=Fraction(0))
        return memo[v]

    for t in range(n):
        e = exact_bl(t)
        if e.denominator & (e.denominator - 1) == 0 and abs(e.numerator) < 2 ** 24 * e.denominator:
            assert Fraction(float(bl[t])) == e          # representable: exact
    assert cp == max(bl)


def test_mean_weight_one_arch_is_min_and_bounds():
    n = 80
    src, dst = random_dags.random_dag(n, 2.5, 3)
    dag = oracle.build_dag(n, src, dst)
    d1 = random_dags.dyadic_durations(n, 1, 3)
    assert np.array_equal(oracle.bottom_level_w(dag, d1, [3], 1)[0], oracle.bottom_level(dag, d1, [3])[0])
    d2 = random_dags.dyadic_durations(n, 2, 3, p_inf=0.2)
    bmin = oracle.bottom_level(dag, d2, [2, 2])[0]
    bmean = oracle.bottom_level_w(dag, d2, [2, 2], 1)[0]
    assert np.all(bmean >= bmin)
    # equal worker counts, every arch enabled: w = (d0 + d1) / 2
    d3 = random_dags.dyadic_durations(n, 2, 4)
    chain_s, chain_d = random_dags.chain(n)
    cd = oracle.build_dag(n, chain_s, chain_d)
    bl = oracle.bottom_level_w(cd, d3, [5, 5], 1)[0]
    tail = np.cumsum(((d3[:, 0].astype(np.float64) + d3[:, 1]) / 2)[::-1])[::-1]
    assert np.array_equal(bl.astype(np.float64), tail)


# ---------------------------------------------------------------- v2 prefix hd

def test_prefix_hd_table2_in_push_order():
    """Pushed in the paper's order tA, tB, tC the running max is 19 from the
    first task on, so the printed Table II gains hold (P:l.180-187)."""
    g = load("table2_gain.json")
    dur = np.array(g["dur_ms"], np.float32)
    gain, hd, flags = oracle.affinity_prefix(dur, [1, 1], [0, 1, 2])
    printed = np.array(g["gain_printed"])
    assert np.all(np.floor(gain.astype(np.float64) * 1000 + 1e-9) / 1000 == printed)
    assert hd.tolist() == g["hd"]


def test_prefix_hd_other_order_hand_worked():
    """Order tB, tA, tC: when tB is pushed hd = |10 - 5| = 5, so
    gain(tB, a1) = (5 + 5) / 10 = 1 and gain(tB, a2) = (-5 + 5) / 10 = 0; tA and
    tC then see hd = 19 (Table II values)."""
    g = load("table2_gain.json")
    dur = np.array(g["dur_ms"], np.float32)
    gain, hd, _ = oracle.affinity_prefix(dur, [1, 1], [1, 0, 2])
    assert gain[1].tolist() == [1.0, 0.0]
    s_gain, _, _ = oracle.affinity(dur, [1, 1])
    assert np.array_equal(gain[[0, 2]], s_gain[[0, 2]])
    assert hd.tolist() == [19.0, 19.0]


@pytest.mark.parametrize("seed", range(4))
def test_prefix_hd_final_and_max_first(seed):
    n = 300
    dur = random_dags.dyadic_durations(n, 2, seed, p_inf=0.2)
    s_gain, s_hd, s_flags = oracle.affinity(dur, [1, 1])
    rng = np.random.default_rng(seed)
    order = rng.permutation(n).astype(np.int32)
    gain, hd, flags = oracle.affinity_prefix(dur, [1, 1], order)
    assert np.array_equal(hd, s_hd) and np.array_equal(flags, s_flags)
    assert np.all((gain >= 0) & (gain <= 1))
    # the task with the largest |d| first: every prefix max is already hd
    absd = np.where(np.isfinite(dur).all(1), np.abs(dur[:, 1] - dur[:, 0]), -1)
    first = int(np.argmax(absd))
    order2 = np.concatenate([[first], np.delete(np.arange(n), first)]).astype(np.int32)
    gain2, _, _ = oracle.affinity_prefix(dur, [1, 1], order2)
    assert np.array_equal(gain2, s_gain)
    # the first pushed two-arch task has d = +-hd or hd = 0: gain in {0, 0.5, 1}
    t0 = int(order[0])
    if np.isfinite(dur[t0]).all():
        assert set(gain[t0].tolist()) <= {0.0, 0.5, 1.0}


# ---------------------------------------------------------------- v3 remaining NOD

def test_fig3_dynamic_scenario():
    """Fig. 3 (P:l.195-198): T1 completed, T2 and T3 ready: NOD(T2) = 2.5, NOD(T3) = 1."""
    g = load("fig3_nod.json")
    idx = {t: i for i, t in enumerate(g["tasks"])}
    src = [idx[u] for u, v in g["edges"]]
    dst = [idx[v] for u, v in g["edges"]]
    dag = oracle.build_dag(len(idx), src, dst)
    done = np.zeros(len(idx), np.uint8)
    done[idx["T1"]] = 1
    nod = oracle.nod_remaining(dag, np.ones((len(idx), 1), np.float32), [1], done)
    for t, v in g["nod_printed"].items():
        assert nod[idx[t], 0] == v
    assert nod[idx["T1"], 0] == 0


@pytest.mark.parametrize("seed", range(3))
def test_nod_remaining_against_fractions(seed):
    n = 300
    src, dst = random_dags.random_dag(n, 3.0, seed, dup=0.2)
    dur = random_dags.dyadic_durations(n, 2, seed, p_inf=0.3)
    dag = oracle.build_dag(n, src, dst)
    succ, pred = _sets(n, src, dst)
    done = np.zeros(n, np.uint8)
    done[dag.level_order[: n // 3]] = 1          # a completed prefix of a topological order
    nod = oracle.nod_remaining(dag, dur, [1, 1], done)
    for a in range(2):
        en = np.isfinite(dur[:, a])
        for t in range(n):
            if not en[t] or done[t]:
                assert nod[t, a] == 0
                continue
            exact = sum((Fraction(1, sum(1 for p in pred[s] if en[p] and not done[p]))
                         for s in succ[t] if en[s] and not done[s]), Fraction(0))
            tol = len(succ[t]) * 2.0 ** -32 + float(exact) * 2.0 ** -24
            assert abs(float(nod[t, a]) - float(exact)) <= tol
    assert np.array_equal(oracle.nod_remaining(dag, dur, [1, 1], np.zeros(n, np.uint8)),
                          oracle.nod(dag, dur, [1, 1]))


# ---------------------------------------------------------------- hierarchical tasks (P:l.318)

def _chol_counts(M):
    """Closed forms of the M x M tiled Cholesky (SURVEY §8(c) a1/a2 pins)."""
    from math import comb
    return M + M * (M - 1) + comb(M, 3), (M - 1) * M * (M + 1) // 2, 3 * M - 2


@pytest.mark.parametrize("N,s", [(3, 2), (5, 2), (4, 3)])
def test_hier_extremes_are_the_plain_tilings(N, s):
    """Hierarchical tasks (reading h1): expanding no task gives the N x N tiled Cholesky,
    expanding every task the (N s) x (N s) one -- n, E, depth from the closed forms, and
    (small case) the same DAG up to relabelling, kernel kinds matched."""
    import networkx as nx
    from workloads import dense
    for p, M in ((0.0, N), (1.0, N * s)):
        rec = dense.hier_cholesky(N, s, p)
        src, dst = rec.edges()
        dag = oracle.build_dag(rec.n, src, dst)
        assert (dag.n, dag.n_edges, dag.n_levels) == _chol_counts(M)
    if N * s <= 8:
        def graph(rec, fine):
            src, dst = rec.edges()
            G = nx.DiGraph()
            for t, kd in enumerate(rec.kinds().tolist()):
                G.add_node(t, kind=kd - 4 if fine else kd)
            G.add_edges_from(zip(src.tolist(), dst.tolist()))
            return G
        Gh = graph(dense.hier_cholesky(N, s, 1.0), True)
        Gf = graph(dense.cholesky(N * s), False)
        assert nx.is_isomorphic(Gh, Gf, node_match=lambda x, y: x["kind"] == y["kind"])


def test_hier_full_expansion_cp_closed_form():
    """Every task expanded: the DAG is the (N s)-tile Cholesky with the fine-task weights,
    so CP = p + (M-1) t + (M-2) max(g, s+p) + s + p (SURVEY §8(c) a4, M = N s) with
    w = min(CPU, GPU) of HIER_MODEL's fine kernels (dyadic: exact in binary32)."""
    import workloads
    from workloads import dense
    N, s = 6, 2
    w = workloads.hier(N, s, 1.0)
    assert set(np.unique(w.kind).tolist()) == {dense.POTRF_F, dense.TRSM_F, dense.SYRK_F, dense.GEMM_F}
    mn = {k: min(v) for k, v in workloads.HIER_MODEL.items()}
    P, T, S, G = mn[dense.POTRF_F], mn[dense.TRSM_F], mn[dense.SYRK_F], mn[dense.GEMM_F]
    M = N * s
    dag = oracle.build_dag(w.n, w.src, w.dst)
    bl, cp = oracle.bottom_level(dag, w.dur, w.workers)
    assert float(cp) == P + (M - 1) * T + (M - 2) * max(G, S + P) + S + P


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_hier_partial_levels_and_cp_against_networkx(seed):
    """Partly expanded DAGs (mixed granularity): levels = networkx generations, CP = the
    networkx longest path with w = min over archs (dyadic weights: exact)."""
    import networkx as nx
    import workloads
    w = workloads.hier(6, 2, 0.5, seed)
    assert 0 < int((w.kind >= 4).sum()) < w.n          # both granularities present
    dag = oracle.build_dag(w.n, w.src, w.dst)
    G = nx.DiGraph()
    G.add_nodes_from(range(w.n))
    G.add_edges_from(zip(w.src.tolist(), w.dst.tolist()))
    gens = list(nx.topological_generations(G))
    assert dag.n_levels == len(gens)
    for lv, g in enumerate(gens):
        assert sorted(g) == sorted(np.where(dag.level == lv)[0].tolist())
    wt = w.dur.min(axis=1)
    for v in G:
        G.nodes[v]["w"] = float(wt[v])
    longest = {}
    for v in reversed(list(nx.topological_sort(G))):
        longest[v] = G.nodes[v]["w"] + max((longest[u] for u in G.successors(v)), default=0.0)
    bl, cp = oracle.bottom_level(dag, w.dur, w.workers)
    assert float(cp) == max(longest.values())
    assert all(float(bl[v]) == longest[v] for v in G)
