"""Pins of the N2 simulation oracle (oracle/mp_sim_oracle.c) against things
other than itself (-m "not gpu").

* Hand-worked PUSH/POP schedules (tests/golden/sim_worked.json; Alg. 1
  P:l.133-136, Alg. 2 P:l.140-160, pop_condition P:l.214-220).
* Closed forms of list scheduling: unbounded workers -> makespan = critical
  path (brute-force longest path); one worker -> makespan = sum of durations.
* Graham's list-scheduling bounds for one arch, the lower bounds for several.
* Trace invariants: exactly once, enabled arch, precedence, no overlap per
  worker, busy/ran totals, and -- without eviction -- work conservation and
  highest-priority-first pops (the heap order of a8, checked from the keys).
* Fig. 4's direction (P:l.222-229): the eviction mechanism removes most of the
  GPU idle time on a tiled Cholesky with 1 GPU and 16 CPUs.
"""
from __future__ import annotations

import json
import os

import numpy as np
import pytest

import oracle
import workloads
from workloads import random_dags

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _dag(n, edges):
    e = np.asarray(edges, np.int32).reshape(-1, 2)
    return oracle.build_dag(n, e[:, 0], e[:, 1])


def _succ(dag):
    return [dag.col[dag.row_ptr[t]:dag.row_ptr[t + 1]].tolist() for t in range(dag.n)]


def _preds(dag):
    p = [[] for _ in range(dag.n)]
    for u, ss in enumerate(_succ(dag)):
        for v in ss:
            p[v].append(u)
    return p


def _longest_path(dag, w):
    """Brute-force DP over a topological order (textbook longest path)."""
    order = list(dag.level_order)
    best = np.zeros(dag.n)
    for v in reversed(order):
        ss = dag.col[dag.row_ptr[v]:dag.row_ptr[v + 1]]
        best[v] = float(w[v]) + (max(best[s] for s in ss) if len(ss) else 0.0)
    return best.max() if dag.n else 0.0


@pytest.mark.parametrize("case", json.load(open(os.path.join(GOLD, "sim_worked.json")))["cases"],
                         ids=lambda c: c["name"])
def test_hand_worked_schedules(case):
    dur = np.array(case["dur_ms"], np.float32)
    dag = _dag(len(dur), case["edges"])
    st, start, worker = oracle.simulate_dag(dag, dur, case["workers"], case["max_tries"], case["eviction"])
    assert start.tolist() == case["start"]
    assert worker.tolist() == case["worker"]
    assert st["makespan"] == case["makespan"]
    assert (st["evictions"], st["dups"], st["rounds"]) == (case["evictions"], case["dups"], case["rounds"])
    assert st["stale"] == case["stale"]          # lazy removals, hand-derived (P:l.130)
    assert st["busy"][:2].tolist() == case["busy"] and st["ran"][:2].tolist() == case["ran"]
    assert st["pops"] == len(dur)


@pytest.mark.parametrize("seed", range(6))
def test_unbounded_workers_reach_critical_path(seed):
    """With at least n workers of one arch every task starts when ready, so
    the makespan is the longest path (dyadic durations: exact)."""
    n = 40
    src, dst = random_dags.random_dag(n, 2.0, seed, dup=0.2)
    dag = oracle.build_dag(n, src, dst)
    dur = random_dags.dyadic_durations(n, 1, seed)
    st, start, _ = oracle.simulate_dag(dag, dur, [n], eviction=bool(seed % 2))
    assert st["makespan"] == _longest_path(dag, dur[:, 0])
    # and each task starts exactly when its last predecessor finishes
    fin = start + dur[:, 0].astype(np.float64)
    for v, ps in enumerate(_preds(dag)):
        assert start[v] == (max(fin[p] for p in ps) if ps else 0.0)


@pytest.mark.parametrize("seed", range(4))
def test_one_worker_makespan_is_total_work(seed):
    n = 30
    src, dst = random_dags.random_dag(n, 1.5, seed)
    dag = oracle.build_dag(n, src, dst)
    dur = random_dags.dyadic_durations(n, 2, seed, p_inf=0.3)
    # arch 1 has no worker: only arch 0 runs; tasks that cannot run on arch 0
    # get a finite arch-0 duration so the instance is valid
    dur[:, 0] = np.where(np.isinf(dur[:, 0]), 1.0, dur[:, 0])
    st, _, worker = oracle.simulate_dag(dag, dur, [1, 0])
    assert st["makespan"] == float(dur[:, 0].astype(np.float64).sum())
    assert np.all(worker == 0)


@pytest.mark.parametrize("seed", range(8))
def test_list_scheduling_bounds_one_arch(seed):
    """Graham: max(CP, S/W) <= makespan <= S/W + (1 - 1/W) CP for a greedy
    list schedule on W identical workers (no eviction on one arch)."""
    rng = np.random.default_rng(seed)
    n = int(rng.integers(20, 80))
    W = int(rng.integers(1, 6))
    src, dst = random_dags.random_dag(n, float(rng.uniform(0.5, 3)), seed)
    dag = oracle.build_dag(n, src, dst)
    dur = random_dags.dyadic_durations(n, 1, seed)
    st, _, _ = oracle.simulate_dag(dag, dur, [W])
    S = float(dur.astype(np.float64).sum())
    cp = _longest_path(dag, dur[:, 0])
    assert max(cp, S / W) <= st["makespan"] + 1e-9
    assert st["makespan"] <= S / W + (1 - 1 / W) * cp + 1e-9


def _check_trace(dag, dur, workers, st, start, worker):
    n, A = dur.shape
    wa = np.repeat(np.arange(A), workers)
    arch = wa[worker]
    d = dur[np.arange(n), arch].astype(np.float64)
    fin = start + d
    assert np.all(np.isfinite(d))                          # ran on an enabled arch
    assert np.all(np.asarray(workers)[arch] > 0)
    for v, ps in enumerate(_preds(dag)):                    # precedence (P:l.89)
        for p in ps:
            assert start[v] >= fin[p]
    for w in range(len(wa)):                                # one task at a time
        idx = np.where(worker == w)[0]
        o = idx[np.argsort(start[idx], kind="stable")]
        assert np.all(start[o][1:] >= fin[o][:-1])
    assert st["pops"] == n and st["makespan"] == (fin.max() if n else 0.0)
    for a in range(A):
        assert st["ran"][a] == int((arch == a).sum())
        assert st["busy"][a] == float(d[arch == a].sum())    # dyadic: exact
    ent = int(sum(np.sum(~np.isinf(dur[:, a])) for a in range(A) if workers[a] > 0))
    assert st["pops"] + st["evictions"] + st["dups"] <= ent
    # every duplicate a pop leaves is later met at its heap's root and dropped
    # (P:l.130): the final dispatch, with every worker idle, drains every heap
    # of an arch that has workers, so lazy removals == duplicates left (s5)
    assert st["stale"] == st["dups"]
    return arch, fin


@pytest.mark.parametrize("seed", range(10))
def test_trace_invariants_random(seed):
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(10, 120))
    A = int(rng.integers(1, 4))
    src, dst = random_dags.random_dag(n, float(rng.uniform(0.5, 3)), seed, dup=0.1)
    dag = oracle.build_dag(n, src, dst)
    dur = random_dags.dyadic_durations(n, A, seed, p_inf=0.25, tiny_set=bool(seed % 3 == 0))
    workers = rng.integers(1, 4, A).astype(np.int32)
    ev = bool(seed % 2)
    st, start, worker = oracle.simulate_dag(dag, dur, workers, int(rng.integers(1, 5)), ev)
    _check_trace(dag, dur, workers, st, start, worker)
    if not ev:
        assert st["evictions"] == 0 and st["rounds"] == 0


@pytest.mark.parametrize("seed", range(8))
def test_no_eviction_greedy_and_priority_order(seed):
    """Without eviction each idle worker pops the highest-priority ready task
    of its arch's heap (key asc, id asc; a8) at every event time, workers
    arch-major in id order (s2): so at each event time T the tasks started on
    arch a are the top-k_a of the ready, not-yet-started tasks enabled on a
    (minus those taken by lower archs at T), and no worker of arch a stays
    idle while such a task is left (work conservation)."""
    rng = np.random.default_rng(200 + seed)
    n = int(rng.integers(20, 100))
    A = 1 + seed % 2
    src, dst = random_dags.random_dag(n, float(rng.uniform(0.5, 2.5)), seed)
    dag = oracle.build_dag(n, src, dst)
    dur = random_dags.dyadic_durations(n, A, seed, p_inf=0.3, tiny_set=bool(seed % 4 == 1))
    workers = rng.integers(1, 4, A).astype(np.int32)
    st, start, worker = oracle.simulate_dag(dag, dur, workers, 4, eviction=False)
    arch, fin = _check_trace(dag, dur, workers, st, start, worker)
    # without eviction every task sits in all its enabled heaps until popped,
    # so a pop leaves exactly (enabled archs - 1) duplicates (P:l.130)
    assert st["dups"] == int(np.sum(np.isfinite(dur).sum(1) - 1))
    key = oracle.score_and_queue(dag, dur, workers)["key"]
    preds = _preds(dag)
    ready_at = np.array([max((fin[p] for p in ps), default=0.0) for ps in preds])
    for T in np.unique(np.concatenate([start, fin])):
        taken = set()
        for a in range(A):
            cand = [t for t in range(n) if ready_at[t] <= T and start[t] >= T and t not in taken
                    and np.isfinite(dur[t, a])]
            cand.sort(key=lambda t: (int(key[t, a]), t))
            got = sorted((t for t in range(n) if start[t] == T and arch[t] == a),
                         key=lambda t: (int(key[t, a]), t))
            assert [t for t in cand[:len(got)]] == got
            taken.update(got)
            running = int(np.sum((arch == a) & (start <= T) & (fin > T)))
            if running < workers[a]:                       # an idle worker of a
                assert len(cand) == len(got)               # nothing left for a


def test_fig4_eviction_removes_gpu_idle_time():
    """Fig. 4 (P:l.222-229): on a tiled Cholesky with one GPU and 16 CPUs the
    eviction mechanism cuts GPU idle time (paper: 29% -> 1%)."""
    w = workloads.cholesky(20)
    dag = oracle.build_dag(w.n, w.src, w.dst)
    idle = {}
    for ev in (False, True):
        st, _, _ = oracle.simulate_dag(dag, w.dur, [16, 1], eviction=ev, trace=False)
        idle[ev] = 1.0 - st["busy"][1] / st["makespan"]
    assert idle[False] > 0.2 and idle[True] < 0.01


def test_replica_sigma_zero_equals_base():
    w = workloads.config("c1")
    dag = oracle.build_dag(w.n, w.src, w.dst)
    a = oracle.simulate_replica(dag, w.dur, [2, 1], 5, 0.0, 3)
    b = oracle.simulate_dag(dag, w.dur, [2, 1])
    assert a[0].tobytes() == b[0].tobytes() and np.array_equal(a[1], b[1]) and np.array_equal(a[2], b[2])


def test_sim_argument_errors():
    dag = _dag(2, [[0, 1]])
    dur = np.ones((2, 1), np.float32)
    with pytest.raises(oracle.OracleError):
        oracle.simulate_dag(dag, dur, [1], max_tries=0)


# ----------------------------------------------------------------------------
# N3: data locality (LS_SDH^2, eq. 3, P:l.205-212), readings l1-l6
# ----------------------------------------------------------------------------

@pytest.mark.parametrize("case", json.load(open(os.path.join(GOLD, "sim_worked.json")))["locality_cases"],
                         ids=lambda c: c["name"])
def test_locality_hand_worked(case):
    dur = np.array(case["dur_ms"], np.float32)
    dag = _dag(len(dur), case["edges"])
    dm = oracle.DataModel(np.array(case["acc_ptr"]), np.array(case["acc_handle"]), np.array(case["acc_mode"]),
                          np.array(case["size"]))
    st, start, worker = oracle.simulate_dag(dag, dur, case["workers"], data=dm, top_n=case["top_n"],
                                            eps=case["eps"], xfer_ms_per_byte=case["xfer_ms_per_byte"])
    assert start.tolist() == case["start"] and worker.tolist() == case["worker"]
    assert st["makespan"] == case["makespan"] and st["moved"] == case["moved"]


def _data(n, seed, H=12):
    return oracle.DataModel(*random_dags.random_data_model(n, H, seed, max_size=1 << 12))


@pytest.mark.parametrize("seed", range(4))
def test_locality_top1_equals_plain_schedule(seed):
    """n = 1 candidate and free transfers: the pick is the heap root, so the
    schedule is the plain N2 one whatever the data model."""
    n = 60
    src, dst = random_dags.random_dag(n, 1.5, seed)
    dag = oracle.build_dag(n, src, dst)
    dur = random_dags.dyadic_durations(n, 2, seed, p_inf=0.2)
    a = oracle.simulate_dag(dag, dur, [2, 1], 3, bool(seed % 2))
    b = oracle.simulate_dag(dag, dur, [2, 1], 3, bool(seed % 2), data=_data(n, seed), top_n=1)
    assert np.array_equal(a[1], b[1]) and np.array_equal(a[2], b[2])
    assert a[0]["makespan"] == b[0]["makespan"]


@pytest.mark.parametrize("seed", range(13))
def test_locality_replay(seed):
    """Replay the schedule independently of the heaps (eviction off, so heap a
    holds exactly the ready, unstarted tasks enabled on a): at every start, in
    (time, worker) order, the task must be the max-LS_SDH^2 candidate among
    the first n in (key, id) order whose gain is within eps of the first
    (ties to the earlier), on the worker's node (arch-0 workers node 0, the
    others one node each); residency follows reads (copy) and writes (only
    copy); finish = start + (delta + missing bytes x cost)."""
    rng = np.random.default_rng(900 + seed)
    wide = seed >= 10          # top_n beyond a warp (33-64): the paper puts no cap on n (P:l.207)
    n = int(rng.integers(20, 90)) if not wide else int(rng.integers(150, 220))
    A = int(rng.integers(1, 4))
    src, dst = random_dags.random_dag(n, float(rng.uniform(0.5, 2.5)) if not wide else 0.3, seed)
    dag = oracle.build_dag(n, src, dst)
    dur = random_dags.dyadic_durations(n, A, seed, p_inf=0.25, tiny_set=bool(seed % 3 == 0))
    workers = rng.integers(1, 3, A).astype(np.int32)
    H = int(rng.integers(2, 10))
    dm = _data(n, seed, H)
    top_n = int(rng.integers(2, 8)) if not wide else int(rng.integers(33, 65))
    eps = float(np.float32(rng.choice([0.0, 0.25, 0.8, 1.0]))) if not wide else 1.0
    cost = float(rng.choice([0.0, 2.0 ** -10]))
    st, start, worker = oracle.simulate_dag(dag, dur, workers, 4, False, data=dm, top_n=top_n, eps=eps,
                                            xfer_ms_per_byte=cost)
    r = oracle.score_and_queue(dag, dur, workers)
    key, gain = r["key"], r["gain"]
    wa = np.repeat(np.arange(A), workers)
    W0 = int(workers[0])
    node = np.array([0 if wa[w] == 0 else 1 + w - W0 for w in range(len(wa))])
    M = int(node.max()) + 1
    res = np.zeros((M, H), bool)
    res[0] = True
    preds = _preds(dag)
    fin = np.full(n, np.inf)
    started = np.zeros(n, bool)
    moved = 0
    max_cand = 0
    for t in sorted(range(n), key=lambda t: (start[t], worker[t])):
        w, T = int(worker[t]), start[t]
        a, m = int(wa[w]), int(node[w])
        ready = [u for u in range(n) if not started[u] and np.isfinite(dur[u, a])
                 and all(fin[p] <= T for p in preds[u])]
        ready.sort(key=lambda u: (int(key[u, a]), u))
        cand = []
        for u in ready[:top_n]:
            if cand and not (np.float32(gain[cand[0], a]) - np.float32(gain[u, a]) <= np.float32(eps)):
                break
            cand.append(u)

        def ls(u):
            v = 0
            for i in range(dm.acc_ptr[u], dm.acc_ptr[u + 1]):
                h = int(dm.acc_handle[i])
                if res[m, h]:
                    z = int(dm.size[h])
                    v += z * z if dm.acc_mode[i] & 2 else z
            return v

        best = max(cand, key=lambda u: (ls(u), -cand.index(u)))
        assert t == best, (t, cand)
        max_cand = max(max_cand, len(cand))
        miss = 0
        for i in range(dm.acc_ptr[t], dm.acc_ptr[t + 1]):
            h = int(dm.acc_handle[i])
            if not res[m, h]:
                miss += int(dm.size[h])
        for i in range(dm.acc_ptr[t], dm.acc_ptr[t + 1]):
            h = int(dm.acc_handle[i])
            if dm.acc_mode[i] & 2:
                res[:, h] = False
            res[m, h] = True
        moved += miss
        started[t] = True
        fin[t] = T + (float(dur[t, a]) + miss * cost)
    assert st["moved"] == moved and st["makespan"] == fin.max()
    if wide:
        assert max_cand > 32


def test_locality_reduces_transfers_cholesky():
    """The point of §V-C: with n = 10, eps = 0.8 (P:l.238) the pick moves
    fewer tiles than the heap root on a tiled Cholesky (2 GPUs, 30 CPUs)."""
    w = workloads.cholesky(16)
    dag = oracle.build_dag(w.n, w.src, w.dst)
    dm = oracle.DataModel(w.acc_ptr, w.acc_handle, w.acc_mode, w.handle_size)
    root = oracle.simulate_dag(dag, w.dur, [30, 2], data=dm, top_n=1, trace=False)[0]
    loc = oracle.simulate_dag(dag, w.dur, [30, 2], data=dm, top_n=10, eps=0.8, trace=False)[0]
    assert loc["moved"] < root["moved"]
