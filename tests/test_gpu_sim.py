"""GPU parity of the N2 simulator (mp_simulate, sm_100a) against the oracle
simulation (oracle/mp_sim_oracle.c): the whole schedule -- start time and
worker of every task -- plus every statistic, bit-exact.

The oracle keeps the paper's binary heaps (P:l.130) and takes the a7 keys;
the GPU takes the a8 queue order and keeps rank bitmaps, so agreement also
checks that the queue order is the heap order.
"""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
import workloads
from workloads import random_dags

pytestmark = pytest.mark.gpu

mp = pytest.importorskip("paper_conf_ipps_tayebbfg24_b200")

DEV = "cuda"


def to_dev(a, dtype=None):
    t = torch.from_numpy(np.ascontiguousarray(a))
    if dtype is not None:
        t = t.to(dtype)
    return t.to(DEV)


def _same_stats(g, o, A):
    assert g["makespan"] == o["makespan"], (g["makespan"], o["makespan"])
    for f in ("pops", "evictions", "dups", "rounds", "moved"):
        assert g[f] == o[f], (f, g[f], o[f])
    assert g["busy"][:A].tobytes() == o["busy"][:A].tobytes()
    assert np.array_equal(g["ran"][:A], o["ran"][:A])


def single_dag(n, src, dst, dur, workers, max_tries=16, eviction=True, kind=mp.MP_CRIT_BOTTOM_LEVEL, data=None,
               **loc):
    """data: (acc_ptr, acc_handle, acc_mode, size) host arrays (N3); loc: top_n / eps / xfer_ms_per_byte."""
    dag = mp.build_dag(n, to_dev(src, torch.int32), to_dev(dst, torch.int32))
    d = to_dev(dur)
    r = mp.score_and_queue(dag, d, workers, kind)
    gdata = None if data is None else mp.DataModel(*data)
    st, start, worker = mp.simulate(dag, d, workers, 0, 0.0, 0, 1, r["qtask"], r["summary"], max_tries, eviction,
                                    trace=True, data=gdata, **loc)
    mp.check(dag)
    od = oracle.build_dag(n, src, dst)
    odata = None if data is None else oracle.DataModel(*data)
    ost, ostart, oworker = oracle.simulate_dag(od, dur, workers, max_tries, eviction, kind, data=odata, **loc)
    g = mp.sim_stats(st)[0]
    assert np.array_equal(start[0].cpu().numpy(), ostart), "start times"
    assert np.array_equal(worker[0].cpu().numpy(), oworker), "workers"
    _same_stats(g, ost, dur.shape[1])
    dag.free()
    return g


@pytest.mark.parametrize("name,workers", [("c1", [2, 1]), ("c1", [1, 1]), ("c2", [30, 2]), ("c2", [16, 1])])
@pytest.mark.parametrize("eviction", [True, False])
def test_cholesky_schedules(name, workers, eviction):
    w = workloads.config(name)
    single_dag(w.n, w.src, w.dst, w.dur, workers, eviction=eviction)


def test_qr_three_arch_and_nod_keys():
    w = workloads.qr(10)
    single_dag(w.n, w.src, w.dst, w.dur, [4, 1, 2])
    single_dag(w.n, w.src, w.dst, w.dur, [4, 1, 2], kind=mp.MP_CRIT_NOD, max_tries=2)


def test_hand_worked_golden_cases():
    import json, os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "sim_worked.json")))
    for c in g["cases"]:
        e = np.array(c["edges"], np.int32).reshape(-1, 2)
        st = single_dag(len(c["dur_ms"]), e[:, 0], e[:, 1], np.array(c["dur_ms"], np.float32), c["workers"],
                        c["max_tries"], c["eviction"])
        assert st["makespan"] == c["makespan"]


@pytest.mark.parametrize("seed", range(12))
def test_random_dags(seed):
    rng = np.random.default_rng(500 + seed)
    n = int(rng.integers(1, 3000))
    A = int(rng.integers(1, 5))
    src, dst = random_dags.random_dag(n, float(rng.uniform(0.3, 4)), seed, dup=0.1)
    dur = random_dags.dyadic_durations(n, A, seed, p_inf=0.3, tiny_set=bool(seed % 3 == 0))
    workers = rng.integers(0, 5, A).astype(np.int32)
    workers[int(rng.integers(0, A))] = int(rng.integers(1, 40))
    # keep every task runnable on an enabled arch
    en = workers > 0
    bad = ~np.any(np.isfinite(dur[:, en]), axis=1)
    dur[bad, int(np.argmax(en))] = 1.0
    single_dag(n, src, dst, dur, workers, int(rng.integers(1, 6)), bool(seed % 2))


def test_many_workers_and_tiny_dag():
    src, dst = random_dags.chain(5)
    dur = np.array([[1, 2]] * 5, np.float32)
    single_dag(5, src, dst, dur, [200, 56])
    single_dag(1, np.zeros(0, np.int32), np.zeros(0, np.int32), np.ones((1, 1), np.float32), [3])


def test_large_dag_global_bitmaps():
    """n large enough that the bitmaps leave shared memory (generic-pointer path)."""
    n, src, dst = random_dags.layered_dag([3000] * 150, 3, 11)
    dur = random_dags.dyadic_durations(n, 2, 11)
    single_dag(n, src, dst, dur, [24, 2])


def _replicas(w, workers, R, r0, sample, eviction=True, max_tries=16):
    dag = mp.build_dag(w.n, to_dev(w.src, torch.int32), to_dev(w.dst, torch.int32))
    r = mp.replicas_simulate(dag, to_dev(w.dur), workers, workloads.C5_SEED, workloads.C5_SIGMA, r0, R,
                             max_tries, eviction, trace=True)
    mp.check(dag)
    st = mp.sim_stats(r["stats"])
    od = oracle.build_dag(w.n, w.src, w.dst)
    for i in sample:
        ost, ostart, oworker = oracle.simulate_replica(od, w.dur, workers, workloads.C5_SEED, workloads.C5_SIGMA,
                                                       r0 + i, max_tries, eviction)
        assert np.array_equal(r["start"][i].cpu().numpy(), ostart)
        assert np.array_equal(r["worker"][i].cpu().numpy(), oworker)
        _same_stats(st[i], ost, w.n_arch)
    dag.free()
    return st


def test_replicas_c1_all():
    _replicas(workloads.config("c1"), [3, 1], 64, 5, range(64))


def test_replicas_c2_sampled():
    R = 300
    st = _replicas(workloads.config("c2"), [30, 2], R, 1000, [0, 1, 77, 150, R - 1])
    assert np.all(st["pops"] == 45760)


def test_replicas_world_size_invariant():
    w = workloads.config("c1")
    dag = mp.build_dag(w.n, to_dev(w.src, torch.int32), to_dev(w.dst, torch.int32))
    d = to_dev(w.dur)
    a = mp.sim_stats(mp.replicas_simulate(dag, d, [2, 1], 9, 0.125, 0, 40)["stats"])
    b1 = mp.sim_stats(mp.replicas_simulate(dag, d, [2, 1], 9, 0.125, 0, 17)["stats"])
    b2 = mp.sim_stats(mp.replicas_simulate(dag, d, [2, 1], 9, 0.125, 17, 23)["stats"])
    assert a.tobytes() == np.concatenate([b1, b2]).tobytes()


def test_sim_rejects_ready_mode_queues():
    w = workloads.config("c1")
    dag = mp.build_dag(w.n, to_dev(w.src, torch.int32), to_dev(w.dst, torch.int32))
    d = to_dev(w.dur)
    done = torch.zeros(w.n, dtype=torch.uint8, device=DEV)
    r = mp.score_and_queue(dag, d, w.workers, done=done)      # READY mode: sources only
    mp.simulate(dag, d, w.workers, 0, 0.0, 0, 1, r["qtask"], r["summary"])
    with pytest.raises(mp.MPError):
        mp.check(dag)


# ----------------------------------------------------------------------------
# N3: data-locality pick (LS_SDH^2) + residency + transfer cost
# ----------------------------------------------------------------------------

def test_locality_hand_worked_golden_cases():
    import json, os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "sim_worked.json")))
    for c in g["locality_cases"]:
        e = np.array(c["edges"], np.int32).reshape(-1, 2)
        data = (np.array(c["acc_ptr"]), np.array(c["acc_handle"]), np.array(c["acc_mode"]), np.array(c["size"]))
        st = single_dag(len(c["dur_ms"]), e[:, 0], e[:, 1], np.array(c["dur_ms"], np.float32), c["workers"],
                        data=data, top_n=c["top_n"], eps=c["eps"], xfer_ms_per_byte=c["xfer_ms_per_byte"])
        assert st["makespan"] == c["makespan"] and st["moved"] == c["moved"]


@pytest.mark.parametrize("seed", range(12))
def test_locality_random(seed):
    rng = np.random.default_rng(700 + seed)
    n = int(rng.integers(5, 2500))
    A = int(rng.integers(1, 4))
    src, dst = random_dags.random_dag(n, float(rng.uniform(0.3, 3)), seed, dup=0.1)
    dur = random_dags.dyadic_durations(n, A, seed, p_inf=0.25, tiny_set=bool(seed % 3 == 0))
    workers = rng.integers(1, 5, A).astype(np.int32)
    H = int(rng.integers(1, 3000))
    data = random_dags.random_data_model(n, H, seed, max_size=1 << 16)
    single_dag(n, src, dst, dur, workers, int(rng.integers(1, 6)), bool(seed % 2), data=data,
               top_n=int(rng.integers(1, 33)), eps=float(rng.choice([0.0, 0.125, 0.8, 1.0])),
               xfer_ms_per_byte=float(rng.choice([0.0, 2.0 ** -12])))


def test_locality_cholesky_c2():
    w = workloads.config("c2")
    data = (w.acc_ptr, w.acc_handle, w.acc_mode, w.handle_size)
    st = single_dag(w.n, w.src, w.dst, w.dur, [30, 2], data=data, top_n=10, eps=0.8, xfer_ms_per_byte=2.0 ** -24)
    assert st["moved"] > 0


def test_locality_global_residency():
    """Many handles: residency bitmaps leave shared memory (generic-pointer path)."""
    n, src, dst = random_dags.layered_dag([400] * 10, 3, 5)
    dur = random_dags.dyadic_durations(n, 2, 5)
    data = random_dags.random_data_model(n, 600_000, 5, max_size=1 << 20)
    single_dag(n, src, dst, dur, [6, 3], data=data, top_n=10, eps=0.8, xfer_ms_per_byte=2.0 ** -20)


def test_locality_replicas_sampled():
    w = workloads.config("c2")
    workers = [30, 2]
    dag = mp.build_dag(w.n, to_dev(w.src, torch.int32), to_dev(w.dst, torch.int32))
    loc = dict(top_n=10, eps=0.8, xfer_ms_per_byte=2.0 ** -24)
    r = mp.replicas_simulate(dag, to_dev(w.dur), workers, workloads.C5_SEED, workloads.C5_SIGMA, 40, 160,
                             trace=True, data=mp.DataModel(w.acc_ptr, w.acc_handle, w.acc_mode, w.handle_size), **loc)
    mp.check(dag)
    st = mp.sim_stats(r["stats"])
    od = oracle.build_dag(w.n, w.src, w.dst)
    odata = oracle.DataModel(w.acc_ptr, w.acc_handle, w.acc_mode, w.handle_size)
    for i in (0, 99, 159):
        ost, ostart, oworker = oracle.simulate_replica(od, w.dur, workers, workloads.C5_SEED, workloads.C5_SIGMA,
                                                       40 + i, data=odata, **loc)
        assert np.array_equal(r["start"][i].cpu().numpy(), ostart)
        assert np.array_equal(r["worker"][i].cpu().numpy(), oworker)
        _same_stats(st[i], ost, 2)
