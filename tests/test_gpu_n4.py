"""GPU parity of the N4 variants (mp_bottom_level_w, mp_affinity_prefix,
mp_nod_remaining) and the LU workload against the oracle, bit-exact."""
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


def bits(a):
    return np.ascontiguousarray(a, dtype=np.float32).view(np.uint32)


def _dags(n, src, dst):
    return mp.build_dag(n, to_dev(src, torch.int32), to_dev(dst, torch.int32)), oracle.build_dag(n, src, dst)


CASES = [("c1", None), ("c2", None), ("c3", None), ("lu16", None)] + [(f"rand{s}", s) for s in range(8)]


def _case(name, seed):
    if seed is None:
        w = workloads.lu(16) if name == "lu16" else workloads.config(name)
        return w.n, w.src, w.dst, w.dur, np.array([3, 2, 1][:w.n_arch], np.int32)
    rng = np.random.default_rng(1000 + seed)
    n = int(rng.integers(1, 5000))
    A = int(rng.integers(1, 5))
    src, dst = random_dags.random_dag(n, float(rng.uniform(0.3, 4)), seed, dup=0.1)
    dur = random_dags.dyadic_durations(n, A, seed, p_inf=0.3, tiny_set=bool(seed % 3 == 0))
    workers = rng.integers(1, 7, A).astype(np.int32)
    return n, src, dst, dur, workers


@pytest.mark.parametrize("name,seed", CASES, ids=[c[0] for c in CASES])
def test_mean_weight_bottom_level(name, seed):
    n, src, dst, dur, workers = _case(name, seed)
    g, o = _dags(n, src, dst)
    bl, cp = mp.bottom_level_w(g, to_dev(dur), workers, mp.MP_WEIGHT_MEAN)
    mp.check(g)
    obl, ocp = oracle.bottom_level_w(o, dur, workers, oracle.WEIGHT_MEAN)
    assert np.array_equal(bits(bl.cpu().numpy()), bits(obl))
    assert bits(cp.cpu().numpy())[0] == bits(np.float32(ocp))
    # MP_WEIGHT_MIN is mp_bottom_level
    bl2, _ = mp.bottom_level_w(g, to_dev(dur), workers, mp.MP_WEIGHT_MIN)
    assert np.array_equal(bits(bl2.cpu().numpy()), bits(oracle.bottom_level(o, dur, workers)[0]))


@pytest.mark.parametrize("name,seed", CASES, ids=[c[0] for c in CASES])
def test_prefix_hd_gains(name, seed):
    n, src, dst, dur, workers = _case(name, seed)
    g, o = _dags(n, src, dst)
    for order in (None, np.random.default_rng(n).permutation(n).astype(np.int32)):
        gain, hd, flags = mp.affinity_prefix(g, to_dev(dur), workers, None if order is None else to_dev(order))
        mp.check(g)
        og, oh, of = oracle.affinity_prefix(dur, workers, order)
        assert np.array_equal(bits(gain.cpu().numpy()), bits(og))
        assert np.array_equal(bits(hd.cpu().numpy()), bits(oh))
        assert np.array_equal(flags.cpu().numpy(), of)


@pytest.mark.parametrize("name,seed", CASES, ids=[c[0] for c in CASES])
def test_nod_remaining(name, seed):
    n, src, dst, dur, workers = _case(name, seed)
    g, o = _dags(n, src, dst)
    rng = np.random.default_rng(7 + n)
    for frac in (0.0, 0.3, 0.7):
        done = np.zeros(n, np.uint8)
        done[o.level_order[: int(frac * n)]] = 1
        nod = mp.nod_remaining(g, to_dev(dur), workers, to_dev(done))
        mp.check(g)
        onod = oracle.nod_remaining(o, dur, workers, done)
        assert np.array_equal(bits(nod.cpu().numpy()), bits(onod))
    done = (rng.random(n) < 0.5).astype(np.uint8)           # arbitrary masks too
    assert np.array_equal(bits(mp.nod_remaining(g, to_dev(dur), workers, to_dev(done)).cpu().numpy()),
                          bits(oracle.nod_remaining(o, dur, workers, done)))


def test_prefix_order_out_of_range_is_an_error():
    w = workloads.config("c1")
    g, _ = _dags(w.n, w.src, w.dst)
    order = torch.arange(w.n, dtype=torch.int32, device=DEV)
    order[3] = w.n
    mp.affinity_prefix(g, to_dev(w.dur), w.workers, order)
    with pytest.raises(mp.MPError):
        mp.check(g)


def test_lu64_full_path_bit_exact():
    """N4 workload: tiled LU 64x64 (getrf, P:l.251) through the whole a1-a9 path."""
    w = workloads.config("lu64")
    g, o = _dags(w.n, w.src, w.dst)
    r = mp.score_and_queue(g, to_dev(w.dur), w.workers)
    mp.check(g)
    orr = oracle.score_and_queue(o, w.dur, w.workers)
    assert g.n_levels == o.n_levels == 190 and g.n_edges == o.n_edges
    assert np.array_equal(bits(r["bl"].cpu().numpy()), bits(orr["bl"]))
    Q = int(orr["qptr"][-1])
    assert np.array_equal(r["qtask"].cpu().numpy()[:Q], orr["qtask"])
    assert r["summary"].cpu().numpy().tobytes() == orr["summary"].tobytes()


def _full_compare(w, kind=oracle.CRIT_BL):
    """The whole a1-a9 path on the GPU vs the oracle, every output bit-exact."""
    g, o = _dags(w.n, w.src, w.dst)
    r = mp.score_and_queue(g, to_dev(w.dur), w.workers, kind)
    mp.check(g)
    orr = oracle.score_and_queue(o, w.dur, w.workers, kind)
    ga = {k: v.cpu().numpy() for k, v in g.arrays().items()}
    assert g.n_levels == o.n_levels and g.n_edges == o.n_edges
    for k in ("row_ptr", "col", "indeg", "level", "level_ptr", "level_order"):
        assert np.array_equal(ga[k], getattr(o, k)), k
    assert np.array_equal(bits(r["bl"].cpu().numpy()), bits(orr["bl"]))
    assert np.array_equal(bits(r["gain"].cpu().numpy()), bits(orr["gain"]))
    assert np.array_equal(bits(r["crit_norm"].cpu().numpy()), bits(orr["crit_norm"]))
    assert np.array_equal(r["key"].cpu().numpy().view(np.uint64), orr["key"])
    Q = int(orr["qptr"][-1])
    assert np.array_equal(r["qptr"].cpu().numpy(), orr["qptr"])
    assert np.array_equal(r["qtask"].cpu().numpy()[:Q], orr["qtask"])
    assert r["summary"].cpu().numpy().tobytes() == orr["summary"].tobytes()
    return g, o


@pytest.mark.parametrize("N,p,seed", [(6, 0.5, 1), (12, 0.3, 2), (16, 1.0, 3), (16, 0.0, 4)])
def test_hier_small_full_path_bit_exact(N, p, seed):
    """N4 hierarchical-task Cholesky (P:l.318): mixed granularity, no / full expansion."""
    w = workloads.hier(N, 2, p, seed)
    _full_compare(w)
    _full_compare(w, oracle.CRIT_NOD)


def test_hier_config_full_path_and_replicas():
    """The bench's hier config (48 x 48 coarse tiles, half expanded: 85,673 tasks) through
    a1-a9, then 40 duration-perturbed replicas of it (a10; n >= 65,536: the general path) against
    the oracle, every replica."""
    w = workloads.config("hier")
    g, o = _full_compare(w)
    R = 40
    cp, summ, q = mp.replicas_run(g, to_dev(w.dur), w.workers, workloads.C5_SEED, workloads.C5_SIGMA, 5, R)
    mp.check(g)
    cp = cp.cpu().numpy()
    gs = mp.summaries(summ).reshape(R, w.n_arch)
    q = q.cpu().numpy()
    for i in range(R):
        ocp, osum, oq, _ = oracle.replica(o, w.dur, w.workers, workloads.C5_SEED, workloads.C5_SIGMA, 5 + i)
        assert bits(cp[i:i + 1])[0] == bits(np.float32(ocp)), i
        assert gs[i].tobytes() == osum.tobytes(), i
        assert np.array_equal(q[i, :len(oq)], oq), i
