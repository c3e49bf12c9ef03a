"""GPU parity: libmp (sm_100a, through the C-ABI) vs the CPU oracle, bit-exact.

Every float output is compared on its bit pattern; integer / index outputs are
compared exactly; queue orders are unique (ties broken by id) so they must be
identical.  Inputs are the seeded workloads of DESIGN.md §3.
"""
from __future__ import annotations

import os
from concurrent.futures import ThreadPoolExecutor

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


def gpu_path(n, src, dst, dur, workers, kind=0, done=None):
    dag = mp.build_dag(n, to_dev(src, torch.int32), to_dev(dst, torch.int32))
    r = mp.score_and_queue(dag, to_dev(dur), workers, kind, None if done is None else to_dev(done))
    mp.check(dag)
    out = {k: (v.cpu().numpy() if isinstance(v, torch.Tensor) else v) for k, v in r.items()}
    out["arrays"] = {k: v.cpu().numpy() for k, v in dag.arrays().items()}
    out["dag"] = dag
    return out


def compare(n, src, dst, dur, workers, kind=0, done=None):
    g = gpu_path(n, src, dst, dur, workers, kind, done)
    od = oracle.build_dag(n, src, dst)
    ga = g["arrays"]
    assert g["dag"].n_edges == od.n_edges and g["dag"].n_levels == od.n_levels
    assert np.array_equal(ga["row_ptr"], od.row_ptr)
    assert np.array_equal(ga["col"], od.col)
    assert np.array_equal(ga["indeg"], od.indeg)
    assert np.array_equal(ga["level"], od.level)
    assert np.array_equal(ga["level_ptr"], od.level_ptr)
    assert np.array_equal(ga["level_order"], od.level_order)
    if n == 0:
        return g
    o = oracle.score_and_queue(od, dur, workers, kind, done)
    assert np.array_equal(bits(g["bl"]), bits(o["bl"])), "bottom-level"
    assert bits(g["cp"])[0] == bits(np.float32(o["cp"]))
    assert np.array_equal(g["flags"], o["flags"])
    assert np.array_equal(bits(g["hd"]), bits(o["hd"]))
    assert np.array_equal(bits(g["gain"]), bits(o["gain"])), "gain"
    if kind == oracle.CRIT_NOD:
        assert np.array_equal(bits(g["nod"]), bits(o["crit"])), "NOD"
    assert np.array_equal(bits(g["crit_norm"]), bits(o["crit_norm"])), "crit_norm"
    assert np.array_equal(g["key"].view(np.uint64), o["key"]), "key"
    assert np.array_equal(g["qptr"], o["qptr"])
    Q = int(o["qptr"][-1])
    assert np.array_equal(g["qtask"][:Q], o["qtask"]), "queue order"
    gs = g["summary"].view(mp.SUMMARY_DTYPE)
    assert gs.tobytes() == o["summary"].tobytes(), (gs, o["summary"])
    return g


@pytest.mark.parametrize("name", ["c1", "c2", "c3"])
def test_configs_bit_exact(name):
    w = workloads.config(name)
    compare(w.n, w.src, w.dst, w.dur, w.workers)


def test_c4_bit_exact():
    w = workloads.config("c4")
    compare(w.n, w.src, w.dst, w.dur, w.workers)


@pytest.mark.parametrize("name", ["c1", "c2", "c3", "c4"])
def test_nod_bit_exact(name):
    w = workloads.config(name)
    compare(w.n, w.src, w.dst, w.dur, w.workers, kind=oracle.CRIT_NOD)


def test_nod_three_arch_masks():
    w = workloads.qr(24)
    compare(w.n, w.src, w.dst, w.dur, w.workers, kind=oracle.CRIT_NOD)


@pytest.mark.parametrize("seed,n,deg,A,p_inf,tiny", [
    (0, 1, 0.0, 2, 0.0, False),
    (1, 2, 1.0, 1, 0.0, False),
    (2, 777, 2.5, 2, 0.2, False),
    (3, 5000, 3.0, 3, 0.3, True),
    (4, 40000, 4.0, 2, 0.1, True),
    (5, 60000, 2.0, 2, 0.0, False),      # > SMALL_CAP: dataflow kernel
    (6, 250000, 3.0, 3, 0.25, True),     # dataflow, 3 archs, ties
])
def test_random_dags(seed, n, deg, A, p_inf, tiny):
    src, dst = random_dags.random_dag(n, deg, seed, dup=0.3, max_span=64)
    dur = random_dags.dyadic_durations(n, A, seed, p_inf=p_inf, tiny_set=tiny)
    compare(n, src, dst, dur, np.ones(A, np.int32))


def test_deep_chain_and_wide_star():
    n = 6000
    s, d = random_dags.chain(n)
    compare(n, s, d, random_dags.dyadic_durations(n, 2, 1), np.ones(2, np.int32))
    n = 70000
    s, d = random_dags.chain(n)             # deep chain through the dataflow kernel
    compare(n, s, d, random_dags.dyadic_durations(n, 2, 2), np.ones(2, np.int32))
    n = 100000
    s, d = random_dags.star(n)              # one node with 99,999 successors
    compare(n, s, d, random_dags.dyadic_durations(n, 2, 3), np.ones(2, np.int32))
    s2, d2 = d.copy(), s.copy()             # fan-in of 99,999
    compare(n, s2, d2, random_dags.dyadic_durations(n, 2, 4), np.ones(2, np.int32))


@pytest.mark.parametrize("seed,n,deg,span", [
    (11, 3000, 3.0, 8),          # chains inside 32-id chunks
    (12, 60000, 6.0, 16),
    (13, 200000, 4.0, None),     # long-range edges
    (14, 100000, 40.0, 4096),    # ~1,280 predecessors per chunk: pending list full -> in-place waits
])
def test_id_order_dags(seed, n, deg, span):
    """Id order is topological (every edge to a larger id, as in a sequential task flow):
    the levels come from the pull dataflow k_lvl_flow instead of the level-synchronous Kahn;
    levels, level order, q-space and the whole score path bit-exact with the oracle."""
    src, dst = random_dags.random_dag(n, deg, seed, dup=0.2, permute=False, max_span=span)
    assert (src < dst).all()
    compare(n, src, dst, random_dags.dyadic_durations(n, 2, seed, p_inf=0.1, tiny_set=True), np.ones(2, np.int32))


def test_id_order_fan_in():
    """One sink with 99,999 predecessors, id order topological (k_lvl_flow, one chunk waiting
    on a full pending list)."""
    n = 100000
    s = np.arange(n - 1, dtype=np.int32)
    d = np.full(n - 1, n - 1, np.int32)
    compare(n, s, d, random_dags.dyadic_durations(n, 2, 5), np.ones(2, np.int32))


def test_one_block_kahn_frontier_spill():
    """a2 ingest, one-block Kahn (n <= 48K): the first sfcap (<= 8192) entries of a frontier
    live in shared memory, the rest spill to the global list -- levels narrower than, equal
    to and wider than the shared part, and a star whose one level holds 39,999 tasks."""
    n = 40000
    s, d = random_dags.star(n)
    compare(n, s, d, random_dags.dyadic_durations(n, 2, 21), np.ones(2, np.int32))
    compare(n, d.copy(), s.copy(), random_dags.dyadic_durations(n, 2, 22), np.ones(2, np.int32))
    n, s, d = random_dags.layered_dag([1, 2047, 2048, 2049, 8191, 8192, 8193, 12000, 5], fan=6, seed=23)
    assert n <= 48 * 1024
    compare(n, s, d, random_dags.dyadic_durations(n, 2, 23, tiny_set=True), np.ones(2, np.int32))


def test_csr_row_length_boundaries():
    """a1 ingest: rows of every length class of the counting-sort builder (warp rank sort
    up to 256 entries, radix path above), heavy duplication, shuffled edge order."""
    rng = np.random.default_rng(77)
    lens = [0, 1, 2, 31, 32, 33, 63, 64, 65, 255, 256, 257, 258, 1000, 4097, 20000, 3, 129]
    n = 30000
    src, dst = [], []
    for i, L in enumerate(lens):
        u = i                                   # sources 0..17, targets above them (acyclic)
        span = max(1, L // 3) if i % 2 else L   # odd rows: ~3 copies of every successor
        v = rng.integers(len(lens), min(n, len(lens) + span + 1), size=L)
        src.append(np.full(L, u, np.int32))
        dst.append(v.astype(np.int32))
    src, dst = np.concatenate(src), np.concatenate(dst)
    p = rng.permutation(len(src))
    src, dst = src[p], dst[p]
    compare(n, src, dst, random_dags.dyadic_durations(n, 2, 12), np.ones(2, np.int32))


def test_layered_skewed_fanin():
    n, s, d = random_dags.layered_dag([3000, 50, 20000, 7, 40000, 1], fan=40, seed=9)
    compare(n, s, d, random_dags.dyadic_durations(n, 2, 9, tiny_set=True), np.ones(2, np.int32))


def test_medium_dags_many_edges():
    """Medium DAGs past k_bl_one's edge budget (1 Mi < E <= 8 Mi, the dataflow kernel):
    levels narrower than a warp next to 30,000-wide levels with up to 60 predecessors per
    task, and a random deep DAG (39,108 levels) with three archs and ties."""
    n, s, d = random_dags.layered_dag([1, 3, 30000, 2, 30000, 30000, 30000, 1, 16, 9000, 17, 5], fan=60, seed=41)
    g = compare(n, s, d, random_dags.dyadic_durations(n, 2, 41, tiny_set=True), np.ones(2, np.int32))
    assert 1 << 20 < g["dag"].n_edges <= 8 << 20
    n = 300000
    s, d = random_dags.random_dag(n, 5.0, 42, dup=0.1, max_span=64)
    g = compare(n, s, d, random_dags.dyadic_durations(n, 3, 42, p_inf=0.2, tiny_set=True), np.ones(3, np.int32))
    assert 1 << 20 < g["dag"].n_edges <= 8 << 20


def test_empty_and_edgeless():
    compare(0, np.zeros(0, np.int32), np.zeros(0, np.int32), np.zeros((0, 2), np.float32), np.ones(2, np.int32))
    n = 5000
    compare(n, np.zeros(0, np.int32), np.zeros(0, np.int32), random_dags.dyadic_durations(n, 2, 5),
            np.ones(2, np.int32))


def test_workers_disable_and_zero_durations():
    w = workloads.config("c2")
    dur = w.dur.copy()
    dur[::7, 0] = 0.0
    dur[::11, 1] = -0.0
    compare(w.n, w.src, w.dst, dur, np.array([3, 1], np.int32))
    compare(w.n, w.src, w.dst, dur, np.array([0, 2], np.int32))


def test_ready_mode():
    w = workloads.config("c2")
    od = oracle.build_dag(w.n, w.src, w.dst)
    rng = np.random.default_rng(1)
    done = np.zeros(w.n, np.uint8)
    done[od.level_order[: w.n // 4]] = 1
    done[rng.integers(0, w.n, 100)] = 1
    compare(w.n, w.src, w.dst, w.dur, w.workers, done=done)


def test_domain_and_graph_errors():
    n = 4
    ok_dur = np.ones((n, 2), np.float32)
    with pytest.raises(mp.MPError) as e:
        mp.build_dag(n, to_dev(np.array([0, 1, 2], np.int32)), to_dev(np.array([1, 2, 0], np.int32)))
    assert e.value.code == mp.MP_ERR_CYCLE
    with pytest.raises(mp.MPError) as e:
        mp.build_dag(n, to_dev(np.array([0], np.int32)), to_dev(np.array([0], np.int32)))
    assert e.value.code == mp.MP_ERR_ARG
    with pytest.raises(mp.MPError) as e:
        mp.build_dag(n, to_dev(np.array([0], np.int32)), to_dev(np.array([4], np.int32)))
    assert e.value.code == mp.MP_ERR_ARG
    dag = mp.build_dag(n, to_dev(np.array([0, 1], np.int32)), to_dev(np.array([1, 2], np.int32)))
    for bad in (np.nan, -1.0, 2.0 ** -42, 2.0 ** 20, -np.inf):
        d = ok_dur.copy()
        d[2, 1] = bad
        mp.bottom_level(dag, to_dev(d), [1, 1])
        with pytest.raises(mp.MPError) as e:
            mp.check(dag)
        assert e.value.code == mp.MP_ERR_DOMAIN
    d = ok_dur.copy()
    d[1] = np.inf
    mp.affinity(dag, to_dev(d), [1, 1])
    with pytest.raises(mp.MPError):
        mp.check(dag)
    mp.check(dag)  # flag cleared
    with pytest.raises(ValueError):
        mp.bottom_level(dag, to_dev(ok_dur), [1, 1, 1])
    with pytest.raises(TypeError):                      # no CPU path
        mp.bottom_level(dag, torch.from_numpy(ok_dur), [1, 1])


def test_deterministic_repeat():
    w = workloads.config("c3")
    a = gpu_path(w.n, w.src, w.dst, w.dur, w.workers)
    b = gpu_path(w.n, w.src, w.dst, w.dur, w.workers)
    for k in ("bl", "gain", "key", "qtask", "summary"):
        assert np.array_equal(a[k], b[k])


# ----------------------------------------------------------------------------
# a10 replicas
# ----------------------------------------------------------------------------

def _replica_check(w, R, r0, sample, sigma=workloads.C5_SIGMA, seed=workloads.C5_SEED):
    dag = mp.build_dag(w.n, to_dev(w.src, torch.int32), to_dev(w.dst, torch.int32))
    base = to_dev(w.dur)
    cp, summ, q = mp.replicas_run(dag, base, w.workers, seed, sigma, r0, R, want_queues=True)
    mp.check(dag)
    cp = cp.cpu().numpy()
    gs = mp.summaries(summ).reshape(R, w.n_arch)
    q = q.cpu().numpy()
    od = oracle.build_dag(w.n, w.src, w.dst)
    for i in sample:
        ocp, osum, oq, oqptr = oracle.replica(od, w.dur, w.workers, seed, sigma, r0 + i)
        assert bits(cp[i:i + 1])[0] == bits(np.float32(ocp)), i
        assert gs[i].tobytes() == osum.tobytes(), (i, gs[i], osum)
        assert np.array_equal(q[i, :len(oq)], oq), i
    return cp, gs, q


def test_replicas_c1_all():
    w = workloads.config("c1")
    _replica_check(w, 300, 0, range(300))


def _oracle_replicas(od, w, rs, sigma=workloads.C5_SIGMA, seed=workloads.C5_SEED):
    """oracle.replica for every r in rs on all host cores (the C oracle drops the
    GIL inside ctypes and keeps no global state per replica call)."""
    with ThreadPoolExecutor(max_workers=max(1, len(os.sched_getaffinity(0)))) as ex:
        return list(ex.map(lambda r: oracle.replica(od, w.dur, w.workers, seed, sigma, r), rs))


def test_replicas_c5_all_full_size():
    """C5 at full size (all replicas when the budget allows): every one
    of the 4096 replicas -- CP, the 32-byte summaries and both 45,760-entry queues --
    bit-exact against the oracle, in the launch configuration bench.py times (one
    mp_replicas_run over all R); then world-size invariance: the two halves
    [0, R/2) and [R/2, R) run as separate calls (two ranks) give identical bytes."""
    w = workloads.config("c5")
    R = workloads.C5_REPLICAS
    dag = mp.build_dag(w.n, to_dev(w.src, torch.int32), to_dev(w.dst, torch.int32))
    base = to_dev(w.dur)
    cp, summ, q = mp.replicas_run(dag, base, w.workers, workloads.C5_SEED, workloads.C5_SIGMA, 0, R)
    mp.check(dag)
    cp_h = cp.cpu().numpy()
    gs = mp.summaries(summ).reshape(R, w.n_arch)
    od = oracle.build_dag(w.n, w.src, w.dst)
    CH = 512
    for c0 in range(0, R, CH):
        res = _oracle_replicas(od, w, range(c0, c0 + CH))
        qc = q[c0:c0 + CH].cpu().numpy()
        for i, (ocp, osum, oq, _) in enumerate(res):
            r = c0 + i
            assert bits(cp_h[r:r + 1])[0] == bits(np.float32(ocp)), r
            assert gs[r].tobytes() == osum.tobytes(), (r, gs[r], osum)
            assert np.array_equal(qc[i, :len(oq)], oq), r
    h = R // 2
    cp2, s2, q2 = mp.replicas_run(dag, base, w.workers, workloads.C5_SEED, workloads.C5_SIGMA, h, R - h)
    mp.check(dag)
    assert np.array_equal(bits(cp2.cpu().numpy()), bits(cp_h[h:]))
    assert mp.summaries(s2).tobytes() == gs[h:].tobytes()
    assert torch.equal(q2, q[h:])


def test_replicas_sigma_zero_equals_single_dag():
    w = workloads.config("c2")
    dag = mp.build_dag(w.n, to_dev(w.src, torch.int32), to_dev(w.dst, torch.int32))
    cp, summ, q = mp.replicas_run(dag, to_dev(w.dur), w.workers, 7, 0.0, 0, 3)
    one = mp.score_and_queue(dag, to_dev(w.dur), w.workers)
    mp.check(dag)
    for i in range(3):
        assert bits(cp.cpu().numpy())[i] == bits(one["cp"].cpu().numpy())[0]
        assert np.array_equal(q.cpu().numpy()[i], one["qtask"].cpu().numpy())
        assert mp.summaries(summ)[i * 2:(i + 1) * 2].tobytes() == one["summary"].cpu().numpy().tobytes()


def test_replicas_rep2_upper_size():
    """n = 60,000 (< 65,536, A = 2): the lanes=replicas path (k_rep2_bl + k_rep2_sort)
    at its largest size class (bl no longer fits one CTA's shared memory); qr(40)
    (n = 22,140) for the same kernels on a QR shape."""
    src, dst = random_dags.random_dag(60000, 2.0, 3, max_span=64)
    dur = random_dags.dyadic_durations(60000, 2, 3)
    W = workloads.Workload("r", 60000, src, dst, dur, ("CPU", "GPU"), np.ones(2, np.int32))
    _replica_check(W, 3, 11, range(3))
    _replica_check(workloads.qr(40), 5, 100, range(5))


def test_replicas_general_path_large_dag():
    """n >= 65,536: the general replica path (perturbation kernel + the single-DAG
    a4-a9 kernels once per replica), 2 and 6 archs, every replica checked."""
    n = 70000
    src, dst = random_dags.random_dag(n, 2.5, 31, dup=0.2, max_span=128)
    dur = random_dags.dyadic_durations(n, 2, 31)
    W = workloads.Workload("g2", n, src, dst, dur, ("CPU", "GPU"), np.ones(2, np.int32))
    _replica_check(W, 4, 7, range(4))
    dur6 = random_dags.dyadic_durations(n, 6, 32, p_inf=0.3, tiny_set=True)
    W6 = workloads.Workload("g6", n, src, dst, dur6, tuple(f"a{i}" for i in range(6)), np.ones(6, np.int32))
    _replica_check(W6, 3, 0, range(3))


@pytest.mark.parametrize("A", [5, 6, 7, 8])
def test_replicas_general_path_many_archs(A):
    """A = 5..8 (> 4, so not the lanes=replicas path): the batched one-CTA-per-replica
    path (k_rep_main + segmented sort + k_rep_out), masks and ties, every replica."""
    w = workloads.config("c1") if A % 2 else workloads.qr(8)
    rng = np.random.default_rng(A)
    n = w.n
    src, dst = random_dags.random_dag(3000, 2.0, 50 + A, dup=0.2, max_span=64) if A >= 7 else (w.src, w.dst)
    if A >= 7:
        n = 3000
    dur = random_dags.dyadic_durations(n, A, 60 + A, p_inf=0.3, tiny_set=bool(A % 2))
    workers = np.ones(A, np.int32)
    if A == 8:
        workers[3] = 0
        en = np.isfinite(dur) & (workers[None, :] > 0)
        dur[~en.any(1), 0] = 1.0
    W = workloads.Workload(f"m{A}", n, src, dst, dur, tuple(f"a{i}" for i in range(A)), workers)
    R = int(rng.integers(40, 70))
    _replica_check(W, R, int(rng.integers(0, 5000)), range(R))


def test_replicas_three_arch_masks_all():
    w = workloads.qr(10)              # A = 3, ACC column has +inf entries
    _replica_check(w, 70, 5, range(70))


def test_replicas_one_arch_and_disabled_arch():
    w = workloads.config("c2")
    one = workloads.Workload("c2a1", w.n, w.src, w.dst, np.ascontiguousarray(w.dur[:, :1]), ("CPU",),
                             np.ones(1, np.int32))
    _replica_check(one, 33, 0, [0, 17, 32])
    dis = workloads.Workload("c2dis", w.n, w.src, w.dst, w.dur, w.arch_names, np.array([1, 0], np.int32))
    _replica_check(dis, 33, 64, [0, 31, 32])


def test_replicas_k1_fast_path_boundaries():
    """Two archs, all enabled: k_rep2_bl's fast path (single-uint64 best_remaining_work in
    units of the smallest binade) on its edges -- equal durations on both archs (every task
    tied best on both at sigma = 0, and near-ties otherwise), durations at the domain's ends
    (span too wide: the 128-bit path), and one task whose lower extreme leaves the domain."""
    w = workloads.config("c1")
    eq = np.ascontiguousarray(np.repeat(w.dur[:, 1:2], 2, axis=1))
    We = workloads.Workload("c1eq", w.n, w.src, w.dst, eq, w.arch_names, w.workers)
    _replica_check(We, 64, 0, range(64), sigma=0.0)
    _replica_check(We, 64, 0, range(64))
    wide = w.dur.copy()
    wide[0, 0] = np.float32(2.0 ** -40)
    wide[1, 1] = np.float32(2.0 ** 19)
    Ww = workloads.Workload("c1wide", w.n, w.src, w.dst, np.ascontiguousarray(wide), w.arch_names, w.workers)
    _replica_check(Ww, 64, 3, range(64))
    edge = w.dur.copy()
    edge[2, 0] = np.float32(2.0 ** -41)            # u = 0 draws go below 2^-41 only if sigma > 0: keep sigma 0
    Wd = workloads.Workload("c1edge", w.n, w.src, w.dst, np.ascontiguousarray(edge), w.arch_names, w.workers)
    _replica_check(Wd, 32, 9, range(32), sigma=0.0)


def test_replicas_k1_dataflow_many_groups():
    """>= 75 groups of 32 replicas: one CTA per group, k_rep2_bl's dataflow mode (ready bytes
    instead of level barriers), on 1, 2 and 3 archs (masks, one-arch tasks)."""
    rng = np.random.default_rng(5)
    c1 = workloads.config("c1")
    R = 2600
    sample = sorted(set([0, 31, 32, R - 1] + rng.integers(0, R, 60).tolist()))
    _replica_check(c1, R, 17, sample)
    one = workloads.Workload("c1a1", c1.n, c1.src, c1.dst, np.ascontiguousarray(c1.dur[:, :1]), ("CPU",),
                             np.ones(1, np.int32))
    _replica_check(one, R, 0, sample)
    _replica_check(workloads.qr(6), R, 3, sample)


def test_replicas_ties_stream_path():
    """sigma = 0 on c2: 41,664 GEMMs share one gain -> key ranges with one value > 16384 entries."""
    w = workloads.config("c2")
    _replica_check(w, 40, 0, [0, 39], sigma=0.0)


@pytest.mark.parametrize("sigma", [2.0 ** -10, 2.0 ** -16, 2.0 ** -21])
def test_replicas_tiny_sigma_clustered_keys(sigma):
    """Small perturbations cluster the duration differences within a few ulps: many equal
    d values and equal-gain runs (some longer than 64 -> general path), 32-bit key bins of
    more than 256 entries (finer sub-ranges), single-valued bins (streamed)."""
    w = workloads.config("c2")
    _replica_check(w, 40, 3, [0, 1, 20, 39], sigma=sigma)


def test_replicas_two_arch_mixed_one_arch_tasks():
    """Two archs with CPU-only tasks (sparse-QR ASM, FMM P2M/M2M/L2L/L2P): d = +-inf classes."""
    a = workloads.sparse_tree(12, 64, 32)
    b = workloads.fmm_tree(5, 1 << 12, 3)
    w = workloads.union(a, b, "mixed")
    assert w.n < 65536 and (~np.isfinite(w.dur[:, 1])).any()
    _replica_check(w, 40, 1000, range(40))


def test_replicas_two_arch_gpu_only_tasks_and_hd_zero():
    w = workloads.config("c1")
    dur = w.dur.copy()
    dur[::3, 0] = np.inf                       # GPU-only tasks
    W = workloads.Workload("g", w.n, w.src, w.dst, dur, w.arch_names, w.workers)
    _replica_check(W, 64, 0, range(64))
    eq = np.ones_like(w.dur)                   # equal durations -> d = 0, hd = 0 -> gain 0.5
    W2 = workloads.Workload("eq", w.n, w.src, w.dst, eq, w.arch_names, w.workers)
    _replica_check(W2, 8, 0, range(8), sigma=0.0)


# ----------------------------------------------------------------------------
# N1: incremental READY-mode push
# ----------------------------------------------------------------------------

@pytest.mark.parametrize("name,A,steps", [("c1", 2, 12), ("c2", 2, 25), ("qr", 3, 20)])
def test_ready_push_sequence_equals_ready_rebuild(name, A, steps):
    w = workloads.qr(10) if name == "qr" else workloads.config(name)
    dag = mp.build_dag(w.n, to_dev(w.src, torch.int32), to_dev(w.dst, torch.int32))
    dur = to_dev(w.dur)
    full = mp.score_and_queue(dag, dur, w.workers)
    key, flags = full["key"], full["flags"]
    od = oracle.build_dag(w.n, w.src, w.dst)
    ofull = oracle.score_and_queue(od, w.dur, w.workers)      # oracle inputs come from the oracle
    okey, oflags = ofull["key"], ofull["flags"]
    done = np.zeros(w.n, np.uint8)
    qptr, qtask, summ = mp.build_queues(dag, key, flags, dur, done=to_dev(done))
    rem = mp.ready_init(dag)
    rng = np.random.default_rng(3)
    for step in range(steps):
        qp = qptr.cpu().numpy()
        qt = qtask.cpu().numpy()
        ready = np.unique(qt[:qp[-1]])
        if len(ready) == 0:
            break
        k = int(rng.integers(1, min(len(ready), 200) + 1))
        batch = rng.choice(ready, k, replace=False).astype(np.int32)
        done[batch] = 1
        qptr, qtask, summ = mp.queues_push(dag, key, flags, dur, to_dev(batch), rem, qptr, qtask)
        mp.check(dag)
        oq_ptr, oq, osum = oracle.build_queues(od, okey, oflags, w.dur, done)
        assert np.array_equal(qptr.cpu().numpy(), oq_ptr), step
        assert np.array_equal(qtask.cpu().numpy()[:oq_ptr[-1]], oq), step
        assert summ.cpu().numpy().tobytes() == osum.tobytes(), step


@pytest.mark.parametrize("name,A", [("c1", 2), ("c2", 2), ("qr", 3)])
def test_push_all_sequence_equals_ready_rebuild(name, A):
    """N1 static-order push (mp_queues_push_all): after every batch the queues equal
    the oracle's READY-mode rebuild, and the old merge push gives the same bytes."""
    w = workloads.qr(10) if name == "qr" else workloads.config(name)
    dag = mp.build_dag(w.n, to_dev(w.src, torch.int32), to_dev(w.dst, torch.int32))
    dur = to_dev(w.dur)
    full = mp.score_and_queue(dag, dur, w.workers)            # ALL-mode queues
    key, flags = full["key"], full["flags"]
    od = oracle.build_dag(w.n, w.src, w.dst)
    ofull = oracle.score_and_queue(od, w.dur, w.workers)
    okey, oflags = ofull["key"], ofull["flags"]
    done_h = np.zeros(w.n, np.uint8)
    done_d = torch.zeros(w.n, dtype=torch.uint8, device=DEV)
    rem = mp.ready_init(dag)
    rem2 = mp.ready_init(dag)
    qptr, qtask, summ = mp.queues_push_all(dag, full["qptr"], full["qtask"], flags, dur,
                                           torch.zeros(0, dtype=torch.int32, device=DEV), rem, done_d)
    q2ptr, q2task, _ = mp.build_queues(dag, key, flags, dur, done=to_dev(done_h))
    rng = np.random.default_rng(11)
    steps = 0
    while True:
        mp.check(dag)
        oq_ptr, oq, osum = oracle.build_queues(od, okey, oflags, w.dur, done_h)
        assert np.array_equal(qptr.cpu().numpy(), oq_ptr), steps
        assert np.array_equal(qtask.cpu().numpy()[:oq_ptr[-1]], oq), steps
        assert summ.cpu().numpy().tobytes() == osum.tobytes(), steps
        assert np.array_equal(q2task.cpu().numpy()[:oq_ptr[-1]], oq), steps
        ready = np.unique(oq)
        if len(ready) == 0:
            break
        k = int(rng.integers(1, min(len(ready), 300) + 1))
        batch = rng.choice(ready, k, replace=False).astype(np.int32)
        done_h[batch] = 1
        qptr, qtask, summ = mp.queues_push_all(dag, full["qptr"], full["qtask"], flags, dur, to_dev(batch), rem,
                                               done_d)
        q2ptr, q2task, _ = mp.queues_push(dag, key, flags, dur, to_dev(batch), rem2, q2ptr, q2task)
        steps += 1
    assert done_h.all() and steps > 0
    # a task completed twice is an argument error
    mp.queues_push_all(dag, full["qptr"], full["qtask"], flags, dur, to_dev(np.array([0], np.int32)), rem, done_d)
    with pytest.raises(mp.MPError):
        mp.check(dag)


@pytest.mark.parametrize("variant", ["merge", "all"])
def test_push_rejects_bad_batches_without_side_effects(variant):
    """N1 batch validation (mp.h): a task listed twice in one batch, a task with its
    still-pending predecessor in the same batch, and a task completed in an earlier
    batch each raise MP_ERR_ARG and leave rem / done / the queues unchanged (no
    thread-timing dependence: the batch is validated before any state changes)."""
    w = workloads.config("c1")           # 0 -> {1, 2, 3}; 1 -> {4, 6, 8}
    dag = mp.build_dag(w.n, to_dev(w.src, torch.int32), to_dev(w.dst, torch.int32))
    dur = to_dev(w.dur)
    full = mp.score_and_queue(dag, dur, w.workers)
    key, flags = full["key"], full["flags"]
    rem = mp.ready_init(dag)
    done_d = torch.zeros(w.n, dtype=torch.uint8, device=DEV)
    empty = torch.zeros(0, dtype=torch.int32, device=DEV)
    q0ptr, q0, _ = mp.build_queues(dag, key, flags, dur, done=torch.zeros(w.n, dtype=torch.uint8, device=DEV))

    def push(batch, qp, qt):
        b = to_dev(np.array(batch, np.int32))
        if variant == "merge":
            return mp.queues_push(dag, key, flags, dur, b, rem, qp, qt)
        return mp.queues_push_all(dag, full["qptr"], full["qtask"], flags, dur, b, rem, done_d)

    if variant == "all":
        q0ptr, q0, _ = push([], None, None)
    mp.check(dag)
    qp, qt, _ = push([0], q0ptr, q0)                 # valid: task 0 completes
    mp.check(dag)
    rem_ok, done_ok = rem.clone(), done_d.clone()
    qp_ok, qt_ok = qp.clone(), qt.clone()
    for bad in ([1, 1], [1, 4], [0], [2, 99], [5]):   # duplicate, pred+succ, completed, out of range, not ready
        qp2, qt2, _ = push(bad, qp_ok, qt_ok)
        with pytest.raises(mp.MPError) as e:
            mp.check(dag)
        assert e.value.code == mp.MP_ERR_ARG, bad
        assert torch.equal(rem, rem_ok), bad
        assert torch.equal(done_d, done_ok), bad
        if variant == "merge":
            Q = int(qp_ok[-1])
            assert torch.equal(qp2, qp_ok) and torch.equal(qt2[:Q], qt_ok[:Q]), bad
    qp3, qt3, _ = push([1, 2, 3], qp_ok, qt_ok)       # still usable after the rejections
    mp.check(dag)
    od = oracle.build_dag(w.n, w.src, w.dst)
    o = oracle.score_and_queue(od, w.dur, w.workers)
    done = np.zeros(w.n, np.uint8)
    done[[0, 1, 2, 3]] = 1
    oqp, oq, _ = oracle.build_queues(od, o["key"], o["flags"], w.dur, done)
    assert np.array_equal(qp3.cpu().numpy(), oqp) and np.array_equal(qt3.cpu().numpy()[:oqp[-1]], oq)


# ----------------------------------------------------------------------------
# randomised sweep: many small DAGs, 1-4 archs, masks, ties, duplicates, both criticalities
# ----------------------------------------------------------------------------

def test_random_sweep_single_dag_and_replicas():
    rng = np.random.default_rng(2024)
    for case in range(40):
        n = int(rng.integers(1, 3000))
        A = int(rng.integers(1, 5))
        src, dst = random_dags.random_dag(n, float(rng.uniform(0.0, 4.0)), case, dup=float(rng.uniform(0, 0.5)),
                                          max_span=int(rng.integers(1, 200)))
        dur = random_dags.dyadic_durations(n, A, case, p_inf=float(rng.uniform(0, 0.5)) if A > 1 else 0.0,
                                           tiny_set=bool(rng.integers(0, 2)))
        if rng.random() < 0.2:
            dur[rng.random((n, A)) < 0.1] = 0.0
            dur[np.all(~np.isfinite(dur), 1)] = 1.0
        workers = np.ones(A, np.int32)
        if A > 1 and rng.random() < 0.2:
            workers[int(rng.integers(0, A))] = 0
            en = np.isfinite(dur) & (workers[None, :] > 0)
            dur[~en.any(1), int(np.argmax(workers))] = 2.0
        kind = oracle.CRIT_NOD if rng.random() < 0.3 else oracle.CRIT_BL
        compare(n, src, dst, dur, workers, kind=kind)
        W = workloads.Workload(f"r{case}", n, src, dst, dur, tuple(f"a{i}" for i in range(A)), workers)
        R = int(rng.integers(1, 70))
        _replica_check(W, R, int(rng.integers(0, 10000)), sorted(set([0, R - 1, R // 2])),
                       sigma=float(rng.choice([0.0, 0.0625, 0.125, 0.25])), seed=int(rng.integers(0, 2**62)))


@pytest.mark.parametrize("name", ["c1", "c2", "c4fmm", "hier"])
def test_score_path_cuda_graph_replay(name):
    """The single-DAG score path has no host state across calls (device-side sort / scan
    epochs), so bench.py captures it in a CUDA graph: every replay must give the oracle's
    bytes (k_bl_small / k_bl_wide / k_bl_flow, the queue sort, the scans)."""
    w = workloads.config(name)
    dag = mp.build_dag(w.n, to_dev(w.src, torch.int32), to_dev(w.dst, torch.int32))
    dur = to_dev(w.dur)
    n, A = w.dur.shape
    o = dict(bl=dict(bl=torch.empty(n, dtype=torch.float32, device=DEV), cp=torch.empty(1, dtype=torch.float32, device=DEV),
                     nod=None),
             aff=dict(gain=torch.empty((n, A), dtype=torch.float32, device=DEV), hd=torch.empty(A, dtype=torch.float32, device=DEV),
                      flags=torch.empty((n, A), dtype=torch.uint8, device=DEV)),
             sc=dict(crit_norm=torch.empty(n, dtype=torch.float32, device=DEV), key=torch.empty((n, A), dtype=torch.int64, device=DEV)),
             q=dict(qptr=torch.empty(A + 1, dtype=torch.int64, device=DEV), qtask=torch.empty(n * A, dtype=torch.int32, device=DEV),
                    summary=torch.empty(A * mp.SUMMARY_BYTES, dtype=torch.uint8, device=DEV)))

    def step():
        bl, cp, _ = mp.bottom_level(dag, dur, w.workers, out=o["bl"])
        gain, hd, flags = mp.affinity(dag, dur, w.workers, out=o["aff"])
        cn, key = mp.score(dag, 0, bl, gain, flags, out=o["sc"])
        mp.build_queues(dag, key, flags, dur, out=o["q"])

    for _ in range(2):
        step()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        step()
    od = oracle.build_dag(w.n, w.src, w.dst)
    ref = oracle.score_and_queue(od, w.dur, w.workers)
    Q = int(ref["qptr"][-1])
    for _ in range(3):
        o["q"]["qtask"].fill_(-1)
        g.replay()
        torch.cuda.synchronize()
        mp.check(dag)
        assert np.array_equal(bits(o["bl"]["bl"].cpu().numpy()), bits(ref["bl"]))
        assert np.array_equal(o["q"]["qptr"].cpu().numpy(), ref["qptr"])
        assert np.array_equal(o["q"]["qtask"].cpu().numpy()[:Q], ref["qtask"])
        assert o["q"]["summary"].cpu().numpy().tobytes() == ref["summary"].tobytes()
