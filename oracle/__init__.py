"""CPU oracle for the MultiPrio scoring / queue-build hot path.

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / `--impl reference` legs may import this package.  The product
path (paper_conf_ipps_tayebbfg24_b200) never imports it and shares no code
with it; see mp_oracle.c for the per-function paper citations.

This module is argument marshalling only: it compiles mp_oracle.c with gcc
(-O2 -ffp-contract=off, no fast-math) into oracle/liboracle.so and calls it
through ctypes on numpy arrays.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "mp_oracle.c")
_SIM_SRC = os.path.join(_HERE, "mp_sim_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

OK, ERR_ARG, ERR_CYCLE, ERR_DOMAIN, ERR_NOMEM = 0, 1, 2, 3, 5
CRIT_BL, CRIT_NOD = 0, 1


class OracleError(RuntimeError):
    def __init__(self, code, where):
        super().__init__(f"oracle {where}: status {code}")
        self.code = code


SUMMARY_DTYPE = np.dtype([("count", "<i4"), ("head", "<i4"), ("brw_lo", "<u8"),
                          ("brw_hi", "<i8"), ("brw", "<f8")])


def build(force: bool = False) -> str:
    """Compile the oracle (plain C, single-threaded)."""
    srcs = [_SRC, _SIM_SRC]
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(map(os.path.getmtime, srcs)):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math",
                               "-fPIC", "-shared", "-o", tmp, *srcs, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        P = C.c_void_p
        i32, i64, u64, f32 = C.c_int32, C.c_int64, C.c_uint64, C.c_float
        _lib.or_build_dag.argtypes = [i32, i64, P, P, P, P, P, P, P, P, P, P]
        _lib.or_check_durations.argtypes = [i32, i32, P, P, P]
        _lib.or_bottom_level.argtypes = [i32, i32, P, P, P, P, P, P, P]
        _lib.or_nod.argtypes = [i32, i32, P, P, P, P, P]
        _lib.or_affinity.argtypes = [i32, i32, P, P, P, P, P]
        _lib.or_score.argtypes = [i32, i32, i32, P, P, P, P, P]
        _lib.or_build_queues.argtypes = [i32, i32, P, P, P, P, P, P, P, P, P]
        _lib.or_perturb.argtypes = [i32, i32, P, u64, f32, i64, P]
        _lib.or_perturb.restype = None
        _lib.or_replica.argtypes = [i32, i32, P, P, P, P, P, u64, f32, i64, P, P, P, P]
        _lib.or_bottom_level_w.argtypes = [i32, i32, P, P, P, P, P, i32, P, P]
        _lib.or_nod_remaining.argtypes = [i32, i32, P, P, P, P, P, P]
        _lib.or_affinity_prefix.argtypes = [i32, i32, P, P, P, P, P, P]
        _lib.or_simulate.argtypes = [i32, i32, P, P, P, P, P, P, P, P, P, P, P]
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


@dataclass
class Dag:
    n: int
    n_edges: int
    n_levels: int
    row_ptr: np.ndarray
    col: np.ndarray
    indeg: np.ndarray
    level: np.ndarray
    level_ptr: np.ndarray
    level_order: np.ndarray


def build_dag(n, src, dst) -> Dag:
    src = _c(src, np.int32)
    dst = _c(dst, np.int32)
    m = len(src)
    row_ptr = np.zeros(n + 1, np.int32)
    col = np.zeros(max(m, 1), np.int32)
    indeg = np.zeros(max(n, 1), np.int32)
    level = np.zeros(max(n, 1), np.int32)
    level_ptr = np.zeros(n + 1, np.int32)
    level_order = np.zeros(max(n, 1), np.int32)
    E = C.c_int64(0)
    L = C.c_int32(0)
    rc = lib().or_build_dag(n, m, _p(src), _p(dst), _p(row_ptr), _p(col), _p(indeg), _p(level),
                            _p(level_ptr), _p(level_order), C.byref(E), C.byref(L))
    if rc:
        raise OracleError(rc, "build_dag")
    return Dag(n, E.value, L.value, row_ptr, col[:E.value].copy(), indeg[:n], level[:n],
               level_ptr[:L.value + 1].copy(), level_order[:n])


def check_durations(dur, workers):
    dur = _c(dur, np.float32)
    n, A = dur.shape
    out = np.empty_like(dur)
    rc = lib().or_check_durations(n, A, _p(dur), _p(_c(workers, np.int32)), _p(out))
    if rc:
        raise OracleError(rc, "check_durations")
    return out


def bottom_level(dag: Dag, dur, workers):
    dur = _c(dur, np.float32)
    n, A = dur.shape
    bl = np.zeros(max(n, 1), np.float32)
    cp = np.zeros(1, np.float32)
    rc = lib().or_bottom_level(n, A, _p(dag.row_ptr), _p(dag.col if dag.n_edges else np.zeros(1, np.int32)),
                               _p(dag.level_order), _p(dur), _p(_c(workers, np.int32)), _p(bl), _p(cp))
    if rc:
        raise OracleError(rc, "bottom_level")
    return bl[:n], cp[0]


WEIGHT_MIN, WEIGHT_MEAN = 0, 1


def bottom_level_w(dag: Dag, dur, workers, wkind=WEIGHT_MIN):
    """N4: bottom-level with node weight min (c2) or HEFT mean cost (v1)."""
    dur = _c(dur, np.float32)
    n, A = dur.shape
    bl = np.zeros(max(n, 1), np.float32)
    cp = np.zeros(1, np.float32)
    rc = lib().or_bottom_level_w(n, A, _p(dag.row_ptr), _p(dag.col if dag.n_edges else np.zeros(1, np.int32)),
                                 _p(dag.level_order), _p(dur), _p(_c(workers, np.int32)), int(wkind), _p(bl), _p(cp))
    if rc:
        raise OracleError(rc, "bottom_level_w")
    return bl[:n], cp[0]


def nod_remaining(dag: Dag, dur, workers, done):
    """N4: NOD against the remaining graph (done tasks removed, v3)."""
    dur = _c(dur, np.float32)
    n, A = dur.shape
    out = np.zeros((max(n, 1), A), np.float32)
    rc = lib().or_nod_remaining(n, A, _p(dag.row_ptr), _p(dag.col if dag.n_edges else np.zeros(1, np.int32)),
                                _p(dur), _p(_c(workers, np.int32)), _p(_c(done, np.uint8)), _p(out))
    if rc:
        raise OracleError(rc, "nod_remaining")
    return out[:n]


def affinity_prefix(dur, workers, order=None):
    """N4: gains with hd(a) as the running max along the push order (v2)."""
    dur = _c(dur, np.float32)
    n, A = dur.shape
    gain = np.zeros((max(n, 1), A), np.float32)
    hd = np.zeros(A, np.float32)
    flags = np.zeros((max(n, 1), A), np.uint8)
    o = None if order is None else _c(order, np.int32)
    rc = lib().or_affinity_prefix(n, A, _p(dur), _p(_c(workers, np.int32)), _p(o), _p(gain), _p(hd), _p(flags))
    if rc:
        raise OracleError(rc, "affinity_prefix")
    return gain[:n], hd, flags[:n]


def nod(dag: Dag, dur, workers):
    dur = _c(dur, np.float32)
    n, A = dur.shape
    out = np.zeros((max(n, 1), A), np.float32)
    rc = lib().or_nod(n, A, _p(dag.row_ptr), _p(dag.col if dag.n_edges else np.zeros(1, np.int32)),
                      _p(dur), _p(_c(workers, np.int32)), _p(out))
    if rc:
        raise OracleError(rc, "nod")
    return out[:n]


def affinity(dur, workers):
    dur = _c(dur, np.float32)
    n, A = dur.shape
    gain = np.zeros((max(n, 1), A), np.float32)
    hd = np.zeros(A, np.float32)
    flags = np.zeros((max(n, 1), A), np.uint8)
    rc = lib().or_affinity(n, A, _p(dur), _p(_c(workers, np.int32)), _p(gain), _p(hd), _p(flags))
    if rc:
        raise OracleError(rc, "affinity")
    return gain[:n], hd, flags[:n]


def score(kind, crit, gain, flags):
    gain = _c(gain, np.float32)
    n, A = gain.shape
    crit = _c(crit, np.float32)
    flags = _c(flags, np.uint8)
    cn = np.zeros(max(n, 1) if kind == CRIT_BL else (max(n, 1), A), np.float32)
    key = np.zeros((max(n, 1), A), np.uint64)
    rc = lib().or_score(n, A, kind, _p(crit), _p(gain), _p(flags), _p(cn), _p(key))
    if rc:
        raise OracleError(rc, "score")
    return cn[:n], key[:n]


def build_queues(dag: Dag, key, flags, dur, done=None):
    key = _c(key, np.uint64)
    n, A = key.shape
    qptr = np.zeros(A + 1, np.int64)
    qtask = np.zeros(max(n * A, 1), np.int32)
    summ = np.zeros(A, SUMMARY_DTYPE)
    done_a = None if done is None else _c(done, np.uint8)
    rc = lib().or_build_queues(n, A, _p(dag.row_ptr), _p(dag.col if dag.n_edges else np.zeros(1, np.int32)),
                               _p(key), _p(_c(flags, np.uint8)), _p(_c(dur, np.float32)), _p(done_a),
                               _p(qptr), _p(qtask), _p(summ))
    if rc:
        raise OracleError(rc, "build_queues")
    return qptr, qtask[:qptr[-1]], summ


def perturb(base, seed, sigma, r):
    base = _c(base, np.float32)
    n, A = base.shape
    out = np.empty_like(base)
    lib().or_perturb(n, A, _p(base), seed, sigma, r, _p(out))
    return out


def replica(dag: Dag, base, workers, seed, sigma, r, want_queue=True):
    base = _c(base, np.float32)
    n, A = base.shape
    cp = np.zeros(1, np.float32)
    summ = np.zeros(A, SUMMARY_DTYPE)
    q = np.zeros(max(n * A, 1), np.int32) if want_queue else None
    qptr = np.zeros(A + 1, np.int64)
    rc = lib().or_replica(n, A, _p(dag.row_ptr), _p(dag.col if dag.n_edges else np.zeros(1, np.int32)),
                          _p(dag.level_order), _p(base), _p(_c(workers, np.int32)), seed, sigma, r,
                          _p(cp), _p(summ), _p(q), _p(qptr))
    if rc:
        raise OracleError(rc, "replica")
    return cp[0], summ, (q[:qptr[-1]] if want_queue else None), qptr


def score_and_queue(dag: Dag, dur, workers, kind=CRIT_BL, done=None):
    """The whole single-DAG path a3-a9 in the paper's order (convenience for tests/bench)."""
    bl, cp = bottom_level(dag, dur, workers)
    gain, hd, flags = affinity(dur, workers)
    crit = bl if kind == CRIT_BL else nod(dag, dur, workers)
    cn, key = score(kind, crit, gain, flags)
    dc = check_durations(dur, workers)
    qptr, qtask, summ = build_queues(dag, key, flags, dc, done)
    return dict(bl=bl, cp=cp, gain=gain, hd=hd, flags=flags, crit=crit, crit_norm=cn, key=key,
                qptr=qptr, qtask=qtask, summary=summ)


# --------------------------------------------------------------------------
# discrete-event MultiPrio simulation (mp_sim_oracle.c)
# --------------------------------------------------------------------------
SIM_STATS_DTYPE = np.dtype([("makespan", "<f8"), ("pops", "<i8"), ("evictions", "<i8"), ("dups", "<i8"),
                            ("rounds", "<i8"), ("moved", "<i8"), ("busy", "<f8", (8,)), ("ran", "<i4", (8,)),
                            ("stale", "<i8")])
SIM_ERR_STUCK = 6


class _SimCfg(C.Structure):
    _fields_ = [("max_tries", C.c_int32), ("eviction", C.c_int32), ("top_n", C.c_int32), ("eps", C.c_float),
                ("n_handles", C.c_int32), ("n_nodes", C.c_int32), ("acc_ptr", C.c_void_p), ("acc_h", C.c_void_p),
                ("acc_mode", C.c_void_p), ("size", C.c_void_p), ("worker_node", C.c_void_p),
                ("xfer_ms_per_byte", C.c_double)]


@dataclass
class DataModel:
    """N3 data model: per-task accesses (CSR), handle sizes (bytes)."""
    acc_ptr: np.ndarray      # int64[n+1]
    acc_handle: np.ndarray   # int32[acc]
    acc_mode: np.ndarray     # uint8[acc]: 1 = R, 2 = W, 3 = RW
    size: np.ndarray         # uint64[H]


def simulate(dag: Dag, dur, workers, key, max_tries=16, eviction=True, trace=True, gain=None, data=None,
             top_n=1, eps=0.8, worker_node=None, xfer_ms_per_byte=0.0):
    """PUSH (Alg. 1) / POP (Alg. 2) simulation of one DAG instance.

    dur: canonical durations (check_durations / perturbed), key: the a7 keys
    that order the heaps, gain: eq. 1 gains (N3 epsilon filter), data: a
    DataModel (N3 LS_SDH^2 and residency).  Returns (stats record,
    start[n] or None, worker[n] or None)."""
    dur = _c(dur, np.float32)
    n, A = dur.shape
    key = _c(key, np.uint64).reshape(n, A)
    st = np.zeros(1, SIM_STATS_DTYPE)
    start = np.zeros(max(n, 1), np.float64) if trace else None
    worker = np.zeros(max(n, 1), np.int32) if trace else None
    indeg = _c(dag.indeg, np.int32) if n else np.zeros(1, np.int32)
    keep = []

    def arr(a, dt):
        if a is None:
            return None
        a = _c(a, dt)
        keep.append(a)
        return _p(a)

    cfg = _SimCfg(int(max_tries), int(bool(eviction)), int(top_n), float(eps),
                  0 if data is None else int(len(data.size)), 0,
                  None if data is None else arr(data.acc_ptr, np.int64),
                  None if data is None else arr(data.acc_handle, np.int32),
                  None if data is None else arr(data.acc_mode, np.uint8),
                  None if data is None else arr(data.size, np.uint64),
                  arr(worker_node, np.int32), float(xfer_ms_per_byte))
    g = None if gain is None else _c(gain, np.float32).reshape(n, A)
    rc = lib().or_simulate(n, A, _p(dag.row_ptr), _p(dag.col if dag.n_edges else np.zeros(1, np.int32)),
                           _p(indeg), _p(dur), _p(_c(workers, np.int32)), _p(key), _p(g), C.byref(cfg),
                           _p(st), _p(start), _p(worker))
    if rc:
        raise OracleError(rc, "simulate")
    return st[0], (start[:n] if trace else None), (worker[:n] if trace else None)


def simulate_dag(dag: Dag, dur, workers, max_tries=16, eviction=True, kind=CRIT_BL, trace=True, **loc):
    """Score the whole DAG (a3-a7), then simulate it (convenience for tests).
    loc: data / top_n / eps / worker_node / xfer_ms_per_byte (N3)."""
    r = score_and_queue(dag, dur, workers, kind=kind)
    dc = check_durations(dur, workers)
    return simulate(dag, dc, workers, r["key"], max_tries, eviction, trace, gain=r["gain"], **loc)


def simulate_replica(dag: Dag, base, workers, seed, sigma, r, max_tries=16, eviction=True, trace=True, **loc):
    """Replica r (a10 perturbation, BL criticality, ALL-mode scores), simulated."""
    d = check_durations(perturb(base, seed, sigma, r), workers)
    return simulate_dag(dag, d, workers, max_tries, eviction, CRIT_BL, trace, **loc)
