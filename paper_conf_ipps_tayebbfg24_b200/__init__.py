"""MultiPrio scoring and queue build on B200 -- Python binding of libmp.

Same names as the C-ABI (include/mp.h); each function marshals torch CUDA
tensors into device pointers plus the current CUDA stream and calls libmp.
Every step of the path runs in libmp's sm_100a kernels; PyTorch only
allocates device memory and provides the stream.  There is no CPU fallback:
a missing libmp.so or a non-CUDA tensor raises.

Paper: Tayeb, Bramas, Faverge, Guermouche, "Dynamic Tasks Scheduling with
Multiple Priorities on Heterogeneous Computing Systems" (IPDPS'24).
"""
from __future__ import annotations

import ctypes as C

import numpy as np
import torch

from . import _lib
from ._lib import (MP_CRIT_BOTTOM_LEVEL, MP_CRIT_NOD, MP_ERR_ARG, MP_ERR_CUDA, MP_ERR_CYCLE,  # noqa: F401
                   MP_ERR_DOMAIN, MP_ERR_NOMEM, MP_OK, MP_WEIGHT_MEAN, MP_WEIGHT_MIN, MPError)

SUMMARY_DTYPE = np.dtype([("count", "<i4"), ("head", "<i4"), ("brw_lo", "<u8"), ("brw_hi", "<i8"),
                          ("brw", "<f8")])
SUMMARY_BYTES = 32


def _ptr(t):
    if t is None:
        return None
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError("libmp takes CUDA tensors (there is no CPU path)")
    if not t.is_contiguous():
        raise ValueError("tensor must be contiguous")
    return C.c_void_p(t.data_ptr())


def _stream():
    return C.c_void_p(torch.cuda.current_stream().cuda_stream)


def _workers(workers, A):
    w = np.ascontiguousarray(np.asarray(workers, dtype=np.int32).reshape(-1))
    if w.size != A:
        raise ValueError(f"workers must have {A} entries")
    return w, w.ctypes.data_as(C.c_void_p)


class Dag:
    """Owning wrapper of an mp_dag handle."""

    def __init__(self, handle, device):
        self._h = handle
        self.device = device
        info = _lib.mp_dag_info()
        _lib.check(_lib.lib().mp_dag_get_info(self._h, C.byref(info)), "mp_dag_get_info")
        self.n = info.n_tasks
        self.n_edges = info.n_edges
        self.n_levels = info.n_levels
        self.max_width = info.max_width
        self._info = info

    @property
    def handle(self):
        if self._h is None:
            raise RuntimeError("DAG already freed")
        return self._h

    def arrays(self) -> dict:
        """Copies of the handle's CSR / level arrays (torch, on the device)."""
        i = self._info
        n, E, L = self.n, self.n_edges, self.n_levels

        def view(ptr, count):
            out = torch.empty(max(count, 0), dtype=torch.int32, device=self.device)
            if count > 0:
                _copy_dev(out, ptr, count * 4)
            return out

        return dict(row_ptr=view(i.d_row_ptr, n + 1), col=view(i.d_col, E), indeg=view(i.d_indeg, n),
                    level=view(i.d_level, n), level_ptr=view(i.d_level_ptr, L + 1),
                    level_order=view(i.d_level_order, n))

    def refresh(self):
        info = _lib.mp_dag_info()
        _lib.check(_lib.lib().mp_dag_get_info(self._h, C.byref(info)), "mp_dag_get_info")
        self.n, self.n_edges, self.n_levels, self.max_width = (info.n_tasks, info.n_edges, info.n_levels,
                                                               info.max_width)
        self._info = info

    def free(self):
        if self._h is not None:
            _lib.lib().mp_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


_cudart = None


def _copy_dev(dst: torch.Tensor, src_ptr: int, nbytes: int):
    """Device-to-device copy from a raw libmp pointer into a torch tensor."""
    global _cudart
    if _cudart is None:
        from cuda.bindings import runtime as _rt  # cuda-python
        _cudart = _rt
    err, = _cudart.cudaMemcpyAsync(dst.data_ptr(), src_ptr, nbytes,
                                   _cudart.cudaMemcpyKind.cudaMemcpyDeviceToDevice,
                                   torch.cuda.current_stream().cuda_stream)
    if int(err) != 0:
        raise RuntimeError(f"cudaMemcpyAsync failed: {err}")


def build_dag(n_tasks: int, src: torch.Tensor, dst: torch.Tensor) -> Dag:
    """a1+a2 (mp_build_dag): deduplicated successor CSR + topological levels."""
    src = src.to(torch.int32).contiguous()
    dst = dst.to(torch.int32).contiguous()
    h = C.c_void_p()
    m = src.numel()
    rc = _lib.lib().mp_build_dag(int(n_tasks), m, _ptr(src) if m else None, _ptr(dst) if m else None,
                                 _stream(), C.byref(h))
    _lib.check(rc, "mp_build_dag")
    return Dag(h, src.device)


def dag_rebuild(dag: Dag, n_tasks: int, src: torch.Tensor, dst: torch.Tensor) -> Dag:
    """mp_dag_rebuild: ingest a new edge list into an existing handle, reusing its buffers."""
    src = src.to(torch.int32).contiguous()
    dst = dst.to(torch.int32).contiguous()
    m = src.numel()
    try:
        rc = _lib.lib().mp_dag_rebuild(dag.handle, int(n_tasks), m, _ptr(src) if m else None,
                                       _ptr(dst) if m else None, _stream())
        _lib.check(rc, "mp_dag_rebuild")
    finally:
        dag.refresh()                   # on error the handle holds an empty DAG
    return dag


def check(dag: Dag):
    """Synchronise the stream and raise on a device-detected error (mp_check)."""
    _lib.check(_lib.lib().mp_check(dag.handle, _stream()), "mp_check")


def bottom_level(dag: Dag, dur: torch.Tensor, workers, nod: bool = False, out=None):
    """a3+a4(+a5) (mp_bottom_level) -> (bl[n], cp[1], nod[n][A] or None)."""
    n, A = dur.shape
    w, wp = _workers(workers, A)
    dev = dur.device
    if out is None:
        out = dict(bl=torch.empty(n, dtype=torch.float32, device=dev),
                   cp=torch.empty(1, dtype=torch.float32, device=dev),
                   nod=torch.empty((n, A), dtype=torch.float32, device=dev) if nod else None)
    rc = _lib.lib().mp_bottom_level(dag.handle, A, _ptr(dur), wp, _ptr(out["bl"]), _ptr(out["cp"]),
                                    _ptr(out["nod"]) if out.get("nod") is not None else None, _stream())
    _lib.check(rc, "mp_bottom_level")
    return out["bl"], out["cp"], out.get("nod")


def bottom_level_w(dag: Dag, dur: torch.Tensor, workers, kind: int = MP_WEIGHT_MIN, out=None):
    """N4 (mp_bottom_level_w): bottom-level with node weight min (c2) or HEFT mean cost (v1) -> (bl, cp)."""
    n, A = dur.shape
    w, wp = _workers(workers, A)
    dev = dur.device
    if out is None:
        out = dict(bl=torch.empty(n, dtype=torch.float32, device=dev),
                   cp=torch.empty(1, dtype=torch.float32, device=dev))
    rc = _lib.lib().mp_bottom_level_w(dag.handle, A, _ptr(dur), wp, int(kind), _ptr(out["bl"]), _ptr(out["cp"]),
                                      _stream())
    _lib.check(rc, "mp_bottom_level_w")
    return out["bl"], out["cp"]


def affinity_prefix(dag: Dag, dur: torch.Tensor, workers, order: torch.Tensor | None = None, out=None):
    """N4 (mp_affinity_prefix): gains with hd as a running max along the push order -> (gain, hd, flags)."""
    n, A = dur.shape
    w, wp = _workers(workers, A)
    dev = dur.device
    if out is None:
        out = dict(gain=torch.empty((n, A), dtype=torch.float32, device=dev),
                   hd=torch.empty(A, dtype=torch.float32, device=dev),
                   flags=torch.empty((n, A), dtype=torch.uint8, device=dev))
    o = None if order is None else order.to(torch.int32).contiguous()
    rc = _lib.lib().mp_affinity_prefix(dag.handle, A, _ptr(dur), wp, _ptr(o), _ptr(out["gain"]), _ptr(out["hd"]),
                                       _ptr(out["flags"]), _stream())
    _lib.check(rc, "mp_affinity_prefix")
    return out["gain"], out["hd"], out["flags"]


def nod_remaining(dag: Dag, dur: torch.Tensor, workers, done: torch.Tensor, out=None):
    """N4 (mp_nod_remaining): NOD on the remaining graph (done tasks removed) -> nod[n][A]."""
    n, A = dur.shape
    w, wp = _workers(workers, A)
    if out is None:
        out = torch.empty((n, A), dtype=torch.float32, device=dur.device)
    rc = _lib.lib().mp_nod_remaining(dag.handle, A, _ptr(dur), wp, _ptr(done.to(torch.uint8).contiguous()),
                                     _ptr(out), _stream())
    _lib.check(rc, "mp_nod_remaining")
    return out


def affinity(dag: Dag, dur: torch.Tensor, workers, out=None):
    """a6 (mp_affinity) -> (gain[n][A], hd[A], flags[n][A] uint8)."""
    n, A = dur.shape
    w, wp = _workers(workers, A)
    dev = dur.device
    if out is None:
        out = dict(gain=torch.empty((n, A), dtype=torch.float32, device=dev),
                   hd=torch.empty(A, dtype=torch.float32, device=dev),
                   flags=torch.empty((n, A), dtype=torch.uint8, device=dev))
    rc = _lib.lib().mp_affinity(dag.handle, A, _ptr(dur), wp, _ptr(out["gain"]), _ptr(out["hd"]),
                                _ptr(out["flags"]), _stream())
    _lib.check(rc, "mp_affinity")
    return out["gain"], out["hd"], out["flags"]


def score(dag: Dag, kind: int, crit: torch.Tensor, gain: torch.Tensor, flags: torch.Tensor, out=None):
    """a7 (mp_score) -> (crit_norm, key[n][A] uint64 as int64)."""
    n, A = gain.shape
    dev = gain.device
    if out is None:
        out = dict(crit_norm=torch.empty(n if kind == MP_CRIT_BOTTOM_LEVEL else (n, A), dtype=torch.float32,
                                         device=dev),
                   key=torch.empty((n, A), dtype=torch.int64, device=dev))
    rc = _lib.lib().mp_score(dag.handle, A, kind, _ptr(crit), _ptr(gain), _ptr(flags), _ptr(out["crit_norm"]),
                             _ptr(out["key"]), _stream())
    _lib.check(rc, "mp_score")
    return out["crit_norm"], out["key"]


def build_queues(dag: Dag, key: torch.Tensor, flags: torch.Tensor, dur: torch.Tensor, done=None, out=None):
    """a8+a9 (mp_build_queues) -> (qptr[A+1] int64, qtask[n*A] int32, summary bytes[A*32])."""
    n, A = key.shape
    dev = key.device
    if out is None:
        out = dict(qptr=torch.empty(A + 1, dtype=torch.int64, device=dev),
                   qtask=torch.empty(max(n * A, 1), dtype=torch.int32, device=dev),
                   summary=torch.empty(A * SUMMARY_BYTES, dtype=torch.uint8, device=dev))
    rc = _lib.lib().mp_build_queues(dag.handle, A, _ptr(key), _ptr(flags), _ptr(dur),
                                    _ptr(done) if done is not None else None, _ptr(out["qptr"]),
                                    _ptr(out["qtask"]), _ptr(out["summary"]), _stream())
    _lib.check(rc, "mp_build_queues")
    return out["qptr"], out["qtask"], out["summary"]


def replicas_run(dag: Dag, base_dur: torch.Tensor, workers, seed: int, sigma: float, r0: int, R: int,
                 want_queues: bool = True, out=None):
    """a10 (mp_replicas_run) -> (cp[R], summary bytes[R*A*32], qtask[R][n*A] or None)."""
    n, A = base_dur.shape
    w, wp = _workers(workers, A)
    dev = base_dur.device
    if out is None:
        out = dict(cp=torch.empty(max(R, 1), dtype=torch.float32, device=dev),
                   summary=torch.empty(max(R, 1) * A * SUMMARY_BYTES, dtype=torch.uint8, device=dev),
                   qtask=torch.empty((max(R, 1), n * A), dtype=torch.int32, device=dev) if want_queues else None)
    rc = _lib.lib().mp_replicas_run(dag.handle, A, _ptr(base_dur), wp, C.c_uint64(seed), C.c_float(sigma), int(r0),
                                    int(R), _ptr(out["cp"]), _ptr(out["summary"]),
                                    _ptr(out["qtask"]) if out.get("qtask") is not None else None, _stream())
    _lib.check(rc, "mp_replicas_run")
    return out["cp"], out["summary"], out.get("qtask")


def ready_init(dag: Dag, rem: torch.Tensor = None) -> torch.Tensor:
    """mp_ready_init: per-task count of predecessors not completed yet (int32[n])."""
    if rem is None:
        rem = torch.empty(max(dag.n, 1), dtype=torch.int32, device=dag.device)
    _lib.check(_lib.lib().mp_ready_init(dag.handle, _ptr(rem), _stream()), "mp_ready_init")
    return rem


def queues_push(dag: Dag, key: torch.Tensor, flags: torch.Tensor, dur: torch.Tensor, batch: torch.Tensor,
                rem: torch.Tensor, qptr_in: torch.Tensor, qtask_in: torch.Tensor, out=None):
    """mp_queues_push (N1): pop+complete `batch`, push the newly ready tasks -> (qptr, qtask, summary)."""
    n, A = key.shape
    dev = key.device
    batch = batch.to(torch.int32).contiguous()
    if out is None:
        out = dict(qptr=torch.empty(A + 1, dtype=torch.int64, device=dev),
                   qtask=torch.empty(max(n * A, 1), dtype=torch.int32, device=dev),
                   summary=torch.empty(A * SUMMARY_BYTES, dtype=torch.uint8, device=dev))
    m = batch.numel()
    rc = _lib.lib().mp_queues_push(dag.handle, A, _ptr(key), _ptr(flags), _ptr(dur), _ptr(batch) if m else None, m,
                                   _ptr(rem), _ptr(qptr_in), _ptr(qtask_in), _ptr(out["qptr"]), _ptr(out["qtask"]),
                                   _ptr(out["summary"]), _stream())
    _lib.check(rc, "mp_queues_push")
    return out["qptr"], out["qtask"], out["summary"]


SIM_STATS_DTYPE = np.dtype([("makespan", "<f8"), ("pops", "<i8"), ("evictions", "<i8"), ("dups", "<i8"),
                            ("rounds", "<i8"), ("moved", "<i8"), ("busy", "<f8", (8,)), ("ran", "<i4", (8,))])
SIM_STATS_BYTES = 144


class DataModel:
    """N3 data model on the device: per-task accesses (CSR) and handle sizes (bytes)."""

    def __init__(self, acc_ptr, acc_handle, acc_mode, size, device="cuda"):
        self.acc_ptr = torch.as_tensor(np.asarray(acc_ptr, np.int64)).to(device)
        self.acc_handle = torch.as_tensor(np.asarray(acc_handle, np.int32)).to(device)
        self.acc_mode = torch.as_tensor(np.asarray(acc_mode, np.uint8)).to(device)
        self.size = torch.as_tensor(np.asarray(size, np.uint64).view(np.int64)).to(device)
        self.n_handles = int(self.size.numel())


def simulate(dag: Dag, base_dur: torch.Tensor, workers, seed: int, sigma: float, r0: int, R: int,
             qtask: torch.Tensor, summary: torch.Tensor, max_tries: int = 16, eviction: bool = True,
             trace: bool = False, out=None, data: DataModel | None = None, top_n: int = 1, eps: float = 0.8,
             worker_node=None, xfer_ms_per_byte: float = 0.0):
    """N2/N3 (mp_simulate_cfg): PUSH/POP simulation of R instances -> (stats bytes[R*144], start, worker).

    qtask/summary: the ALL-mode queues of mp_replicas_run ([R][n*A], [R*A*32])
    or, for one DAG (R=1, r0=0, sigma=0), of mp_build_queues.  data/top_n/eps/
    worker_node/xfer_ms_per_byte: N3 data locality (P:l.205-212, l.238)."""
    n, A = base_dur.shape
    w, wp = _workers(workers, A)
    dev = base_dur.device
    if out is None:
        out = dict(stats=torch.empty(max(R, 1) * SIM_STATS_BYTES, dtype=torch.uint8, device=dev),
                   start=torch.empty((max(R, 1), n), dtype=torch.float64, device=dev) if trace else None,
                   worker=torch.empty((max(R, 1), n), dtype=torch.int32, device=dev) if trace else None)
    wn = None if worker_node is None else np.ascontiguousarray(np.asarray(worker_node, np.int32))
    cfg = _lib.mp_sim_config(int(max_tries), int(bool(eviction)), int(top_n), float(eps),
                             0 if data is None else data.n_handles, 0,
                             None if data is None else _ptr(data.acc_ptr),
                             None if data is None or data.acc_handle.numel() == 0 else _ptr(data.acc_handle),
                             None if data is None or data.acc_mode.numel() == 0 else _ptr(data.acc_mode),
                             None if data is None or data.n_handles == 0 else _ptr(data.size),
                             None if wn is None else wn.ctypes.data_as(C.c_void_p), float(xfer_ms_per_byte))
    rc = _lib.lib().mp_simulate_cfg(dag.handle, A, _ptr(base_dur), wp, C.c_uint64(seed), C.c_float(sigma),
                                    int(r0), int(R), _ptr(qtask), _ptr(summary), C.byref(cfg), _ptr(out["stats"]),
                                    _ptr(out.get("start")), _ptr(out.get("worker")), _stream())
    _lib.check(rc, "mp_simulate_cfg")
    return out["stats"], out.get("start"), out.get("worker")


def sim_stats(stats_bytes: torch.Tensor) -> np.ndarray:
    """Host view of mp_sim_stats records."""
    return stats_bytes.detach().cpu().numpy().view(SIM_STATS_DTYPE)


def replicas_simulate(dag: Dag, base_dur: torch.Tensor, workers, seed: int, sigma: float, r0: int, R: int,
                      max_tries: int = 16, eviction: bool = True, trace: bool = False, **loc):
    """a10 queues of R replicas (mp_replicas_run), then their simulation (mp_simulate_cfg).
    loc: data / top_n / eps / worker_node / xfer_ms_per_byte (N3)."""
    cp, summ, q = replicas_run(dag, base_dur, workers, seed, sigma, r0, R, want_queues=True)
    st, start, worker = simulate(dag, base_dur, workers, seed, sigma, r0, R, q, summ, max_tries, eviction, trace,
                                 **loc)
    return dict(cp=cp, summary=summ, qtask=q, stats=st, start=start, worker=worker)


def queues_push_all(dag: Dag, qptr_all: torch.Tensor, qtask_all: torch.Tensor, flags: torch.Tensor,
                    dur: torch.Tensor, batch: torch.Tensor, rem: torch.Tensor, done: torch.Tensor, out=None):
    """mp_queues_push_all (N1, static order): complete `batch`, compact the ALL-mode queues
    to the READY-mode queues -> (qptr, qtask, summary).  `rem` (mp_ready_init) and `done`
    (uint8[n], zero at the start) are updated in place."""
    n, A = flags.shape
    dev = flags.device
    batch = batch.to(torch.int32).contiguous()
    if out is None:
        out = dict(qptr=torch.empty(A + 1, dtype=torch.int64, device=dev),
                   qtask=torch.empty(max(n * A, 1), dtype=torch.int32, device=dev),
                   summary=torch.empty(A * SUMMARY_BYTES, dtype=torch.uint8, device=dev))
    m = batch.numel()
    rc = _lib.lib().mp_queues_push_all(dag.handle, A, _ptr(qptr_all), _ptr(qtask_all), _ptr(flags), _ptr(dur),
                                       _ptr(batch) if m else None, m, _ptr(rem), _ptr(done), _ptr(out["qptr"]),
                                       _ptr(out["qtask"]), _ptr(out["summary"]), _stream())
    _lib.check(rc, "mp_queues_push_all")
    return out["qptr"], out["qtask"], out["summary"]


def summaries(summary_bytes: torch.Tensor) -> np.ndarray:
    """Host view of mp_queue_summary records."""
    return summary_bytes.detach().cpu().numpy().view(SUMMARY_DTYPE)


def score_and_queue(dag: Dag, dur: torch.Tensor, workers, kind: int = MP_CRIT_BOTTOM_LEVEL, done=None):
    """The whole single-DAG path a3..a9 on device tensors (async on the current stream)."""
    bl, cp, nod = bottom_level(dag, dur, workers, nod=(kind == MP_CRIT_NOD))
    gain, hd, flags = affinity(dag, dur, workers)
    crit = bl if kind == MP_CRIT_BOTTOM_LEVEL else nod
    crit_norm, key = score(dag, kind, crit, gain, flags)
    qptr, qtask, summ = build_queues(dag, key, flags, dur, done)
    return dict(bl=bl, cp=cp, nod=nod, gain=gain, hd=hd, flags=flags, crit_norm=crit_norm, key=key, qptr=qptr,
                qtask=qtask, summary=summ)


def build_info() -> str:
    return _lib.lib().mp_build_info().decode()


MB_SYNC, MB_CLUSTER, MB_GRID, MB_CHAIN = 0, 1, 2, 3


def microbench(kind: int, L: int, sink: torch.Tensor, arg: int = 0, chain: torch.Tensor | None = None):
    """mp_microbench: launch one per-level latency microkernel (L level boundaries of `kind`)
    on the current stream; the caller times it (bench.py's t_level)."""
    _lib.check(_lib.lib().mp_microbench(int(kind), int(L), int(arg), _ptr(chain) if chain is not None else None,
                                        _ptr(sink), _stream()), "mp_microbench")


def launch_count() -> int:
    """Kernels libmp has launched in this process (mp_launch_count)."""
    return int(_lib.lib().mp_launch_count())


def prof_enable(on: bool = True):
    _lib.lib().mp_prof_enable(1 if on else 0)


def prof_reset():
    _lib.lib().mp_prof_reset()


def prof_query(name: str):
    """(total device ms, launches) of kernel `name` since prof_reset (mp_prof_query)."""
    ms = C.c_double()
    cnt = C.c_int64()
    _lib.check(_lib.lib().mp_prof_query(name.encode(), C.byref(ms), C.byref(cnt)), "mp_prof_query")
    return ms.value, cnt.value


def prof_names() -> list:
    """Kernels timed since prof_reset (mp_prof_names)."""
    need = int(_lib.lib().mp_prof_names(None, 0))
    buf = C.create_string_buffer(need + 1)
    _lib.lib().mp_prof_names(buf, need + 1)
    return [x for x in buf.value.decode().split(",") if x]
