"""ctypes binding of libmp.so (include/mp.h).  Argument marshalling only.

Loads the in-tree libmp.so and fails loudly when it is missing: there is no
CPU fallback anywhere in the product path.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libmp.so")

MP_OK, MP_ERR_ARG, MP_ERR_CYCLE, MP_ERR_DOMAIN, MP_ERR_CUDA, MP_ERR_NOMEM = range(6)
MP_CRIT_BOTTOM_LEVEL, MP_CRIT_NOD = 0, 1
MP_WEIGHT_MIN, MP_WEIGHT_MEAN = 0, 1

EXPORTS = (
    "mp_build_dag", "mp_dag_rebuild", "mp_dag_get_info", "mp_bottom_level", "mp_affinity", "mp_score",
    "mp_build_queues", "mp_replicas_run", "mp_ready_init", "mp_queues_push", "mp_simulate", "mp_simulate_cfg",
    "mp_bottom_level_w", "mp_affinity_prefix", "mp_nod_remaining", "mp_queues_push_all",
    "mp_check", "mp_free", "mp_status_str", "mp_last_error", "mp_build_info", "mp_launch_count", "mp_prof_enable", "mp_prof_reset", "mp_prof_query", "mp_prof_names",
    "mp_microbench",
)


class MPError(RuntimeError):
    def __init__(self, code: int, where: str, detail: str):
        names = {0: "MP_OK", 1: "MP_ERR_ARG", 2: "MP_ERR_CYCLE", 3: "MP_ERR_DOMAIN", 4: "MP_ERR_CUDA",
                 5: "MP_ERR_NOMEM"}
        super().__init__(f"{where}: {names.get(code, code)}: {detail}")
        self.code = code


class mp_dag_info(C.Structure):
    _fields_ = [("n_tasks", C.c_int32), ("n_edges", C.c_int64), ("n_levels", C.c_int32),
                ("max_width", C.c_int32), ("d_row_ptr", C.c_void_p), ("d_col", C.c_void_p),
                ("d_indeg", C.c_void_p), ("d_level", C.c_void_p), ("d_level_ptr", C.c_void_p),
                ("d_level_order", C.c_void_p)]


class mp_sim_config(C.Structure):
    _fields_ = [("max_tries", C.c_int32), ("eviction", C.c_int32), ("top_n", C.c_int32), ("eps", C.c_float),
                ("n_handles", C.c_int32), ("n_nodes", C.c_int32), ("d_acc_ptr", C.c_void_p),
                ("d_acc_handle", C.c_void_p), ("d_acc_mode", C.c_void_p), ("d_size", C.c_void_p),
                ("h_worker_node", C.c_void_p), ("xfer_ms_per_byte", C.c_double)]


_lib = None


def lib():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"libmp.so not built ({LIB_PATH}); run `python -c 'import __graft_entry__ as g; "
                           f"g.build()'` -- there is no CPU fallback")
    L = C.CDLL(LIB_PATH)
    P, i32, i64, u64, f32 = C.c_void_p, C.c_int32, C.c_int64, C.c_uint64, C.c_float
    L.mp_build_dag.argtypes = [i32, i64, P, P, P, C.POINTER(P)]
    L.mp_dag_rebuild.argtypes = [P, i32, i64, P, P, P]
    L.mp_dag_get_info.argtypes = [P, C.POINTER(mp_dag_info)]
    L.mp_bottom_level.argtypes = [P, i32, P, P, P, P, P, P]
    L.mp_affinity.argtypes = [P, i32, P, P, P, P, P, P]
    L.mp_score.argtypes = [P, i32, C.c_int, P, P, P, P, P, P]
    L.mp_build_queues.argtypes = [P, i32, P, P, P, P, P, P, P, P]
    L.mp_replicas_run.argtypes = [P, i32, P, P, u64, f32, i64, i32, P, P, P, P]
    L.mp_ready_init.argtypes = [P, P, P]
    L.mp_queues_push.argtypes = [P, i32, P, P, P, P, i32, P, P, P, P, P, P, P]
    L.mp_simulate.argtypes = [P, i32, P, P, u64, f32, i64, i32, P, P, i32, i32, P, P, P, P]
    L.mp_simulate_cfg.argtypes = [P, i32, P, P, u64, f32, i64, i32, P, P, C.POINTER(mp_sim_config), P, P, P, P]
    L.mp_bottom_level_w.argtypes = [P, i32, P, P, C.c_int, P, P, P]
    L.mp_affinity_prefix.argtypes = [P, i32, P, P, P, P, P, P, P]
    L.mp_nod_remaining.argtypes = [P, i32, P, P, P, P, P]
    L.mp_queues_push_all.argtypes = [P, i32, P, P, P, P, P, i32, P, P, P, P, P, P]
    L.mp_check.argtypes = [P, P]
    L.mp_microbench.argtypes = [i32, i32, i32, P, P, P]
    L.mp_free.argtypes = [P]
    L.mp_free.restype = None
    L.mp_status_str.argtypes = [C.c_int]
    L.mp_status_str.restype = C.c_char_p
    L.mp_last_error.restype = C.c_char_p
    L.mp_build_info.restype = C.c_char_p
    L.mp_launch_count.restype = C.c_uint64
    L.mp_prof_enable.argtypes = [C.c_int]
    L.mp_prof_enable.restype = None
    L.mp_prof_reset.restype = None
    L.mp_prof_query.argtypes = [C.c_char_p, C.POINTER(C.c_double), C.POINTER(C.c_int64)]
    L.mp_prof_names.argtypes = [C.c_char_p, C.c_int64]
    L.mp_prof_names.restype = C.c_int64
    for name in EXPORTS:
        if name not in ("mp_free", "mp_status_str", "mp_last_error", "mp_build_info", "mp_dag_get_info",
                        "mp_launch_count", "mp_prof_enable", "mp_prof_reset", "mp_prof_names"):
            getattr(L, name).restype = C.c_int
    L.mp_dag_get_info.restype = C.c_int
    _lib = L
    return L


def check(rc: int, where: str):
    if rc != MP_OK:
        raise MPError(rc, where, lib().mp_last_error().decode())
