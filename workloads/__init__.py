"""Seeded synthetic workloads shaped like the paper's experiments (C1-C5).

This package is the ONLY code shared by the oracle side (tests) and the CUDA
side (tests, bench): it produces inputs -- edge lists and duration tables --
and holds none of the method's arithmetic (no bottom-levels, gains, scores,
queues, and not the replica perturbation, which each side implements on its
own).  Recipes: SURVEY.md §8(d) "Synthetic inputs" and Appendix B;
DESIGN.md §3 restates them.

Configs (BASELINE.json order):
  c1  tiled Cholesky 4x4, fixed durations                        (A=2)
  c2  tiled Cholesky 64x64, StarPU-like per-kernel model         (A=2)
  c3  tiled QR 128x128 (split diagonal), 3 resource types        (A=3)
  c4  sparse-QR-like tree (G=42) U FMM octree (H=8, 2^19 parts)  (A=2)
  c5  replicas of c2 (R=4096, sigma=1/8, seed 20240311)
  c4fmm  c4's FMM octree part alone (TBFMM-shaped)
  hier   N4: Cholesky with hierarchical tasks
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from . import dense, fmm, sparse_qr
from .stf import STFRecorder

INF = np.float32(np.inf)

# Duration models, ms, dyadic.  GEMM 20x slower on CPU
# matches "a matrix-matrix multiplication that is 20x slower on CPU"
# (§VII).
CHOL_MODEL = {  # (CPU, GPU)
    dense.POTRF: (6.0, 3.0),
    dense.TRSM: (12.0, 1.0),
    dense.SYRK: (12.0, 0.75),
    dense.GEMM: (30.0, 1.5),
}
QR_MODEL = {  # (CPU, GPU, ACC); inf = no implementation (PAPER.md l.91, l.135 can_exec)
    dense.GEQRT: (16.0, 4.0, np.inf),
    dense.TSQRT: (24.0, 4.0, np.inf),
    dense.UNMQR: (24.0, 2.0, 3.0),
    dense.TSMQR: (48.0, 3.0, 2.5),
}
SPQR_MODEL = {  # (CPU, GPU): QR tile kernels use the QR CPU/GPU columns; ASM is CPU-only
    sparse_qr.GEQRT: (16.0, 4.0),
    sparse_qr.TSQRT: (24.0, 4.0),
    sparse_qr.UNMQR: (24.0, 2.0),
    sparse_qr.TSMQR: (48.0, 3.0),
    sparse_qr.ASM: (0.125, np.inf),
}
# Hierarchical Cholesky: coarse tasks keep CHOL_MODEL; a
# fine sub-task (tile s = 2 times smaller: 1/8 of the flops) costs 1/8 on a CPU and, GPUs
# being far less efficient on small tiles, 4/8 of the coarse GPU time (reading h3) -- so the
# DAG mixes large GPU-friendly tasks with small CPU-friendly ones, as §VII describes.
HIER_MODEL = dict(CHOL_MODEL)
HIER_MODEL.update({
    dense.POTRF_F: (0.75, 1.5),
    dense.TRSM_F: (1.5, 0.5),
    dense.SYRK_F: (1.5, 0.375),
    dense.GEMM_F: (3.75, 0.75),
})
LU_MODEL = {  # (CPU, GPU), SURVEY §8(f) N4
    dense.GETRF: (12.0, 6.0),
    dense.TRSM_L: (12.0, 1.0),
    dense.TRSM_U: (12.0, 1.0),
    dense.GEMM_LU: (30.0, 1.5),
}

C5_SEED = 20240311
C5_SIGMA = 0.125
C5_REPLICAS = 4096


@dataclass
class Workload:
    name: str
    n: int
    src: np.ndarray          # int32[E_in] raw edges (duplicates allowed)
    dst: np.ndarray          # int32[E_in]
    dur: np.ndarray          # float32[n][A], +inf = cannot execute
    arch_names: tuple
    workers: np.ndarray      # int32[A], >0 enables the arch
    kind: np.ndarray | None = None
    meta: dict = field(default_factory=dict)
    # N3 data model (STF workloads): accesses per task and handle sizes in bytes
    acc_ptr: np.ndarray | None = None
    acc_handle: np.ndarray | None = None
    acc_mode: np.ndarray | None = None
    handle_size: np.ndarray | None = None

    @property
    def n_arch(self) -> int:
        return self.dur.shape[1]


def _table(kind: np.ndarray, model: dict) -> np.ndarray:
    kmax = max(model) + 1
    A = len(next(iter(model.values())))
    tab = np.full((kmax, A), np.inf, np.float32)
    for k, v in model.items():
        tab[k] = v
    return np.ascontiguousarray(tab[kind])


# tile of the paper's Chameleon runs: 960 x 960 doubles
TILE_BYTES = 960 * 960 * 8


def _from_stf(name, s: STFRecorder, model, arch_names, **meta) -> Workload:
    src, dst = s.edges()
    kind = s.kinds()
    dur = _table(kind, model)
    ap, ah, am = s.accesses()
    H = int(ah.max()) + 1 if len(ah) else 0
    return Workload(name, s.n, src, dst, dur, arch_names,
                    np.ones(dur.shape[1], np.int32), kind, dict(meta),
                    ap, ah, am, np.full(H, TILE_BYTES, np.uint64))


def cholesky(N: int) -> Workload:
    return _from_stf(f"cholesky{N}", dense.cholesky(N), CHOL_MODEL, ("CPU", "GPU"), tiles=N)


def qr(N: int, split_diag: bool = True) -> Workload:
    return _from_stf(f"qr{N}", dense.qr(N, split_diag), QR_MODEL, ("CPU", "GPU", "ACC"),
                     tiles=N, split_diag=split_diag)


def hier(N: int, s: int = 2, p_expand: float = 0.5, seed: int = 31) -> Workload:
    """Cholesky with hierarchical tasks (N4): N x N coarse tiles, expanded tasks at s x s
    sub-tiles (dense.hier_cholesky).  Durations: HIER_MODEL (defined for s = 2)."""
    assert s == 2, "HIER_MODEL's fine-task durations are defined for s = 2"
    return _from_stf(f"hier{N}", dense.hier_cholesky(N, s, p_expand, seed), HIER_MODEL, ("CPU", "GPU"),
                     tiles=N, split=s, p_expand=p_expand, seed=seed)


def lu(N: int) -> Workload:
    return _from_stf(f"lu{N}", dense.lu(N), LU_MODEL, ("CPU", "GPU"), tiles=N)


def sparse_tree(G: int = 42, leaf: int = 64, nb: int = 32) -> Workload:
    s, nfr = sparse_qr.sparse_qr_tree(G, leaf, nb)
    return _from_stf(f"spqr{G}", s, SPQR_MODEL, ("CPU", "GPU"), fronts=nfr, G=G, leaf=leaf, nb=nb)


def fmm_tree(H: int = 8, npart: int = 1 << 19, seed: int = 7) -> Workload:
    d = fmm.fmm_octree(H, npart, seed=seed)
    dur = np.stack([d["cpu_ms"], d["gpu_ms"]], 1).astype(np.float32)
    return Workload(f"fmm{H}", d["n"], d["src"], d["dst"], np.ascontiguousarray(dur), ("CPU", "GPU"),
                    np.ones(2, np.int32), d["kind"], dict(H=H, npart=npart, leaves=d["n_leaves"]))


def union(a: Workload, b: Workload, name: str) -> Workload:
    assert a.arch_names == b.arch_names
    off = np.int32(a.n)
    return Workload(name, a.n + b.n,
                    np.concatenate([a.src, b.src + off]), np.concatenate([a.dst, b.dst + off]),
                    np.ascontiguousarray(np.concatenate([a.dur, b.dur])), a.arch_names,
                    np.ones(a.n_arch, np.int32),
                    np.concatenate([a.kind, b.kind + 16]),
                    dict(parts={a.name: a.n, b.name: b.n}))


_CACHE: dict = {}


def config(name: str) -> Workload:
    """Return the named BASELINE config (c1..c5; c5 = the c2 DAG, replicas are a run option)."""
    name = name.lower()
    if name in _CACHE:
        return _CACHE[name]
    if name == "c1":
        w = cholesky(4)
    elif name in ("c2", "c5"):
        w = cholesky(64)
        if name == "c5":
            w.meta.update(replicas=C5_REPLICAS, sigma=C5_SIGMA, seed=C5_SEED)
    elif name == "c3":
        w = qr(128, split_diag=True)
    elif name == "c4":
        w = union(sparse_tree(42, 64, 32), fmm_tree(8, 1 << 19, 7), "c4")
    elif name == "c4fmm":       # c4's FMM part alone (the 13-level single-DAG case)
        w = fmm_tree(8, 1 << 19, 7)
    elif name == "hier":        # N4: hierarchical tasks (48 x 48 coarse tiles, half expanded)
        w = hier(48, 2, 0.5, 31)
    elif name == "lu64":
        w = lu(64)
    else:
        raise KeyError(name)
    w.name = name
    _CACHE[name] = w
    return w
