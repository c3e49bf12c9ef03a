"""Tiled dense linear-algebra DAGs recorded through the STF recorder.

Shapes follow the paper's Chameleon experiments (§VI-A:
potrf, getrf, geqrf over tiled matrices); recipes are SURVEY.md Appendix B.
Input generators only -- no MultiPrio arithmetic here.
"""
from __future__ import annotations

from .stf import STFRecorder

# kernel kinds (indices into the per-workload duration tables)
POTRF, TRSM, SYRK, GEMM = 0, 1, 2, 3
GEQRT, TSQRT, UNMQR, TSMQR = 0, 1, 2, 3
GETRF, TRSM_L, TRSM_U, GEMM_LU = 0, 1, 2, 3


def cholesky(N: int) -> STFRecorder:
    """Right-looking tiled Cholesky (lower), STF order of SURVEY App. A/B.

    Per k: POTRF(k); TRSM(k,i) for i>k; then for i>k: SYRK(k,i) followed by
    GEMM(k,i,j) for k<j<i.  Handles are tiles A[i][j].
    """
    s = STFRecorder()
    A = lambda i, j: i * N + j  # noqa: E731
    for k in range(N):
        s.submit(POTRF, writes=(A(k, k),))
        for i in range(k + 1, N):
            s.submit(TRSM, reads=(A(k, k),), writes=(A(i, k),))
        for i in range(k + 1, N):
            s.submit(SYRK, reads=(A(i, k),), writes=(A(i, i),))
            for j in range(k + 1, i):
                s.submit(GEMM, reads=(A(i, k), A(j, k)), writes=(A(i, j),))
    return s


def qr(N: int, split_diag: bool = True) -> STFRecorder:
    """Flat-tree tiled QR (Chameleon geqrf-like).

    GEQRT(k) RW A[k][k] (+ V[k] when split_diag); UNMQR(k,j) R V[k] (or
    A[k][k]) RW A[k][j]; TSQRT(k,i) RW A[k][k], A[i][k]; TSMQR(k,i,j)
    R A[i][k] RW A[k][j], A[i][j].  With split_diag the Householder
    reflectors of the diagonal tile live in a separate workspace V[k], which
    removes the UNMQR->TSQRT WAR edges (depth 3N-2 instead of 4N-3).
    """
    s = STFRecorder()
    A = lambda i, j: i * N + j  # noqa: E731
    V = lambda k: N * N + k  # noqa: E731
    for k in range(N):
        if split_diag:
            s.submit(GEQRT, writes=(A(k, k), V(k)))
        else:
            s.submit(GEQRT, writes=(A(k, k),))
        vk = V(k) if split_diag else A(k, k)
        for j in range(k + 1, N):
            s.submit(UNMQR, reads=(vk,), writes=(A(k, j),))
        for i in range(k + 1, N):
            s.submit(TSQRT, writes=(A(k, k), A(i, k)))
            for j in range(k + 1, N):
                s.submit(TSMQR, reads=(A(i, k),), writes=(A(k, j), A(i, j)))
    return s


def lu(N: int) -> STFRecorder:
    """Tiled LU without pivoting (getrf), SURVEY §8(f) N4 workload."""
    s = STFRecorder()
    A = lambda i, j: i * N + j  # noqa: E731
    for k in range(N):
        s.submit(GETRF, writes=(A(k, k),))
        for j in range(k + 1, N):
            s.submit(TRSM_L, reads=(A(k, k),), writes=(A(k, j),))
        for i in range(k + 1, N):
            s.submit(TRSM_U, reads=(A(k, k),), writes=(A(i, k),))
        for i in range(k + 1, N):
            for j in range(k + 1, N):
                s.submit(GEMM_LU, reads=(A(i, k), A(k, j)), writes=(A(i, j),))
    return s


# fine-granularity kernel kinds of the hierarchical Cholesky (sub-tasks of an expanded task)
POTRF_F, TRSM_F, SYRK_F, GEMM_F = 4, 5, 6, 7


def hier_cholesky(N: int, s: int = 2, p_expand: float = 0.5, seed: int = 31) -> STFRecorder:
    """Tiled Cholesky with hierarchical tasks (§VII:
    "hierarchical tasks ... submit subgraphs at runtime ... expos[ing] different task
    sizes in the DAG").  Reading h1: the matrix has N x N coarse tiles,
    each split into s x s fine tiles (the handles); a coarse task that is *expanded*
    (each independently with probability p_expand, seeded -- reading h2) submits, in its
    place, the fine-tile tasks of the same operation restricted to its tiles, in
    right-looking order; a task that is not expanded accesses every fine tile of its
    coarse tiles (the lower triangle of a diagonal tile).  Dependencies are then
    inferred by the STF rules at fine-tile granularity, so an expanded sub-graph
    inherits exactly the predecessors and successors of the data its sub-tasks touch.
    p_expand = 0 gives cholesky(N) (coarse tasks only); p_expand = 1 gives the same
    DAG as cholesky(N * s) (every task at fine granularity)."""
    import numpy as np
    rng = np.random.default_rng(seed)
    rec = STFRecorder()
    M = N * s
    F = lambda I, J: I * M + J  # noqa: E731  fine tile handle

    def tile(i, j):   # fine handles of coarse tile (i, j); lower triangle of a diagonal tile
        return tuple(F(I, J) for I in range(i * s, (i + 1) * s) for J in range(j * s, (j + 1) * s)
                     if i != j or I >= J)

    def expand():
        return p_expand >= 1.0 or (p_expand > 0.0 and rng.random() < p_expand)

    for k in range(N):
        K = range(k * s, (k + 1) * s)
        if expand():                                   # POTRF(k): fine Cholesky of tile (k, k)
            for Kf in K:
                rec.submit(POTRF_F, writes=(F(Kf, Kf),))
                for I in range(Kf + 1, (k + 1) * s):
                    rec.submit(TRSM_F, reads=(F(Kf, Kf),), writes=(F(I, Kf),))
                for I in range(Kf + 1, (k + 1) * s):
                    rec.submit(SYRK_F, reads=(F(I, Kf),), writes=(F(I, I),))
                    for J in range(Kf + 1, I):
                        rec.submit(GEMM_F, reads=(F(I, Kf), F(J, Kf)), writes=(F(I, J),))
        else:
            rec.submit(POTRF, writes=tile(k, k))
        for i in range(k + 1, N):
            Ii = range(i * s, (i + 1) * s)
            if expand():                               # TRSM(k, i): X L^T = B, column by column
                for Kf in K:
                    for I in Ii:
                        rec.submit(TRSM_F, reads=(F(Kf, Kf),), writes=(F(I, Kf),))
                    for J in range(Kf + 1, (k + 1) * s):
                        for I in Ii:
                            rec.submit(GEMM_F, reads=(F(I, Kf), F(J, Kf)), writes=(F(I, J),))
            else:
                rec.submit(TRSM, reads=tile(k, k), writes=tile(i, k))
        for i in range(k + 1, N):
            Ii = range(i * s, (i + 1) * s)
            if expand():                               # SYRK(k, i): A(i,i) -= A(i,k) A(i,k)^T
                for Kf in K:
                    for I in Ii:
                        rec.submit(SYRK_F, reads=(F(I, Kf),), writes=(F(I, I),))
                        for J in range(i * s, I):
                            rec.submit(GEMM_F, reads=(F(I, Kf), F(J, Kf)), writes=(F(I, J),))
            else:
                rec.submit(SYRK, reads=tile(i, k), writes=tile(i, i))
            for j in range(k + 1, i):
                if expand():                           # GEMM(k, i, j): A(i,j) -= A(i,k) A(j,k)^T
                    for Kf in K:
                        for I in Ii:
                            for J in range(j * s, (j + 1) * s):
                                rec.submit(GEMM_F, reads=(F(I, Kf), F(J, Kf)), writes=(F(I, J),))
                else:
                    rec.submit(GEMM, reads=tile(i, k) + tile(j, k), writes=tile(i, j))
    return rec
