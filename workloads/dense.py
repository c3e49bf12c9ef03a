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
