"""Small seeded random DAGs and duration tables for property / parity tests.

Input generators only -- no MultiPrio arithmetic.  Every generator returns raw
(src, dst) int32 edge lists (possibly with duplicates when `dup` > 0) whose
ids are randomly permuted so that id order is not a topological order.
"""
from __future__ import annotations

import numpy as np


def random_dag(n: int, avg_deg: float, seed: int, dup: float = 0.0, permute: bool = True,
               max_span: int | None = None):
    """Random DAG: edges u->v drawn with u < v in a hidden order, then ids permuted."""
    rng = np.random.default_rng(seed)
    if n < 2:
        return np.zeros(0, np.int32), np.zeros(0, np.int32)
    m = int(round(avg_deg * n))
    u = rng.integers(0, n - 1, m)
    if max_span is None:
        v = u + 1 + (rng.random(m) * (n - 1 - u)).astype(np.int64)
    else:
        v = np.minimum(u + 1 + rng.integers(0, max_span, m), n - 1)
    if dup > 0 and m > 0:
        k = int(dup * m)
        pick = rng.integers(0, m, k)
        u = np.concatenate([u, u[pick]])
        v = np.concatenate([v, v[pick]])
    perm = rng.permutation(n) if permute else np.arange(n)
    return perm[u].astype(np.int32), perm[v].astype(np.int32)


def layered_dag(widths, fan: int, seed: int):
    """Layered DAG with given level widths; each node gets up to `fan` preds from the previous layer."""
    rng = np.random.default_rng(seed)
    starts = np.concatenate([[0], np.cumsum(widths)])
    src, dst = [], []
    for l in range(1, len(widths)):
        a0, a1 = starts[l - 1], starts[l]
        for v in range(starts[l], starts[l + 1]):
            k = rng.integers(1, fan + 1)
            ps = rng.integers(a0, a1, k)
            src.extend(ps.tolist())
            dst.extend([v] * k)
    n = int(starts[-1])
    perm = rng.permutation(n)
    return n, perm[np.asarray(src, np.int64)].astype(np.int32), perm[np.asarray(dst, np.int64)].astype(np.int32)


def chain(n: int):
    s = np.arange(n - 1, dtype=np.int32)
    return s, s + 1


def star(n: int):
    """Root 0 -> leaves 1..n-1."""
    return np.zeros(n - 1, np.int32), np.arange(1, n, dtype=np.int32)


def dyadic_durations(n: int, A: int, seed: int, denom: int = 64, hi: int = 64,
                     p_inf: float = 0.0, tiny_set: bool = False):
    """Durations k/denom ms (exact in binary32 and in every partial sum we form).

    p_inf: probability that (t,a) cannot execute (+inf); each task keeps >= 1
    executable arch.  tiny_set: draw from {1,2,3}/4 to force ties.
    """
    rng = np.random.default_rng(seed)
    if tiny_set:
        d = rng.integers(1, 4, (n, A)).astype(np.float32) / 4.0
    else:
        d = rng.integers(1, hi * denom, (n, A)).astype(np.float32) / np.float32(denom)
    if p_inf > 0 and A > 1:
        mask = rng.random((n, A)) < p_inf
        keep = rng.integers(0, A, n)
        mask[np.arange(n), keep] = False
        d[mask] = np.inf
    return d.astype(np.float32)


def random_data_model(n: int, H: int, seed: int, max_acc: int = 3, max_size: int = 1 << 20):
    """Random N3 data model: each task accesses 0..max_acc distinct handles of
    [0, H) in mode R (1), W (2) or RW (3); sizes are integers in [1, max_size].
    Returns (acc_ptr int64[n+1], acc_handle int32[], acc_mode uint8[], size uint64[H])."""
    rng = np.random.default_rng(seed)
    k = rng.integers(0, max_acc + 1, n)
    ptr = np.zeros(n + 1, np.int64)
    ptr[1:] = np.cumsum(k)
    hs, ms = [], []
    for t in range(n):
        h = rng.choice(H, size=min(int(k[t]), H), replace=False)
        hs.append(h)
        ms.append(rng.integers(1, 4, len(h)))
    ptr[1:] = np.cumsum([len(h) for h in hs])
    acc_h = np.concatenate(hs).astype(np.int32) if n else np.zeros(0, np.int32)
    acc_m = np.concatenate(ms).astype(np.uint8) if n else np.zeros(0, np.uint8)
    size = rng.integers(1, max_size + 1, H).astype(np.uint64)
    return ptr, acc_h, acc_m, size
