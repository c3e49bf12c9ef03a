"""FMM octree task DAG (TBFMM-shaped), generated vectorised with numpy.

Shape source: PAPER.md l.263-270 (§VI-B, TBFMM: "the DAG of the TBFMM is very
disconnected, so the critical path with infinite resources is very short");
recipe: SURVEY.md Appendix B "FMM(H=8, 2^19, clusters, seed 7)".
Input generator only -- no MultiPrio arithmetic here.

Tasks (cell granularity, occupied cells only; leaves at level H-1):
  P2M, P2P, L2P per leaf; M2M at levels H-2..2; M2L at levels 2..H-1;
  L2L at levels 3..H-1.
Edges:
  up(child) -> M2M(parent)                 (up = P2M at leaves, M2M above)
  up(src)   -> M2L(tgt), src in IL(tgt)    (children of the parent's
                                            neighbours, not adjacent; <= 189)
  M2L(parent), L2L(parent) -> L2L(child)
  M2L(leaf), L2L(leaf), P2P(leaf) -> L2P(leaf)
Durations (ms, dyadic): P2M, L2P = np * 2^-10 (CPU only); M2M = 2^-4 *
children, L2L = 2^-4 (CPU only); M2L = |IL| * 2^-6 CPU, |IL| * 2^-9 GPU;
P2P = np * n_nbr * 2^-16 CPU, * 2^-20 GPU (n_nbr = particles in the 27-cell
neighbourhood, self included).
"""
from __future__ import annotations

import numpy as np

P2M, M2M, M2L, L2L, P2P, L2P = 0, 1, 2, 3, 4, 5
KIND_NAMES = ("P2M", "M2M", "M2L", "L2L", "P2P", "L2P")


def _split(code, side):
    z = code % side
    y = (code // side) % side
    x = code // (side * side)
    return x, y, z


def _join(x, y, z, side):
    return (x * side + y) * side + z


def _particles(npart, nclusters, seed):
    rng = np.random.default_rng(seed)
    centers = rng.random((nclusters, 3))
    sig = 10.0 ** rng.uniform(-2.3, -1.0, nclusters)
    lab = rng.integers(0, nclusters, npart)
    pts = centers[lab] + rng.standard_normal((npart, 3)) * sig[lab, None]
    return np.clip(pts, 0.0, np.nextafter(1.0, 0.0))


def fmm_octree(H: int = 8, npart: int = 1 << 19, nclusters: int = 64, seed: int = 7,
               uniform: bool = False):
    """Return dict(n, src, dst, kind, cpu_ms, gpu_ms) (gpu_ms = inf if CPU-only)."""
    leaf_lvl = H - 1
    if uniform:
        pts = np.random.default_rng(seed).random((npart, 3))
    else:
        pts = _particles(npart, nclusters, seed)
    side = 1 << leaf_lvl
    ijk = np.minimum((pts * side).astype(np.int64), side - 1)
    leaf_codes_all = _join(ijk[:, 0], ijk[:, 1], ijk[:, 2], side)
    leaf_codes, n_p = np.unique(leaf_codes_all, return_counts=True)

    # occupied cells per level (sorted codes)
    cells = {leaf_lvl: leaf_codes}
    for l in range(leaf_lvl - 1, 1, -1):
        s_child = 1 << (l + 1)
        x, y, z = _split(cells[l + 1], s_child)
        cells[l] = np.unique(_join(x >> 1, y >> 1, z >> 1, 1 << l))

    # ---- task id assignment (submission order) ----
    nxt = 0
    ids = {}

    def alloc(name, count):
        nonlocal nxt
        ids[name] = np.arange(nxt, nxt + count, dtype=np.int64)
        nxt += count

    alloc(("P2M", leaf_lvl), len(leaf_codes))
    for l in range(leaf_lvl - 1, 1, -1):
        alloc(("M2M", l), len(cells[l]))
    for l in range(2, leaf_lvl + 1):
        alloc(("M2L", l), len(cells[l]))
    for l in range(3, leaf_lvl + 1):
        alloc(("L2L", l), len(cells[l]))
    alloc(("P2P", leaf_lvl), len(leaf_codes))
    alloc(("L2P", leaf_lvl), len(leaf_codes))
    n = nxt

    kind = np.empty(n, np.int32)
    cpu = np.empty(n, np.float64)
    gpu = np.full(n, np.inf)
    src_l, dst_l = [], []

    def up(l):
        return ids[("P2M", l)] if l == leaf_lvl else ids[("M2M", l)]

    def index_of(l, codes):
        c = cells[l]
        pos = np.searchsorted(c, codes)
        pos = np.minimum(pos, len(c) - 1)
        ok = c[pos] == codes
        return pos, ok

    # P2M / L2P
    for name, kk in (("P2M", P2M), ("L2P", L2P)):
        t = ids[(name, leaf_lvl)]
        kind[t] = kk
        cpu[t] = n_p * 2.0 ** -10
    # M2M: children -> parent
    for l in range(leaf_lvl - 1, 1, -1):
        sc = 1 << (l + 1)
        x, y, z = _split(cells[l + 1], sc)
        ppos, ok = index_of(l, _join(x >> 1, y >> 1, z >> 1, 1 << l))
        assert ok.all()
        src_l.append(up(l + 1))
        dst_l.append(ids[("M2M", l)][ppos])
        nchild = np.bincount(ppos, minlength=len(cells[l]))
        t = ids[("M2M", l)]
        kind[t] = M2M
        cpu[t] = nchild * 2.0 ** -4
    # M2L: interaction lists
    o = np.arange(6)
    off = np.stack(np.meshgrid(o, o, o, indexing="ij"), -1).reshape(-1, 3)  # 216
    for l in range(2, leaf_lvl + 1):
        s = 1 << l
        c = cells[l]
        tgt_ids = ids[("M2L", l)]
        il_count = np.zeros(len(c), np.int64)
        chunk = 1 << 15
        for a in range(0, len(c), chunk):
            cc = c[a:a + chunk]
            x, y, z = _split(cc, s)
            bx, by, bz = ((x >> 1) - 1) * 2, ((y >> 1) - 1) * 2, ((z >> 1) - 1) * 2
            cx = bx[:, None] + off[None, :, 0]
            cy = by[:, None] + off[None, :, 1]
            cz = bz[:, None] + off[None, :, 2]
            inr = (cx >= 0) & (cx < s) & (cy >= 0) & (cy < s) & (cz >= 0) & (cz < s)
            adj = ((np.abs(cx - x[:, None]) <= 1) & (np.abs(cy - y[:, None]) <= 1)
                   & (np.abs(cz - z[:, None]) <= 1))
            cand = inr & ~adj
            codes = _join(np.where(cand, cx, 0), np.where(cand, cy, 0), np.where(cand, cz, 0), s)
            pos, ok = index_of(l, codes)
            ok &= cand
            rows, cols = np.nonzero(ok)
            il_count[a:a + len(cc)] = ok.sum(1)
            src_l.append(up(l)[pos[rows, cols]])
            dst_l.append(tgt_ids[a + rows])
        kind[tgt_ids] = M2L
        cpu[tgt_ids] = il_count * 2.0 ** -6
        gpu[tgt_ids] = il_count * 2.0 ** -9
    # L2L: M2L(parent), L2L(parent) -> L2L(child)
    for l in range(3, leaf_lvl + 1):
        x, y, z = _split(cells[l], 1 << l)
        ppos, ok = index_of(l - 1, _join(x >> 1, y >> 1, z >> 1, 1 << (l - 1)))
        assert ok.all()
        t = ids[("L2L", l)]
        src_l.append(ids[("M2L", l - 1)][ppos])
        dst_l.append(t)
        if l - 1 >= 3:
            src_l.append(ids[("L2L", l - 1)][ppos])
            dst_l.append(t)
        kind[t] = L2L
        cpu[t] = 2.0 ** -4
    # P2P: particle counts of the 27-neighbourhood
    x, y, z = _split(leaf_codes, side)
    n_nbr = np.zeros(len(leaf_codes), np.int64)
    for dx in (-1, 0, 1):
        for dy in (-1, 0, 1):
            for dz in (-1, 0, 1):
                nx, ny, nz = x + dx, y + dy, z + dz
                inr = (nx >= 0) & (nx < side) & (ny >= 0) & (ny < side) & (nz >= 0) & (nz < side)
                codes = _join(np.where(inr, nx, 0), np.where(inr, ny, 0), np.where(inr, nz, 0), side)
                pos, ok = index_of(leaf_lvl, codes)
                ok &= inr
                n_nbr += np.where(ok, n_p[pos], 0)
    t = ids[("P2P", leaf_lvl)]
    kind[t] = P2P
    cpu[t] = n_p * n_nbr * 2.0 ** -16
    gpu[t] = n_p * n_nbr * 2.0 ** -20
    # L2P <- M2L(leaf), L2L(leaf), P2P(leaf)
    t = ids[("L2P", leaf_lvl)]
    for name in ("M2L", "L2L", "P2P"):
        src_l.append(ids[(name, leaf_lvl)])
        dst_l.append(t)

    src = np.concatenate(src_l).astype(np.int32)
    dst = np.concatenate(dst_l).astype(np.int32)
    return dict(n=n, src=src, dst=dst, kind=kind,
                cpu_ms=cpu.astype(np.float32), gpu_ms=gpu.astype(np.float32),
                n_leaves=len(leaf_codes))
