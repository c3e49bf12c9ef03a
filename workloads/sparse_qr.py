"""Sparse-QR-like multifrontal elimination-tree DAG (QR_MUMPS-shaped).

Shape source: PAPER.md l.272-308 (§VI-C, QR_MUMPS multifrontal QR with
METIS ordering); recipe: SURVEY.md Appendix B "Sparse-QR-like (G, leaf, nb)".
Input generator only -- no MultiPrio arithmetic here.

Nested dissection of a G^3 grid by recursive bisection of the longest box
axis; the separator is the middle cross-section.  Each front is a partial
tile QR (tile size nb) of an (nf+cf) x (nf+cf) tile matrix whose first
p = ceil(nf/nb) tile-columns are eliminated; the remaining contribution block
is assembled into the parent by ASM tasks (extend-add).  All dependencies are
inferred by the STF recorder from tile-handle accesses in post-order.
"""
from __future__ import annotations

from .stf import STFRecorder

GEQRT, TSQRT, UNMQR, TSMQR, ASM = 0, 1, 2, 3, 4


def _faces_interior(box, G):
    (x0, x1), (y0, y1), (z0, z1) = box
    ex, ey, ez = x1 - x0, y1 - y0, z1 - z0
    c = 0
    if x0 > 0:
        c += ey * ez
    if x1 < G:
        c += ey * ez
    if y0 > 0:
        c += ex * ez
    if y1 < G:
        c += ex * ez
    if z0 > 0:
        c += ex * ey
    if z1 < G:
        c += ex * ey
    return c


def _build_tree(G, leaf, nb):
    """Return fronts in post-order: list of (nf, cf, [child indices])."""
    fronts = []

    def rec(box):
        ext = [b[1] - b[0] for b in box]
        vol = ext[0] * ext[1] * ext[2]
        if vol <= 0:
            return None
        if vol <= leaf:
            nf = vol
            cf = min(_faces_interior(box, G), 4 * nf + nb)
            fronts.append((nf, cf, []))
            return len(fronts) - 1
        ax = max(range(3), key=lambda a: ext[a])
        lo, hi = box[ax]
        mid = (lo + hi) // 2
        left = list(box)
        right = list(box)
        left[ax] = (lo, mid)
        right[ax] = (mid + 1, hi)
        kids = []
        for b in (tuple(left), tuple(right)):
            k = rec(b)
            if k is not None:
                kids.append(k)
        nf = vol // ext[ax]
        cf = min(_faces_interior(box, G), 4 * nf + nb)
        fronts.append((nf, cf, kids))
        return len(fronts) - 1

    rec(((0, G), (0, G), (0, G)))
    return fronts


def sparse_qr_tree(G: int = 42, leaf: int = 64, nb: int = 32) -> tuple[STFRecorder, int]:
    """Record the multifrontal tile-QR DAG.  Returns (recorder, n_fronts)."""
    fronts = _build_tree(G, leaf, nb)
    s = STFRecorder()
    dims = []  # (mt, p) per front
    for f, (nf, cf, _) in enumerate(fronts):
        mt = -(-(nf + cf) // nb)
        p = -(-nf // nb)
        dims.append((mt, p))

    # handle encoding: tiles of front f and reflector workspace V(f,k)
    def T(f, i, j):
        return (f << 24) | (i << 12) | j

    def V(f, k):
        return (f << 24) | (1 << 23) | k

    for f, (nf, cf, kids) in enumerate(fronts):
        mt, p = dims[f]
        nt = mt
        # extend-add of the children's contribution blocks (post-order)
        for c in kids:
            mtc, pc = dims[c]
            for i in range(pc, mtc):
                ii = min(i - pc, mt - 1)
                for j in range(pc, mtc):
                    jj = min(j - pc, nt - 1)
                    s.submit(ASM, reads=(T(c, i, j),), writes=(T(f, ii, jj),))
        # partial tile QR over the first p tile-columns
        for k in range(p):
            s.submit(GEQRT, writes=(T(f, k, k), V(f, k)))
            for j in range(k + 1, nt):
                s.submit(UNMQR, reads=(V(f, k),), writes=(T(f, k, j),))
            for i in range(k + 1, mt):
                s.submit(TSQRT, writes=(T(f, k, k), T(f, i, k)))
                for j in range(k + 1, nt):
                    s.submit(TSMQR, reads=(T(f, i, k),), writes=(T(f, k, j), T(f, i, j)))
    return s, len(fronts)
