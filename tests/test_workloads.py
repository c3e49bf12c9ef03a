"""Workload generators reproduce the recipe statistics of SURVEY.md Appendix B (inputs only)."""
import numpy as np
import pytest

import oracle
import workloads


def test_c1_c2_c3_sizes():
    for name, n, E, L in (("c1", 20, 30, 10), ("c2", 45760, 131040, 190), ("c3", 707264, 2088896, 382)):
        w = workloads.config(name)
        d = oracle.build_dag(w.n, w.src, w.dst)
        assert (w.n, d.n_edges, d.n_levels) == (n, E, L)


def test_c4_recipe_statistics():
    sp = workloads.sparse_tree(42, 64, 32)
    assert sp.meta["fronts"] == 1797 and sp.n == 1057031
    assert np.bincount(sp.kind).tolist() == [2970, 28555, 28555, 925083, 71868]
    fm = workloads.fmm_tree(8, 1 << 19, 7)
    assert fm.n == 1099435 and len(fm.src) == 24008280
    assert np.bincount(fm.dst).max() == 189 and np.bincount(fm.src).max() == 190
    # durations: finite where the model has an implementation, +inf = cannot execute
    assert np.all(np.isfinite(sp.dur[:, 0])) and np.isinf(sp.dur[sp.kind == 4, 1]).all()


def test_lu_size_and_durations_domain():
    w = workloads.config("lu64")
    assert w.n == 89440
    d = oracle.build_dag(w.n, w.src, w.dst)
    assert d.n_edges == 260064 and d.n_levels == 190
    for name in ("c1", "c2", "c3"):
        wd = workloads.config(name)
        oracle.check_durations(wd.dur, wd.workers)   # inside the domain (reading c20)
