"""Times mp_bottom_level (per-kernel device ms via the libmp profiler) on the medium
single-DAG shapes: c3, c4, lu64, hier and the two k_bl_clu parity DAGs.  Prints one line
per DAG: the bl kernel(s) taken and their mean ms per call.  (An experiment tool: the
dispatch thresholds of path.cuh are compile-time macros; rebuild with -D to compare.)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch

import paper_conf_ipps_tayebbfg24_b200 as mp
import workloads
from workloads import random_dags


def dags():
    for name in sys.argv[1:] or ["c3", "c4", "lu64", "hier", "layered", "rand300k"]:
        if name == "layered":
            n, s, d = random_dags.layered_dag([1, 3, 30000, 2, 30000, 30000, 30000, 1, 16, 9000, 17, 5], fan=60,
                                              seed=41)
            yield name, n, s, d, random_dags.dyadic_durations(n, 2, 41), np.ones(2, np.int32)
        elif name == "rand300k":
            n = 300000
            s, d = random_dags.random_dag(n, 5.0, 42, dup=0.1, max_span=64)
            yield name, n, s, d, random_dags.dyadic_durations(n, 3, 42), np.ones(3, np.int32)
        else:
            w = workloads.config(name)
            yield name, w.n, w.src, w.dst, w.dur, w.workers


for name, n, s, d, dur, workers in dags():
    dag = mp.build_dag(n, torch.from_numpy(s).cuda(), torch.from_numpy(d).cuda())
    du = torch.from_numpy(np.ascontiguousarray(dur, np.float32)).cuda()
    for _ in range(3):
        mp.bottom_level(dag, du, workers)
    torch.cuda.synchronize()
    mp.prof_enable(True)
    mp.prof_reset()
    K = 20
    for _ in range(K):
        mp.bottom_level(dag, du, workers)
    torch.cuda.synchronize()
    ks = {k: round(mp.prof_query(k)[0] / K, 4) for k in mp.prof_names() if k.startswith("k_bl")}
    mp.prof_enable(False)
    mp.check(dag)
    print(f"{name:10s} n={n} E={dag.n_edges} L={dag.n_levels} {ks}", flush=True)
