"""compute-sanitizer run of k_bl_flow with its pending lists (n > 51,200, E > 1 Mi, not
wide): a 15-level layered DAG (~1.3 M distinct edges, some chunks with more pending successors
than the 1024-entry list holds -> the in-place wait) and, for NOD, the same DAG."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_tayebbfg24_b200 as mp  # noqa: E402
from workloads import random_dags  # noqa: E402

n, s, d = random_dags.layered_dag([1, 3, 20000, 2, 20000, 20000, 1, 16, 9000, 17, 5, 3000, 20000, 40, 20000], fan=40, seed=43)
dag = mp.build_dag(n, torch.from_numpy(s).cuda(), torch.from_numpy(d).cuda())
assert dag.n_edges > (1 << 20) and n < 16384 * dag.n_levels, (dag.n_edges, dag.n_levels)
dur = torch.from_numpy(random_dags.dyadic_durations(n, 2, 43, p_inf=0.1)).cuda()
mp.prof_enable(True)
mp.score_and_queue(dag, dur, [1, 1])
torch.cuda.synchronize()
ks = [k for k in mp.prof_names() if k.startswith("k_bl")]
mp.prof_enable(False)
mp.check(dag)
print("bl kernels:", ks, "n", n, "E", dag.n_edges, "L", dag.n_levels)
print("run ok")
