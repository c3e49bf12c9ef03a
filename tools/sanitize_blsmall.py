"""compute-sanitizer run of k_bl_small (TMA-staged CSR slices): c2, c1, a 6000-task chain,
a star, a random DAG whose wide levels do not fit the staging buffers."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_ipps_tayebbfg24_b200 as mp
import workloads
from workloads import random_dags

dev = "cuda"
cases = [workloads.config("c2"), workloads.config("c1")]
for n, (s, d) in ((6000, random_dags.chain(6000)), (40000, random_dags.star(40000)),
                  (50000, random_dags.random_dag(50000, 3.0, 7, max_span=20000))):
    cases.append(workloads.Workload("r", n, s, d, random_dags.dyadic_durations(n, 2, 7), ("CPU", "GPU"),
                                    torch.ones(2, dtype=torch.int32).numpy()))
for w in cases:
    dag = mp.build_dag(w.n, torch.from_numpy(w.src).to(dev), torch.from_numpy(w.dst).to(dev))
    mp.bottom_level(dag, torch.from_numpy(w.dur).to(dev), w.workers)
    mp.check(dag)
torch.cuda.synchronize()
print("sanitize bl_small run ok")
