"""compute-sanitizer run at the sizes where the risky kernels switch on (ROUND 2):
k_bl_flow (n > 51,200: relaxed-memory dataflow), the grid-cooperative k_kahn (n > 48 Ki),
k_rep2_bl's dataflow mode (>= 75 groups of 32 replicas: one CTA per group) and its cluster
mode (few groups), k_rep2_sort on the c2 DAG, the general replica path (n >= 65,536)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_ipps_tayebbfg24_b200 as mp
import workloads
from workloads import random_dags

dev = "cuda"


def dag_of(n, s, d):
    return mp.build_dag(n, torch.from_numpy(s).to(dev), torch.from_numpy(d).to(dev))


# grid k_kahn + k_bl_flow + NOD on a 60k-task random DAG, and a 70k chain
for n, (s, d) in ((60000, random_dags.random_dag(60000, 2.5, 3, dup=0.2, max_span=64)),
                  (70000, random_dags.chain(70000))):
    dag = dag_of(n, s, d)
    dur = torch.from_numpy(random_dags.dyadic_durations(n, 2, 3, p_inf=0.1)).to(dev)
    mp.score_and_queue(dag, dur, [1, 1])
    mp.score_and_queue(dag, dur, [1, 1], kind=mp.MP_CRIT_NOD)
    mp.check(dag)
# general replica path (n >= 65,536): the single-DAG kernels once per replica
n = 66000
s, d = random_dags.random_dag(n, 2.0, 4, max_span=64)
dag = dag_of(n, s, d)
mp.replicas_run(dag, torch.from_numpy(random_dags.dyadic_durations(n, 2, 4)).to(dev), [1, 1], 5, 0.125, 0, 2)
mp.check(dag)
# K1 dataflow mode (75+ groups, one CTA each) on c1, K1 cluster mode + K2 on c2
w = workloads.config("c1")
dag = dag_of(w.n, w.src, w.dst)
mp.replicas_run(dag, torch.from_numpy(w.dur).to(dev), w.workers, 1, 0.125, 0, 2400)
mp.check(dag)
w = workloads.config("c2")
dag = dag_of(w.n, w.src, w.dst)
mp.replicas_run(dag, torch.from_numpy(w.dur).to(dev), w.workers, workloads.C5_SEED, workloads.C5_SIGMA, 0, 64)
mp.check(dag)
torch.cuda.synchronize()
print("sanitize large run ok")
