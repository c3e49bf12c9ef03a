"""Small end-to-end run for compute-sanitizer (memcheck / racecheck / synccheck)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_ipps_tayebbfg24_b200 as mp
import workloads
from workloads import random_dags

dev = "cuda"
for w in (workloads.config("c1"), workloads.qr(6)):
    dag = mp.build_dag(w.n, torch.from_numpy(w.src).to(dev), torch.from_numpy(w.dst).to(dev))
    dur = torch.from_numpy(w.dur).to(dev)
    mp.score_and_queue(dag, dur, w.workers)
    mp.score_and_queue(dag, dur, w.workers, kind=mp.MP_CRIT_NOD)
    mp.replicas_run(dag, dur, w.workers, 1, 0.125, 0, 40)
    mp.check(dag)
n = 3000
s, d = random_dags.random_dag(n, 2.0, 1, dup=0.2, max_span=40)
dur = random_dags.dyadic_durations(n, 2, 1, p_inf=0.2)
dag = mp.build_dag(n, torch.from_numpy(s).to(dev), torch.from_numpy(d).to(dev))
mp.score_and_queue(dag, torch.from_numpy(dur).to(dev), [1, 1])
mp.replicas_run(dag, torch.from_numpy(dur).to(dev), [1, 1], 3, 0.125, 5, 33)
mp.check(dag)
torch.cuda.synchronize()
print("sanitize run ok")
