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
# N1 push, N2/N3 simulation, N4 variants
w = workloads.config("c1")
dag = mp.build_dag(w.n, torch.from_numpy(w.src).to(dev), torch.from_numpy(w.dst).to(dev))
dur = torch.from_numpy(w.dur).to(dev)
r = mp.score_and_queue(dag, dur, w.workers)
mp.simulate(dag, dur, [3, 1], 0, 0.0, 0, 1, r["qtask"], r["summary"], 4, True, trace=True)
data = mp.DataModel(w.acc_ptr, w.acc_handle, w.acc_mode, w.handle_size)
mp.simulate(dag, dur, [3, 2], 0, 0.0, 0, 1, r["qtask"], r["summary"], 4, True, trace=True, data=data, top_n=10,
            eps=0.8, xfer_ms_per_byte=2.0 ** -24)
mp.replicas_simulate(dag, dur, [2, 1], 7, 0.125, 0, 20, data=data, top_n=4, eps=0.5)
mp.bottom_level_w(dag, dur, w.workers, mp.MP_WEIGHT_MEAN)
mp.affinity_prefix(dag, dur, w.workers, torch.randperm(w.n, device=dev).to(torch.int32))
mp.nod_remaining(dag, dur, w.workers, torch.zeros(w.n, dtype=torch.uint8, device=dev))
rem = mp.ready_init(dag)
q0 = mp.build_queues(dag, r["key"], r["flags"], dur, done=torch.zeros(w.n, dtype=torch.uint8, device=dev))
mp.queues_push(dag, r["key"], r["flags"], dur, q0[1][:1].clone(), rem, q0[0], q0[1])
mp.check(dag)
n = 2000
s, d = random_dags.random_dag(n, 2.0, 2)
dur = torch.from_numpy(random_dags.dyadic_durations(n, 3, 2, p_inf=0.2)).to(dev)
dag = mp.build_dag(n, torch.from_numpy(s).to(dev), torch.from_numpy(d).to(dev))
r = mp.score_and_queue(dag, dur, [2, 1, 1])
data = mp.DataModel(*random_dags.random_data_model(n, 5000, 2), device=dev)
mp.simulate(dag, dur, [2, 1, 1], 0, 0.0, 0, 1, r["qtask"], r["summary"], 3, True, trace=True, data=data, top_n=8)
mp.affinity_prefix(dag, dur, [2, 1, 1])
mp.check(dag)
torch.cuda.synchronize()
print("sanitize run ok")
