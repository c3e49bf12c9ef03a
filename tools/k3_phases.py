#!/usr/bin/env python
"""Per-phase cycle split of k_rep3_sort on the c5 workload (debug build, GPU box only).

  python tools/k2_phases.py        # rebuilds libmp.so with -DMP_PHASES in place (scratch copy!)
Phases are separated by block barriers; thread 0 of every CTA accumulates clock64 deltas."""
import ctypes as C, os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ipps_tayebbfg24_b200 import build as B
subprocess.check_call([B.NVCC, *B.FLAGS, "-DMP_PHASES", *os.environ.get("K2_DEFS", "").split(), "-o", B.LIB,
                       os.path.join(B.CSRC, "libmp.cu")])
import numpy as np, torch
import paper_conf_ipps_tayebbfg24_b200 as mp, workloads
from paper_conf_ipps_tayebbfg24_b200 import _lib
L = _lib.lib()
L.mp_debug_k2_phases.argtypes = [C.c_void_p, C.c_int]
w = workloads.config("c2")
dev = torch.device("cuda:0")
dag = mp.build_dag(w.n, torch.from_numpy(w.src).to(dev), torch.from_numpy(w.dst).to(dev))
dur = torch.from_numpy(w.dur).to(dev)
R = 4096
buf = np.zeros(32, np.uint64)
for it in range(3):
    L.mp_debug_k2_phases(buf.ctypes.data, 1)
    mp.replicas_run(dag, dur, w.workers, workloads.C5_SEED, workloads.C5_SIGMA, 0, R)
    torch.cuda.synchronize()
L.mp_debug_k2_phases(buf.ctypes.data, 1)
names = {17: "P1 hash+fine hist", 18: "S scan", 20: "P2 scatter", 21: "P3 bin sort", 22: "P3b same-gain bits", 23: "P5 emission"}

tot = buf[16:].sum()
for i in sorted(names):  # cycles of CTA 0 of each cluster
    print(f"{names[i]:28s} {100.0 * buf[i] / tot:5.1f}%  {buf[i] / R / 1.965e3:8.2f} us/replica")
