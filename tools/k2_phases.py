#!/usr/bin/env python
"""Per-phase cycle split of k_rep2_sort on the c5 workload (debug build, GPU box only).

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
names = {1: "P0 hash+D+minmax", 2: "pass1 coarse hist", 3: "sub-bins", 4: "pass2 fine hist+fb", 5: "prefix+groups",
         7: "rounds (place+rank+out)", 8: "Ps copy", 9: "eq bits", 10: "members+crit", 11: "emission", 12: "summary", 13: "  round: scan+place", 14: "  round: rank+out"}
tot = buf.sum()
for i in sorted(names):
    print(f"{names[i]:28s} {100.0 * buf[i] / tot:5.1f}%  {buf[i] / R / 1.965e3:8.2f} us/replica")
print(f"deferred positions per replica {buf[20] / R:8.1f}   near-tie pairs per replica {buf[21] / R:8.1f}")
