"""Per-kernel time of mp_dag_rebuild on a config's DAG and on its depth probe (chain of L
tasks + isolated tasks, same n).  Usage: python tools/ingest_breakdown.py c4 [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_tayebbfg24_b200 as mp  # noqa: E402
import workloads  # noqa: E402


def run(dag, n, src, dst, reps):
    for _ in range(3):
        mp.dag_rebuild(dag, n, src, dst)
    torch.cuda.synchronize()
    mp.prof_reset()
    mp.prof_enable(True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        mp.dag_rebuild(dag, n, src, dst)
    e1.record()
    torch.cuda.synchronize()
    mp.prof_enable(False)
    tot = e0.elapsed_time(e1) / reps
    ks = {k: mp.prof_query(k)[0] / reps for k in mp.prof_names() if mp.prof_query(k)[1] > 0}
    return tot, dict(sorted(ks.items(), key=lambda x: -x[1]))


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "c4"
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
    w = workloads.config(cfg)
    dev = torch.device("cuda:0")
    src, dst = torch.from_numpy(w.src).to(dev), torch.from_numpy(w.dst).to(dev)
    dag = mp.build_dag(w.n, src, dst)
    L = dag.n_levels
    tot, ks = run(dag, w.n, src, dst, reps)
    print(f"{cfg}: rebuild {tot:.3f} ms, L = {L}:", {k: round(v, 3) for k, v in ks.items()})
    sp = torch.arange(L - 1, dtype=torch.int32, device=dev)
    dp = sp + 1
    dagp = mp.build_dag(w.n, sp, dp)
    tot, ks = run(dagp, w.n, sp, dp, reps)
    print(f"{cfg} probe: rebuild {tot:.3f} ms:", {k: round(v, 3) for k, v in ks.items()})


if __name__ == "__main__":
    main()
