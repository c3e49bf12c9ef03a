"""Replica sharding over NCCL: world-size invariance on >= 2 GPUs.

Each rank runs mp_replicas_run on its contiguous block of global replica ids,
packs the 68-byte records and all_gather_into_tensor's them over NCCL; the
reassembled records must equal, byte for byte, one process running all R
replicas on one GPU -- and the oracle on sampled replicas.  Skips on a box
with fewer than 2 GPUs (the gloo test covers the host-side logic on CPU).
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch

import oracle
import workloads

pytestmark = pytest.mark.gpu

R_TOTAL = 301        # not a multiple of the world size: ragged shards


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist

    import paper_conf_ipps_tayebbfg24_b200 as mp
    from paper_conf_ipps_tayebbfg24_b200 import dist as mpd
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(rank)
    dev = torch.device("cuda", rank)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=dev)
    try:
        w = workloads.config("c2")
        dag = mp.build_dag(w.n, torch.from_numpy(w.src).to(dev), torch.from_numpy(w.dst).to(dev))
        r0, cnt = mpd.shard_range(R_TOTAL, world, rank)
        slots = mpd.shard_range(R_TOTAL, world, 0)[1]
        cp, summ, _ = mp.replicas_run(dag, torch.from_numpy(w.dur).to(dev), w.workers, workloads.C5_SEED,
                                      workloads.C5_SIGMA, r0, cnt, want_queues=False)
        mp.check(dag)
        local = mpd.pack_records(cp, summ, cnt, w.n_arch, slots)
        g = mpd.gather_records(local)
        cp_all, s_all = mpd.unpack_records(g, R_TOTAL, world, w.n_arch)
        if rank == 0:
            q.put((cp_all.cpu().numpy().tobytes(), s_all.cpu().numpy().tobytes()))
    finally:
        dist.destroy_process_group()


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="needs >= 2 GPUs")
def test_nccl_world_size_invariance():
    import torch.multiprocessing as tmp

    import paper_conf_ipps_tayebbfg24_b200 as mp
    world = min(torch.cuda.device_count(), 8)
    ctx = tmp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(k, world, port, q)) for k in range(world)]
    for p in procs:
        p.start()
    got = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    w = workloads.config("c2")
    dag = mp.build_dag(w.n, torch.from_numpy(w.src).cuda(), torch.from_numpy(w.dst).cuda())
    cp, summ, _ = mp.replicas_run(dag, torch.from_numpy(w.dur).cuda(), w.workers, workloads.C5_SEED,
                                  workloads.C5_SIGMA, 0, R_TOTAL, want_queues=False)
    mp.check(dag)
    assert got[0] == cp.cpu().numpy().tobytes()
    assert got[1] == summ.cpu().numpy().tobytes()
    od = oracle.build_dag(w.n, w.src, w.dst)
    gs = np.frombuffer(got[1], np.uint8).reshape(R_TOTAL, -1)
    for r in (0, R_TOTAL // 2, R_TOTAL - 1):
        ocp, osum, _, _ = oracle.replica(od, w.dur, w.workers, workloads.C5_SEED, workloads.C5_SIGMA, r,
                                         want_queue=False)
        assert np.frombuffer(got[0], np.float32)[r] == np.float32(ocp)
        assert gs[r].tobytes() == osum.tobytes()
