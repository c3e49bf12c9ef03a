"""Multi-process replica sharding + summary allgather on CPU (gloo, world_size 2).

The per-rank replica results come from the oracle (tests may call it); what is
under test is the product's shard assignment, record packing, collective and
reassembly by global replica id (world-size invariance).
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as tmp

import oracle
import workloads
from paper_conf_ipps_tayebbfg24_b200 import dist as mpd


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _oracle_records(R_range, w, od):
    cps, sums = [], []
    for r in R_range:
        cp, summ, _, _ = oracle.replica(od, w.dur, w.workers, workloads.C5_SEED, workloads.C5_SIGMA, r,
                                        want_queue=False)
        cps.append(np.float32(cp))
        sums.append(summ.tobytes())
    cp_t = torch.from_numpy(np.array(cps, np.float32))
    s_t = torch.from_numpy(np.frombuffer(b"".join(sums), np.uint8).copy())
    return cp_t, s_t


def _worker(rank, world, port, R, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        w = workloads.config("c1")
        od = oracle.build_dag(w.n, w.src, w.dst)
        r0, cnt = mpd.shard_range(R, world, rank)
        slots = mpd.shard_range(R, world, 0)[1]
        cp, s = _oracle_records(range(r0, r0 + cnt), w, od)
        local = mpd.pack_records(cp, s, cnt, w.n_arch, slots)
        g = mpd.gather_records(local)
        cp_all, s_all = mpd.unpack_records(g, R, world, w.n_arch)
        if rank == 0:
            q.put((cp_all.numpy().tobytes(), s_all.numpy().tobytes()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("R", [6, 7])
def test_gloo_world2_gather_equals_single_process(R):
    ctx = tmp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(k, 2, port, R, q)) for k in range(2)]
    for p in procs:
        p.start()
    got = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    w = workloads.config("c1")
    od = oracle.build_dag(w.n, w.src, w.dst)
    cp, s = _oracle_records(range(R), w, od)
    assert got[0] == cp.numpy().tobytes()
    assert got[1] == s.numpy().tobytes()


def test_shard_range_partitions():
    for R in (0, 1, 7, 4096, 4097):
        for W in (1, 2, 3, 4, 8):
            seen = []
            for k in range(W):
                r0, c = mpd.shard_range(R, W, k)
                seen.extend(range(r0, r0 + c))
            assert seen == list(range(R))
