"""bench.py host logic (-m "not gpu"): the N-rank self-launch command and the config
tables; the GPU arms themselves run on the B200 box."""
from __future__ import annotations

import importlib.util
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench():
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def test_spawn_ranks_relaunches_under_torchrun(monkeypatch):
    b = _bench()
    seen = {}
    monkeypatch.setattr(b.subprocess, "call", lambda cmd: seen.setdefault("cmd", cmd) and 0)
    monkeypatch.setattr(sys, "argv", ["bench.py", "--gpus", "8", "--steps", "5"])
    args = b.parse()
    assert args.scaling == "strong" and args.replicas == 4096      # BASELINE config 5: 4096 in total
    b.spawn_ranks(args)
    cmd = seen["cmd"]
    assert cmd[1:3] == ["-m", "torch.distributed.run"]
    assert "--nproc-per-node=8" in cmd and "127.0.0.1" in cmd
    assert cmd[-4:] == ["--gpus", "8", "--steps", "5"] and cmd[-5].endswith("bench.py")


def test_every_config_has_a_workload_text_and_a_base_workload():
    b = _bench()
    for c in b.REPLICA_CFGS + b.SINGLE_CFGS + ("c2push", "c2n4"):
        assert b.workload_text(c)
    assert b.base_workload("c5").name == "c2" and b.base_workload("hier").name == "hier"
