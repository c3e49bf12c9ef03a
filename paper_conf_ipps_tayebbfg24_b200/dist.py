"""Replica sharding across GPUs (one process per GPU) and the summary allgather.

North_star: "Only the batched-replica mode ... shards across the 8 GPUs of one
box, with an NCCL allgather over NVLink of per-replica critical-path and
queue-head summaries; a single DAG stays on one GPU."  Replicas are
independent (their perturbation is keyed by the GLOBAL replica id, so results
do not depend on the world size); rank k owns the contiguous block
shard_range(R, W, k).  The only collective is one all_gather_into_tensor of
fixed-size per-replica records (CP + A queue summaries).
"""
from __future__ import annotations

import torch
import torch.distributed as dist

from . import SUMMARY_BYTES


def shard_range(R: int, world: int, rank: int) -> tuple[int, int]:
    """(r0, count) of rank's contiguous replica block; counts differ by at most 1."""
    if world < 1 or not (0 <= rank < world) or R < 0:
        raise ValueError("bad shard arguments")
    q, r = divmod(R, world)
    count = q + (1 if rank < r else 0)
    r0 = rank * q + min(rank, r)
    return r0, count


def record_bytes(n_arch: int, extra: int = 0) -> int:
    return 4 + n_arch * SUMMARY_BYTES + extra


def pack_records(cp: torch.Tensor, summary: torch.Tensor, count: int, n_arch: int, slots: int,
                 out: torch.Tensor | None = None, extra: torch.Tensor | None = None) -> torch.Tensor:
    """[slots, 4 + A*32 (+ k)] uint8 records (CP float bits, the A summaries, then `extra`'s k
    bytes per replica, e.g. the N2 simulation statistics); rows >= count are zero."""
    k = 0 if extra is None else extra.numel() // max(count, 1)
    rb = record_bytes(n_arch, k)
    if out is None:
        out = torch.zeros((slots, rb), dtype=torch.uint8, device=cp.device)
    if count:
        q = 4 + n_arch * SUMMARY_BYTES
        out[:count, :4].copy_(cp[:count].contiguous().view(torch.uint8).view(count, 4))
        out[:count, 4:q].copy_(summary[:count * n_arch * SUMMARY_BYTES].view(count, n_arch * SUMMARY_BYTES))
        if k:
            out[:count, q:q + k].copy_(extra.reshape(-1)[:count * k].view(count, k))
    return out


def gather_records(local: torch.Tensor, group=None, out: torch.Tensor | None = None) -> torch.Tensor:
    """all_gather_into_tensor of every rank's [slots, rb] records -> [world*slots, rb]."""
    world = dist.get_world_size(group)
    if out is None:
        out = torch.empty((world * local.shape[0], local.shape[1]), dtype=local.dtype, device=local.device)
    dist.all_gather_into_tensor(out, local.contiguous(), group=group)
    return out


def unpack_records(gathered: torch.Tensor, R: int, world: int, n_arch: int, extra: int = 0):
    """Reassemble (cp[R] float32, summary bytes[R*A*32]) ordered by global replica id
    (plus the extra bytes [R, extra] when extra > 0)."""
    slots = gathered.shape[0] // world
    rows = []
    for k in range(world):
        r0, c = shard_range(R, world, k)
        rows.append(gathered[k * slots:k * slots + c])
    g = torch.cat(rows, 0) if rows else gathered[:0]
    cp = g[:, :4].contiguous().view(torch.float32).reshape(-1)
    q = 4 + n_arch * SUMMARY_BYTES
    summ = g[:, 4:q].contiguous().reshape(-1)
    if extra:
        return cp, summ, g[:, q:q + extra].contiguous()
    return cp, summ
