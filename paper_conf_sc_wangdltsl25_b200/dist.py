"""Batch sharding over GPUs.

The batch dimension shards with no exchange step: every rank runs the same
kernel on its own contiguous slice of the global batch.  The only collective
is an all_gather of a tiny fixed-size per-rank record (device time, checksum,
entries) used for reporting -- never a data-path collective.

Works with any torch.distributed backend (NCCL on the GPU box, gloo in the
CPU tests).
"""
from __future__ import annotations

from dataclasses import dataclass


def shard_range(global_batch: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous balanced slice [lo, hi) of a fixed global batch (strong scaling)."""
    if world < 1 or not (0 <= rank < world) or global_batch < 0:
        raise ValueError("bad shard arguments")
    return global_batch * rank // world, global_batch * (rank + 1) // world


def weak_range(batch_per_rank: int, rank: int) -> tuple[int, int]:
    """Slice of rank ``rank`` when every rank owns ``batch_per_rank`` entries (weak scaling)."""
    return rank * batch_per_rank, (rank + 1) * batch_per_rank


@dataclass
class RankRecord:
    time_ms: float
    checksum: float
    entries: float


def aggregate(records: list[RankRecord]) -> dict:
    """Whole-job view: the slowest rank's time bounds the job (max over ranks)."""
    t = max(r.time_ms for r in records)
    return {"time_ms": t, "entries": sum(r.entries for r in records),
            "checksum": sum(r.checksum for r in records),
            "spread": (t / min(r.time_ms for r in records)) if min(r.time_ms for r in records) > 0 else None,
            "ranks": len(records)}


def gather_records(rec: RankRecord, device=None) -> list[RankRecord]:
    """all_gather of the per-rank record (the only cross-GPU traffic)."""
    import torch
    import torch.distributed as dist

    t = torch.tensor([rec.time_ms, rec.checksum, rec.entries], dtype=torch.float64, device=device)
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return [rec]
    out = [torch.zeros_like(t) for _ in range(dist.get_world_size())]
    dist.all_gather(out, t)
    return [RankRecord(*[float(x) for x in o.cpu().tolist()]) for o in out]
