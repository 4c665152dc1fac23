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


CHECKSUM_MOD = (1 << 31) - 1  # Mersenne prime; products of residues stay < 2^62


def position_checksum(C, entry0: int, n_entries: int, elems_per_entry: int) -> int:
    """World-size-invariant checksum of a rank's outputs: entries
    [entry0, entry0 + n_entries) of the GLOBAL batch, each ``elems_per_entry``
    values, given as a tensor on any device (16-bit, FP32 or FP64 storage).

        h = sum_e  w(entry0 + e) * (sum_i (i + 1) * v(e, i)  mod P)   mod P

    with v = the raw bits folded to 16 bits and w(e) = (e mod 65 521) + 1, so
    the total is exactly additive over any contiguous sharding: the sum of the
    ranks' checksums (mod P) equals the single-process checksum iff every
    entry's outputs are bit-identical in position (SURVEY.md 8(c) world-size
    invariance).  All arithmetic is int64 without overflow."""
    import torch

    if n_entries == 0:
        return 0
    x = C.reshape(n_entries, elems_per_entry)
    if x.dtype in (torch.float16, torch.bfloat16):
        v = x.view(torch.int16).to(torch.int64) & 0xFFFF
    elif x.dtype == torch.float32:
        b = x.view(torch.int32).to(torch.int64) & 0xFFFFFFFF
        v = (b ^ (b >> 16)) & 0xFFFF
    elif x.dtype == torch.float64:
        b = x.view(torch.int64)
        v = (b ^ (b >> 16) ^ (b >> 32) ^ (b >> 48)) & 0xFFFF
    else:
        raise TypeError(f"unsupported dtype {x.dtype}")
    i = torch.arange(1, elems_per_entry + 1, dtype=torch.int64, device=x.device)
    per = (v * i).sum(dim=1) % CHECKSUM_MOD  # < 2^16 * 2^16 * 2^16 per entry before the mod
    w = (torch.arange(entry0, entry0 + n_entries, dtype=torch.int64, device=x.device) % 65521) + 1
    return int(((per * w) % CHECKSUM_MOD).sum().item() % CHECKSUM_MOD)


def combine_checksums(parts) -> int:
    """Whole-job checksum from the ranks' position_checksum values."""
    return int(sum(int(p) for p in parts) % CHECKSUM_MOD)


@dataclass
class RankRecord:
    time_ms: float
    checksum: float
    entries: float


def aggregate(records: list[RankRecord]) -> dict:
    """Whole-job view: the slowest rank's time bounds the job (max over ranks).
    ``checksum`` sums the ranks' values; for position_checksum records use
    ``position_checksum`` (the exact residue) instead."""
    t = max(r.time_ms for r in records)
    return {"time_ms": t, "entries": sum(r.entries for r in records),
            "checksum": sum(r.checksum for r in records),
            "position_checksum": combine_checksums(r.checksum for r in records)
            if all(float(r.checksum).is_integer() for r in records) else None,
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
