"""Multi-rank host logic on CPU (gloo, world size 2): batch sharding,
world-size invariance of the generated entries, and the stats gather."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import kami_inputs as ki
from paper_conf_sc_wangdltsl25_b200 import dist as kdist


def test_shard_ranges_cover_exactly():
    for B in (0, 1, 7, 65536, 10 ** 6):
        for W in (1, 2, 3, 4, 8):
            rs = [kdist.shard_range(B, r, W) for r in range(W)]
            assert rs[0][0] == 0 and rs[-1][1] == B
            assert all(rs[i][1] == rs[i + 1][0] for i in range(W - 1))
            assert max(h - l for l, h in rs) - min(h - l for l, h in rs) <= 1
    assert kdist.weak_range(65536, 3) == (3 * 65536, 4 * 65536)
    with pytest.raises(ValueError):
        kdist.shard_range(10, 2, 2)


def test_aggregate_takes_max_time():
    agg = kdist.aggregate([kdist.RankRecord(2.0, 1.5, 10), kdist.RankRecord(3.0, -0.5, 12)])
    assert agg["time_ms"] == 3.0 and agg["entries"] == 22 and agg["checksum"] == 1.0 and agg["spread"] == 1.5


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        B = 10
        lo, hi = kdist.shard_range(B, rank, world)
        A, Bm = ki.operands(16, 16, 16, hi - lo, "f16", "unif", seed=5, entry0=lo)
        rec = kdist.RankRecord(time_ms=1.0 + rank, checksum=float(A.double().sum() + Bm.double().sum()),
                               entries=float(hi - lo))
        recs = kdist.gather_records(rec)
        q.put((rank, [(r.time_ms, r.checksum, r.entries) for r in recs], A.view(torch.int16).tolist()))
    finally:
        dist.destroy_process_group()


def test_gloo_two_ranks_gather_and_invariance():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort()
    # both ranks see the same gathered records, max time = slowest rank
    assert res[0][1] == res[1][1]
    agg = kdist.aggregate([kdist.RankRecord(*r) for r in res[0][1]])
    assert agg["time_ms"] == 2.0 and agg["entries"] == 10
    # world-size invariance: the shards concatenate to the single-process batch
    A_full, B_full = ki.operands(16, 16, 16, 10, "f16", "unif", seed=5)
    got = torch.tensor(res[0][2] + res[1][2], dtype=torch.int16)
    assert torch.equal(got, A_full.view(torch.int16))
    tot = float(A_full.double().sum() + B_full.double().sum())
    assert abs(agg["checksum"] - tot) < 1e-9


def test_position_checksum_additive_over_shards():
    """The bench checksum is exactly additive over any contiguous sharding
    (world-size invariance), and sensitive to a changed or moved entry."""
    B, m, n = 37, 8, 16
    C = ki.draw(9, 0, 0, B, m, n, "f16", "unif")
    whole = kdist.position_checksum(C, 0, B, m * n)
    for W in (1, 2, 3, 4, 8):
        parts = []
        for r in range(W):
            lo, hi = kdist.shard_range(B, r, W)
            parts.append(kdist.position_checksum(C.view(B, -1)[lo:hi], lo, hi - lo, m * n))
        assert kdist.combine_checksums(parts) == whole
    C2 = C.clone().view(B, -1)
    C2[5, 3] = C2[5, 3] + 1  # one output changed
    assert kdist.position_checksum(C2, 0, B, m * n) != whole
    C3 = C.clone().view(B, -1)
    C3[[4, 9]] = C3[[9, 4]]  # two entries swapped
    assert kdist.position_checksum(C3, 0, B, m * n) != whole
    for dt in ("f64", "f32"):
        X = ki.draw(9, 0, 0, B, m, n, dt, "unif")
        a = kdist.position_checksum(X, 0, B, m * n)
        b = kdist.combine_checksums([kdist.position_checksum(X.view(B, -1)[:20], 0, 20, m * n),
                                     kdist.position_checksum(X.view(B, -1)[20:], 20, B - 20, m * n)])
        assert a == b


def _bench_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # the bench's per-rank logic, CPU stand-in for the GPU output: strong
        # scaling shards the global batch, every rank checksums its own shard
        B, m, n = 21, 4, 8
        lo, hi = kdist.shard_range(B, rank, world)
        C = ki.draw(4, 1, lo, hi - lo, m, n, "f16", "unif")
        rec = kdist.RankRecord(time_ms=1.0 + rank, checksum=float(kdist.position_checksum(C, lo, hi - lo, m * n)),
                               entries=float(hi - lo))
        agg = kdist.aggregate(kdist.gather_records(rec))
        q.put((rank, agg["position_checksum"], agg["entries"], agg["time_ms"]))
    finally:
        dist.destroy_process_group()


def test_gloo_two_ranks_strong_scaling_checksum_matches_single_process():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_bench_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    single = kdist.position_checksum(ki.draw(4, 1, 0, 21, 4, 8, "f16", "unif"), 0, 21, 32)
    assert res[0][1] == res[1][1] == single
    assert res[0][2] == 21 and res[0][3] == 2.0
