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
