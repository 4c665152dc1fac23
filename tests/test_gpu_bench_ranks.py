"""The N > 1 bench path end to end on one GPU: two
torchrun ranks share cuda:0 (KAMI_BENCH_SHARED_GPU=1, stats over gloo because
NCCL refuses two ranks on one device), each runs its own shard of the batch,
and rank 0 prints the whole-job line (max over ranks, weak scaling)."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _bench(nproc, extra=()):
    env = dict(os.environ, KAMI_BENCH_SHARED_GPU="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), "bench.py", "--gpus", str(nproc),
           "--steps", "4", "--warmup", "3", "--workload", "f16-32", "--no-cpu-baseline", *extra]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout  # rank 0 alone prints
    return json.loads(lines[0])


def test_two_ranks_one_line_whole_job():
    d = _bench(2)
    assert d["n_gpus"] == 2 and d["scaling"] == "weak"
    assert d["config"]["global_batch"] == 2 * d["config"]["batch_per_gpu"]
    assert d["config"]["parallelism"] == "batch-sharded dp2"
    assert d["value"] > 0 and d["gpu_launches"] == 4
    assert d["roofline"]["kernel"].startswith("kami_tc16_1d_kernel")
    # whole-job TFLOP/s = both ranks' flops / the slowest rank's time
    flops = 2.0 * 32 ** 3 * d["config"]["global_batch"] * d["steps"]
    assert abs(d["value"] - flops / (d["ms_per_step"] * d["steps"] * 1e-3) / 1e12) <= 1e-6 * d["value"]
    assert d["e2e"]["value"] > 0
    assert len(d["ranks"]["time_ms"]) == 2 and d["ranks"]["spread"] >= 1.0
    assert abs(max(d["ranks"]["time_ms"]) - d["ms_per_step"] * d["steps"]) <= 1e-6 * d["ms_per_step"] * d["steps"]

