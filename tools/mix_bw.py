"""HBM ceiling for the traffic mixes of the batched-GEMM workloads, measured
with plain torch streaming kernels (context for roofline.frac; not a product
path): copy (1 read : 1 write), add (2 : 1, the m = n = k mix), addcmul
(3 : 1) and a pure read (reduction).  Each is timed 'cold' (3 warm-ups, 20
reps) and 'sustained' (after a 1.5 s burst of the same op, the way bench.py
times), with nvidia-smi SM clocks sampled during the sustained timing."""
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from bench import ClockSampler  # noqa: E402

N = 1 << 29  # 2^29 fp16 = 1 GiB per operand
dev = "cuda"
a = torch.randn(N, device=dev).half()
b = torch.randn(N, device=dev).half()
c = torch.empty(N, device=dev, dtype=torch.half)
d = torch.randn(N, device=dev).half()


def timed(fn, reps=20, burst=0.0):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    smp = None
    if burst:
        smp = ClockSampler(0)
        smp.start()
        t_end = time.time() + burst
        while time.time() < t_end:
            for _ in range(10):
                fn()
            torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for s, e in ev:
        s.record()
        fn()
        e.record()
    torch.cuda.synchronize()
    if smp:
        smp.stop()
    ts = sorted(s.elapsed_time(e) for s, e in ev)
    return ts[len(ts) // 2] * 1e-3, (smp.summary() if smp else None)


ops = {
    "copy_1r1w": (lambda: c.copy_(a), 2),
    "add_2r1w": (lambda: torch.add(a, b, out=c), 3),
    "addcmul_3r1w": (lambda: torch.addcmul(a, b, d, out=c), 4),
    "sum_read": (lambda: torch.sum(a, dtype=torch.float32), 1),
    "fill_0r1w": (lambda: c.fill_(1.5), 1),
    # 1 read : 8 writes (the low-rank k = 16 mix): a 1/8-size source broadcast into c
    "bcast_1r8w": (lambda: c.view(8, N // 8).copy_(a[: N // 8].view(1, N // 8).expand(8, N // 8)), 1.125),
}
out = {}
for name, (fn, nbuf) in ops.items():
    t, _ = timed(fn)
    ts, clk = timed(fn, burst=1.5)
    out[name] = {"cold_GBs": nbuf * N * 2 / t / 1e9, "sustained_GBs": nbuf * N * 2 / ts / 1e9, "clocks": clk}
print(json.dumps(out, indent=1))
