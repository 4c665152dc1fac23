"""HBM ceiling for the traffic mixes of the batched-GEMM workloads, measured
with plain torch streaming kernels (context for roofline.frac; not a product
path): copy (1 read : 1 write), add (2 : 1, the m = n = k mix), sum of three
(3 : 1) and a pure read (reduction)."""
import json
import torch

N = 1 << 29  # 2^29 fp16 = 1 GiB per operand
dev = "cuda"
a = torch.randn(N // 2, device=dev).half().repeat(2)
b = torch.randn(N, device=dev).half()
c = torch.empty(N, device=dev, dtype=torch.half)
d = torch.randn(N, device=dev).half()


def timed(fn, reps=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for s, e in ev:
        s.record()
        fn()
        e.record()
    torch.cuda.synchronize()
    ts = sorted(s.elapsed_time(e) for s, e in ev)
    return ts[len(ts) // 2] * 1e-3


out = {}
t = timed(lambda: c.copy_(a))
out["copy_1r1w_GBs"] = 2 * N * 2 / t / 1e9
t = timed(lambda: torch.add(a, b, out=c))
out["add_2r1w_GBs"] = 3 * N * 2 / t / 1e9
t = timed(lambda: torch.addcmul(a, b, d, out=c))
out["addcmul_3r1w_GBs"] = 4 * N * 2 / t / 1e9
s = torch.empty((), device=dev, dtype=torch.float32)
t = timed(lambda: torch.sum(a, dtype=torch.float32))
out["sum_read_GBs"] = N * 2 / t / 1e9
print(json.dumps(out))
