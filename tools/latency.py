"""Per-launch latency of the tcgen05 path at tiny batches (BASELINE configs[0]
regime): CUDA-event time per launch for a torch no-op kernel, and kami f16
m=n=k=16 / 32 / 64 at several batch sizes, with and without an L2 flush
between launches, plus the host-side cost of one API call.

    python tools/latency.py
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import kami_inputs as ki  # noqa: E402
import paper_conf_sc_wangdltsl25_b200 as kami  # noqa: E402


def timed(fn, reps=50, flush=None):
    for _ in range(5):
        fn()
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for a, b in evs:
        if flush is not None:
            flush.zero_()
        a.record()
        fn()
        b.record()
    torch.cuda.synchronize()
    t = sorted(a.elapsed_time(b) * 1e3 for a, b in evs)
    return t[len(t) // 2], t[0]


def main():
    torch.cuda.set_device(0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    x = torch.zeros(1, device="cuda")
    out = {}
    out["torch_noop_us"] = timed(lambda: x.add_(0))
    for (m, batch) in [(16, 8), (16, 64), (16, 1024), (16, 8192), (32, 1024), (64, 1024), (64, 8192)]:
        A, B = ki.operands(m, m, m, batch, "f16", "unif", seed=0, device="cuda")
        C = torch.empty(batch * m * m, dtype=torch.float16, device="cuda")
        f = lambda: kami.gemm_strided_batched(m, m, m, batch, "f16", "row", A, B, C)  # noqa: E731
        hot = timed(f)
        cold = timed(f, flush=flush)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(200):
            f()
        host = (time.perf_counter() - t0) / 200 * 1e6
        torch.cuda.synchronize()
        out[f"f16_{m}^3_x{batch}"] = {"hot_us(med,min)": hot, "cold_us(med,min)": cold, "host_call_us": host,
                                      "kernel": kami.last_kernel()}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
