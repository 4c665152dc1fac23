"""Measured throughput of every candidate schedule on the BASELINE.json
configs (round 2): the data the planner's model is checked against
(tests/test_planner_model.py).

For each config and each candidate (kernel family, algo, p) the strided
batched GEMM is timed like bench.py: inputs generated on the device, K
launches captured in one CUDA graph and replayed between two CUDA events
(3 warm-ups; input sets rotated past L2 for the L2-resident config), median
of 3 replays.  Writes profiles/r2/variant_sweep_r2.json:
    {"configs": [{"cfg": name, "dtype", "m", "n", "k", "batch",
                  "candidates": [{"algo", "p", "kernel", "tflops"}, ...]}]}
Run on the GPU box:  python tools/variant_sweep_r2.py [--quick]
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import kami_inputs as ki  # noqa: E402
import paper_conf_sc_wangdltsl25_b200 as kami  # noqa: E402

CONFIGS = [
    # name, dtype, m, n, k, batch
    ("c0 f16-16", "f16", 16, 16, 16, 1024),
    ("c1 f16-32", "f16", 32, 32, 32, 65536),
    ("c1 f16-64", "f16", 64, 64, 64, 65536),
    ("c1 f16-128", "f16", 128, 128, 128, 65536),
    ("c2 f64-16", "f64", 16, 16, 16, 32768),
    ("c2 f64-32", "f64", 32, 32, 32, 32768),
    ("c2 f64-64", "f64", 64, 64, 64, 32768),
    ("c3 lr-8", "f16", 256, 256, 8, 16384),
    ("c3 lr-16", "f16", 256, 256, 16, 16384),
    ("c3 lr-32", "f16", 256, 256, 32, 16384),
    ("c4 bf16-16", "bf16", 16, 16, 16, 125000),
    ("c4 bf16-48", "bf16", 48, 48, 48, 125000),
    ("c4 bf16-96", "bf16", 96, 96, 96, 125000),
    ("c4 bf16-192", "bf16", 192, 192, 192, 20000),
    ("c4 bf16-16x128x16", "bf16", 16, 128, 16, 125000),
    ("c4 f64-128 (a7)", "f64", 128, 128, 128, 8192),
    # the BF16 sweep's slowest r1 points (thin m / n, k <= 32)
    ("c4 bf16-16x192x16", "bf16", 16, 192, 16, 125000),
    ("c4 bf16-192x16x16", "bf16", 192, 16, 16, 125000),
    ("c4 bf16-16x64x16", "bf16", 16, 64, 16, 125000),
    ("c4 bf16-16x128x32", "bf16", 16, 128, 32, 125000),
    ("c4 bf16-16x32x16", "bf16", 16, 32, 16, 125000),
    ("c4 bf16-16x256x16", "bf16", 16, 256, 16, 125000),
    ("c4 bf16-128x16x16", "bf16", 128, 16, 16, 125000),
    ("c4 bf16-32x128x16", "bf16", 32, 128, 16, 125000),
    ("c4 bf16-64x16x16", "bf16", 64, 16, 16, 125000),
    ("c4 bf16-32x16x16", "bf16", 32, 16, 16, 125000),
    ("c4 bf16-256x16x16", "bf16", 256, 16, 16, 125000),
    ("c4 bf16-16x192x32", "bf16", 16, 192, 32, 125000),
    ("c4 bf16-192x16x32", "bf16", 192, 16, 32, 125000),
    ("c4 bf16-16x16x32", "bf16", 16, 16, 32, 125000),
    ("c4 bf16-128x32x16", "bf16", 128, 32, 16, 125000),
    ("c4 bf16-40x24x56 (8-grid)", "bf16", 40, 24, 56, 125000),
    ("c4 bf16-32x192x16", "bf16", 32, 192, 16, 125000),
    ("c4 bf16-32x256x16", "bf16", 32, 256, 16, 125000),
    ("c4 bf16-16x256x32", "bf16", 16, 256, 32, 125000),
    ("c4 f64-96x40x72 (a7)", "f64", 96, 40, 72, 32768),
]

# candidate schedules: (algo, p); the library rejects the ones a shape has no kernel for
CANDIDATES = {
    "16": [("1d", 0), ("1d_xt", 0), ("1d_tmem", 0), ("3d_tmem", 0), ("1d", 1), ("1d", 2), ("1d", 4), ("1d", 8), ("2d", 0),
           ("3d", 0), ("nonca", 0), ("auto", 0)],
    "f64": [("1d_tma", 0), ("1d", 0), ("1d", 1), ("1d", 2), ("1d", 8), ("2d", 0), ("3d", 0), ("nonca", 0),
            ("auto", 0)],
}


def time_call(fn, steps, sets):
    for i in range(3):
        fn(i % len(sets))
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for i in range(steps):
            fn(i % len(sets))
    g.replay()
    torch.cuda.synchronize()
    out = []
    for _ in range(3):
        if len(sets) > 1:
            torch.empty(256 << 20, dtype=torch.uint8, device="cuda").fill_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        out.append(e0.elapsed_time(e1) / steps)
    return statistics.median(out)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r2", "variant_sweep_r2.json"))
    a = ap.parse_args()
    res = []
    for name, dtype, m, n, k, batch in CONFIGS:
        es = 8 if dtype == "f64" else 2
        bytes_ = batch * (m * k + k * n + m * n) * es
        R = 1 if bytes_ >= 126e6 else int(-(-3 * 126e6 // bytes_))
        sets = []
        for r in range(R):
            A, B = ki.operands(m, n, k, batch, dtype, "unif", seed=0, entry0=r * batch, device="cuda")
            C = torch.empty(batch * m * n, dtype=A.dtype, device="cuda")
            sets.append((A, B, C))
        cands = []
        for algo, p in CANDIDATES["f64" if dtype == "f64" else "16"]:
            def fn(i, algo=algo, p=p):
                A, B, C = sets[i]
                kami.gemm_strided_batched(m, n, k, batch, dtype, "row", A, B, C, algo=algo, p=p,
                                          stream=torch.cuda.current_stream())
            try:
                fn(0)
                torch.cuda.synchronize()
            except kami.KamiError:
                continue
            kern = kami.last_kernel()
            ms = time_call(fn, a.steps, sets)
            tf = 2.0 * m * n * k * batch / (ms * 1e-3) / 1e12
            cands.append({"algo": algo, "p": p, "kernel": kern, "tflops": tf, "ms": ms})
            print(f"{name:22s} {algo:8s} p={p:<2d} {kern:40s} {tf:9.2f} TF/s", flush=True)
        res.append({"cfg": name, "dtype": dtype, "m": m, "n": n, "k": k, "batch": batch, "candidates": cands})
        del sets
        torch.cuda.empty_cache()
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump({"note": "tools/variant_sweep_r2.py: CUDA-graph timing, median of 3 replays of 20 launches",
               "gpu": torch.cuda.get_device_name(), "configs": res}, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
