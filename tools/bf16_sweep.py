"""BASELINE.json configs[4]: BF16 sweep over m, n, k in {16, 32, 64, 128, 192, 256}.

    python tools/bf16_sweep.py [--orders 16,32,64,128,192,256] [--squares-only]
                               [--global-batch 1000000] [--gpus-share 8] [--out profiles/r1/bf16_sweep.json]

Timing: the reps launches are captured in one CUDA graph and replayed
between two CUDA events (as bench.py).  Reading (R16/SURVEY 8(d)): uniform size per point, 10^6 entries per
point globally, sharded over 8 B200 -> 125 000 entries per GPU; one GPU runs
its shard (chunked when the shard does not fit the memory budget).  Each point
reports TFLOP/s and the fraction of its HBM roofline (measured copy
bandwidth).  Parity of these points is checked by the GPU tests
(tests/test_gpu_fullsize.py), not here: tools never run the oracle.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import kami_inputs as ki  # noqa: E402
import paper_conf_sc_wangdltsl25_b200 as kami  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--orders", default="16,32,64,128,192,256")
    ap.add_argument("--squares-only", action="store_true")
    ap.add_argument("--global-batch", type=int, default=1000000)
    ap.add_argument("--gpus-share", type=int, default=8)
    ap.add_argument("--mem-budget-gb", type=float, default=40.0)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r1", "bf16_sweep.json"))
    a = ap.parse_args()
    orders = [int(x) for x in a.orders.split(",")]
    pts = [(m, n, k) for m in orders for n in orders for k in orders]
    if a.squares_only:
        pts = [(s, s, s) for s in orders]
    else:  # squares first
        pts = [(s, s, s) for s in orders] + [p for p in pts if not (p[0] == p[1] == p[2])]
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {"hbm_gbs": 6650.0}
    hbm = peaks["hbm_gbs"]
    shard = a.global_batch // a.gpus_share
    results = []
    for (m, n, k) in pts:
        per_entry = (m * k + k * n + m * n) * 2
        chunk = min(shard, int(a.mem_budget_gb * 1e9 // per_entry))
        A, B = ki.operands(m, n, k, chunk, "bf16", "unif", seed=0, device="cuda")
        C = torch.empty(chunk * m * n, dtype=torch.bfloat16, device="cuda")
        for _ in range(2):
            kami.gemm_strided_batched(m, n, k, chunk, "bf16", "row", A, B, C)
        torch.cuda.synchronize()
        # the reps x (shard / chunk) launches are captured in one CUDA graph and
        # replayed between two events, as bench.py times its steps: eager
        # launches put the host's per-call work (planning, tensor-map encode)
        # between kernels of a few tens of microseconds (r1/r2 sweeps before
        # this change: 16^3 0.69 eager vs 0.83 in a graph)
        n_launch = 0

        def body():
            nonlocal n_launch
            for _ in range(a.reps):
                done = 0
                while done < shard:  # the shard is streamed through the resident chunk
                    nb = min(chunk, shard - done)
                    kami.gemm_strided_batched(m, n, k, nb, "bf16", "row", A, B, C)
                    done += nb
                    n_launch += 1
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):  # (the binding launches on torch's current = capture stream)
            body()
        g.replay()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        t = e0.elapsed_time(e1) * 1e-3 / a.reps
        flops = 2.0 * m * n * k * shard
        bytes_ = per_entry * shard
        roof = min(hbm * 1e9 * flops / bytes_, 2250e12)
        r = {"m": m, "n": n, "k": k, "entries_per_gpu": shard, "chunk": chunk, "tflops": flops / t / 1e12,
             "gbs": bytes_ / t / 1e9, "roofline_tflops": roof / 1e12, "frac": flops / t / roof,
             "ms": t * 1e3, "kernel": kami.last_kernel(), "launches_per_rep": n_launch // a.reps}
        results.append(r)
        print(json.dumps(r), flush=True)
        del A, B, C
        torch.cuda.empty_cache()
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump({"config": "BASELINE.json configs[4] BF16 sweep, 1e6 entries/point over 8 GPUs -> per-GPU shard",
               "hbm_gbs_peak": hbm, "points": results, "when": time.strftime("%Y-%m-%dT%H:%M:%S")},
              open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
