"""Thin-m shapes: the transposed-product kernel (1d_xt) against the SS tcgen05
kernel (1d, p = 0), the warp-level 1D and AUTO, bf16, 125 000 entries per shape
(the BF16 sweep's batch, inputs larger than L2), CUDA events over 10 reps.
    python tools/xt_ab.py [--dtype bf16] [--batch 125000]"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_sc_wangdltsl25_b200 as kami  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--dtype", default="bf16")
ap.add_argument("--batch", type=int, default=125000)
ap.add_argument("--reps", type=int, default=10)
a = ap.parse_args()
hbm = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
td = torch.bfloat16 if a.dtype == "bf16" else torch.float16
for m in (16, 32):
    for n in (64, 128, 192, 256):
        for k in (16, 32, 64):
            A = torch.empty(a.batch * m * k, dtype=td, device="cuda").uniform_(-1, 1)
            B = torch.empty(a.batch * k * n, dtype=td, device="cuda").uniform_(-1, 1)
            C = torch.empty(a.batch * m * n, dtype=td, device="cuda")
            byts = (m * k + k * n + m * n) * 2.0 * a.batch
            row = {"m": m, "n": n, "k": k}
            for algo, p in (("1d_xt", 0), ("1d", 0), ("auto", 0)):
                try:
                    run = lambda: kami.gemm_strided_batched(m, n, k, a.batch, a.dtype, "row", A, B, C, algo=algo, p=p)  # noqa: E731
                    for _ in range(3):
                        run()
                    torch.cuda.synchronize()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    for _ in range(a.reps):
                        run()
                    e1.record()
                    torch.cuda.synchronize()
                    t = e0.elapsed_time(e1) / a.reps * 1e-3
                    row[algo] = round(byts / t / 1e9 / hbm, 3)
                    row[algo + "_k"] = kami.last_kernel()
                except kami.KamiError as ex:
                    row[algo] = str(ex)[:40]
            print(json.dumps(row), flush=True)
            del A, B, C
