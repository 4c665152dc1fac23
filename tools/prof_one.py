"""Run one workload's kernel a few times (for ncu).  Not a benchmark.

    python tools/prof_one.py --workload f16-64 [--algo 1d --p 4] [--iters 5]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import kami_inputs as ki  # noqa: E402
import paper_conf_sc_wangdltsl25_b200 as kami  # noqa: E402
from bench import parse_workload  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="f16-64")
ap.add_argument("--algo", default="auto")
ap.add_argument("--p", type=int, default=0)
ap.add_argument("--iters", type=int, default=5)
ap.add_argument("--batch", type=int, default=0)
a = ap.parse_args()
dtype, m, n, k, batch, _ = parse_workload(a.workload)
if a.batch:
    batch = a.batch
A, B = ki.operands(m, n, k, batch, dtype, "unif", device="cuda")
C = torch.zeros(batch * m * n, dtype=ki.TORCH_DTYPES[ki.OUT_DTYPE[dtype]], device="cuda")
for _ in range(a.iters):
    if "upd" in a.workload:
        kami.gemm_strided_batched_axpby(m, n, k, batch, dtype, "row", 1.0, A, B, 1.0, C)
    else:
        kami.gemm_strided_batched(m, n, k, batch, dtype, "row", A, B, C, algo=a.algo, p=a.p)
torch.cuda.synchronize()
print(kami.last_kernel())
