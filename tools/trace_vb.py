"""Role trace of the pointer-array tcgen05 kernel (tc16_vb.cu, KAMI_VB_DEBUG=4):
clock64 stamps of CTA 0's producer / MMA / epilogue events per stage or unit.

    python tools/trace_vb.py [order] [batch]
"""
import ctypes
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["KAMI_VB_DEBUG"] = "4"
import kami_inputs as ki  # noqa: E402
import paper_conf_sc_wangdltsl25_b200 as kami  # noqa: E402

m = n = k = int(sys.argv[1]) if len(sys.argv) > 1 else 64
batch = int(sys.argv[2]) if len(sys.argv) > 2 else 32768
A, B = ki.operands(m, n, k, batch, "f16", "unif", device="cuda")
C = torch.empty(batch * m * n, dtype=A.dtype, device="cuda")
es = 2
idx = torch.arange(batch, device="cuda")
pa = (A.data_ptr() + idx * (m * k * es)).to(torch.int64)
pb = (B.data_ptr() + idx * (k * n * es)).to(torch.int64)
pc = (C.data_ptr() + idx * (m * n * es)).to(torch.int64)
for _ in range(3):
    kami.gemm_batched(m, n, k, batch, "f16", "row", pa, pb, pc)
torch.cuda.synchronize()
out = (ctypes.c_longlong * (8 * 1024))()
kami.lib().kami_debug_vb_trace(out)
t = np.array(out).reshape(8, 1024).astype(np.int64)
t0 = t[0, 0]
names = ["prod_empty_ok", "prod_issued", "mma_full_ok", "mma_commit_tfull", "epi_tfull_ok", "epi_done",
         "mma_tempty_ok"]
for i in range(0, 24):
    print(i, " ".join(f"{names[e]}={t[e, i] - t0}" for e in range(7)))
# steady-state periods (events 20..60)
for e in range(7):
    v = t[e, 20:60]
    v = v[v > 0]
    if len(v) > 2:
        print(f"{names[e]:18s} period {np.median(np.diff(v)):.0f} cycles")
pi = t[1, 20:60] - t[0, 20:60]
print("producer issue time per stage (median)", np.median(pi))
