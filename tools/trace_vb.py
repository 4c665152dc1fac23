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

mix = len(sys.argv) > 1 and (sys.argv[1] == "mix" or sys.argv[1].startswith("u"))
uni = int(sys.argv[1][1:]) if mix and sys.argv[1].startswith("u") else 0  # "u64": uniform 64^3 via vbatched
m = n = k = 64 if mix else (int(sys.argv[1]) if len(sys.argv) > 1 else 64)
batch = int(sys.argv[2]) if len(sys.argv) > 2 else 32768
es = 2
if mix:  # tools/vb_bench.py --mode vb recipe: orders from {16,...,256}^3
    rng = np.random.default_rng(0)
    sz = rng.choice(np.array([uni] if uni else [16, 32, 64, 128, 192, 256]), size=(batch, 3))
    mm, nn, kk = sz[:, 0], sz[:, 1], sz[:, 2]
    offA = np.concatenate([[0], np.cumsum(mm * kk)])
    offB = np.concatenate([[0], np.cumsum(kk * nn)])
    offC = np.concatenate([[0], np.cumsum(mm * nn)])
    A = torch.rand(int(offA[-1]), device="cuda").half()
    B = torch.rand(int(offB[-1]), device="cuda").half()
    C = torch.empty(int(offC[-1]), dtype=A.dtype, device="cuda")
    dm, dn, dk = (torch.tensor(x, dtype=torch.int32, device="cuda") for x in (mm, nn, kk))
    pa = torch.tensor(A.data_ptr() + offA[:-1] * es, dtype=torch.int64, device="cuda")
    pb = torch.tensor(B.data_ptr() + offB[:-1] * es, dtype=torch.int64, device="cuda")
    pc = torch.tensor(C.data_ptr() + offC[:-1] * es, dtype=torch.int64, device="cuda")
    run = lambda: kami.gemm_vbatched(batch, dm, dn, dk, 256, 256, 256, "f16", "row", pa, pb, pc)  # noqa: E731
    # CTA 0's live units in order (units u = 0, grid, 2 grid, ...; u = entry * 2 + m-tile)
    grid = 148
    live = [(e, mt) for u in range(0, 2 * batch, grid) for e, mt in [divmod(u, 2)] if mt * 128 < mm[e]]
    print("CTA 0 live units (m,n,k,mt):", [(int(mm[e]), int(nn[e]), int(kk[e]), mt) for e, mt in live[:30]])
else:
    A, B = ki.operands(m, n, k, batch, "f16", "unif", device="cuda")
    C = torch.empty(batch * m * n, dtype=A.dtype, device="cuda")
    idx = torch.arange(batch, device="cuda")
    pa = (A.data_ptr() + idx * (m * k * es)).to(torch.int64)
    pb = (B.data_ptr() + idx * (k * n * es)).to(torch.int64)
    pc = (C.data_ptr() + idx * (m * n * es)).to(torch.int64)
    run = lambda: kami.gemm_batched(m, n, k, batch, "f16", "row", pa, pb, pc)  # noqa: E731
for _ in range(3):
    run()
torch.cuda.synchronize()
out = (ctypes.c_longlong * (8 * 1024))()
kami.lib().kami_debug_vb_trace(out)
t = np.array(out).reshape(8, 1024).astype(np.int64)
t0 = t[0, 0]
names = ["prod_empty_ok", "prod_issued", "mma_full_ok", "mma_commit_tfull", "epi_tfull_ok", "epi_done",
         "mma_tempty_ok"]
for i in range(0, 40):
    print(i, " ".join(f"{names[e]}={t[e, i] - t0}" for e in range(7)))
# steady-state periods (events 20..60)
for e in range(7):
    v = t[e, 20:60]
    v = v[v > 0]
    if len(v) > 2:
        print(f"{names[e]:18s} period {np.median(np.diff(v)):.0f} cycles")
pi = t[1, 20:60] - t[0, 20:60]
print("producer issue time per stage (median)", np.median(pi))
lat = t[2, 20:200] - t[1, 20:200]
lat = lat[(t[2, 20:200] > 0) & (t[1, 20:200] > 0)]
print("issue -> MMA start per stage (median / p90)", np.median(lat), np.percentile(lat, 90))
wait_slot = t[0, 20:200] - t[1, 19:199]
print("producer wait for a free slot after the previous issue (median)", np.median(wait_slot[wait_slot > -1e12]))
n_st = int((t[1] > 0).sum())
print("stages traced", n_st, "span cycles", int(t[1, n_st - 1] - t[1, 0]), "per stage", (t[1, n_st - 1] - t[1, 0]) / max(1, n_st - 1))
