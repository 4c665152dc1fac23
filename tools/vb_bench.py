"""Throughput of the pointer-array / variable-size path (tc16_vb.cu).

    python tools/vb_bench.py [--mode ptr|vb] [--dtype f16] [--shape 64x64x64] [--batch 65536]

ptr: uniform-size pointer-array batch (entries scattered: pointers permuted);
vb : mixed orders drawn from {16,32,64,128,192,256}^3 (BF16 sweep grid), the
     "one mixed-size batch" reading of BASELINE configs[4].
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import kami_inputs as ki  # noqa: E402
import paper_conf_sc_wangdltsl25_b200 as kami  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--mode", default="ptr")
ap.add_argument("--dtype", default="f16")
ap.add_argument("--shape", default="64x64x64")
ap.add_argument("--batch", type=int, default=65536)
ap.add_argument("--reps", type=int, default=10)
ap.add_argument("--density", type=float, default=0.5)
ap.add_argument("--orders", default="16,32,64,128,192,256", help="vb mode: the order set")
ap.add_argument("--nmax", type=int, default=256, help="vb mode: max_n passed to the call")
ap.add_argument("--morders", default="", help="vb mode: m's own order set (default --orders)")
ap.add_argument("--norders", default="", help="vb mode: n's own order set")
ap.add_argument("--korders", default="", help="vb mode: k's own order set")
ap.add_argument("--algo", default="auto", help="zmorton mode: auto / 1d / 2d")
ap.add_argument("--sortalloc", action="store_true", help="vb mode: entries allocated in (m, n, k) class order")
ap.add_argument("--noperm", action="store_true", help="ptr mode: pointers in entry order (no scatter)")
a = ap.parse_args()
hbm = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
    os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
if a.mode == "spmm":
    m, n, k = (int(x) for x in a.shape.split("x"))
    rp, cb, v, B = ki.bsr_operands(m, n, k, a.batch, a.dtype, density=a.density, device="cuda")
    C = torch.empty(a.batch * m * n, dtype=B.dtype, device="cuda")
    run = lambda: kami.spmm_bsr_strided_batched(m, n, k, a.batch, a.dtype, rp, cb, v, B, C)  # noqa: E731
    nnzb = float(rp[:, -1].sum())
    flops = 2.0 * nnzb * 256 * n  # useful (sparse) flops
    byts = nnzb * (512 + 4) + a.batch * ((m // 16 + 1) * 4 + (k * n + m * n) * 2)
elif a.mode == "zmorton":
    # the same block-sparse matrices in Z-Morton block storage, built here with
    # torch (codes = interleaved block row / column bits, sorted per entry)
    m, n, k = (int(x) for x in a.shape.split("x"))
    rp, cb, v, B = ki.bsr_operands(m, n, k, a.batch, a.dtype, density=a.density, device="cuda")
    mb = m // 16
    cnt = (rp[:, 1:] - rp[:, :-1]).long()
    br = torch.repeat_interleave(torch.arange(mb, device="cuda").repeat(a.batch), cnt.reshape(-1))
    nnz = rp[:, -1].long()
    ent = torch.repeat_interleave(torch.arange(a.batch, device="cuda"), nnz)
    slot = torch.arange(int(nnz.sum()), device="cuda") - torch.repeat_interleave(torch.cumsum(nnz, 0) - nnz, nnz)
    bc = cb[ent, slot].long()
    z = torch.zeros_like(br)
    for t in range(4):
        z |= ((bc >> t) & 1) << (2 * t)
        z |= ((br >> t) & 1) << (2 * t + 1)
    key = ent * 1024 + z
    order = torch.argsort(key)
    zc = torch.full_like(cb, -1)
    newslot = slot  # ranks within the entry after sorting
    ent_s, z_s, old_s = ent[order], z[order], slot[order]
    rank = torch.arange(len(order), device="cuda") - torch.repeat_interleave(torch.cumsum(nnz, 0) - nnz, nnz)
    zc[ent_s, rank] = z_s.int()
    zv = torch.zeros_like(v)
    zv[ent_s, rank] = v[ent_s, old_s]
    nz = nnz.int()
    C = torch.empty(a.batch * m * n, dtype=B.dtype, device="cuda")
    run = lambda: kami.spmm_zmorton_strided_batched(m, n, k, a.batch, a.dtype, nz, zc, zv, B, C, algo=a.algo)  # noqa: E731
    nnzb = float(nnz.sum())
    flops = 2.0 * nnzb * 256 * n
    byts = nnzb * (512 + 4) + a.batch * (4 + (k * n + m * n) * 2)
elif a.mode == "ptr":
    m, n, k = (int(x) for x in a.shape.split("x"))
    A, B = ki.operands(m, n, k, a.batch, a.dtype, "unif", device="cuda")
    C = torch.empty(a.batch * m * n, dtype=A.dtype, device="cuda")
    perm = torch.arange(a.batch, device="cuda") if a.noperm else torch.randperm(a.batch, device="cuda")
    es = A.element_size()
    pa = (A.data_ptr() + perm * (m * k * es)).to(torch.int64)
    pb = (B.data_ptr() + perm * (k * n * es)).to(torch.int64)
    pc = (C.data_ptr() + perm * (m * n * es)).to(torch.int64)
    run = lambda: kami.gemm_batched(m, n, k, a.batch, a.dtype, "row", pa, pb, pc)  # noqa: E731
    flops = 2.0 * m * n * k * a.batch
    byts = (m * k + k * n + m * n) * es * a.batch
else:
    rng = np.random.default_rng(0)
    orders = np.array([int(x) for x in a.orders.split(",")])
    sz = rng.choice(orders, size=(a.batch, 3))
    for i, o in enumerate((a.morders, a.norders, a.korders)):
        if o:
            sz[:, i] = rng.choice(np.array([int(x) for x in o.split(",")]), size=a.batch)
    if a.sortalloc:  # memory order = the kernel's class-sorted unit order (address locality experiment)
        sz = sz[np.lexsort((sz[:, 2], sz[:, 1], sz[:, 0]))]
    mm, nn, kk = sz[:, 0], sz[:, 1], sz[:, 2]
    es = 8 if a.dtype == "f64" else 2
    offA = np.concatenate([[0], np.cumsum(mm * kk)])
    offB = np.concatenate([[0], np.cumsum(kk * nn)])
    offC = np.concatenate([[0], np.cumsum(mm * nn)])
    A = torch.empty(int(offA[-1]), dtype={"bf16": torch.bfloat16, "f64": torch.float64}.get(a.dtype, torch.float16),
                    device="cuda")
    B = torch.empty(int(offB[-1]), dtype=A.dtype, device="cuda")
    A.uniform_(-1, 1)
    B.uniform_(-1, 1)
    C = torch.empty(int(offC[-1]), dtype=A.dtype, device="cuda")
    dm = torch.tensor(mm, dtype=torch.int32, device="cuda")
    dn = torch.tensor(nn, dtype=torch.int32, device="cuda")
    dk = torch.tensor(kk, dtype=torch.int32, device="cuda")
    pa = torch.tensor(A.data_ptr() + offA[:-1] * es, dtype=torch.int64, device="cuda")
    pb = torch.tensor(B.data_ptr() + offB[:-1] * es, dtype=torch.int64, device="cuda")
    pc = torch.tensor(C.data_ptr() + offC[:-1] * es, dtype=torch.int64, device="cuda")
    run = lambda: kami.gemm_vbatched(a.batch, dm, dn, dk, 256, a.nmax, 256, a.dtype, "row", pa, pb, pc)  # noqa: E731
    flops = float((2.0 * mm * nn * kk).sum())
    byts = float(((mm * kk + kk * nn + mm * nn) * es).sum())
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
print(json.dumps({"mode": a.mode, "dtype": a.dtype, "shape": a.shape, "batch": a.batch, "tflops": flops / t / 1e12,
                  "gbs": byts / t / 1e9, "frac_hbm": byts / t / 1e9 / hbm, "ms": t * 1e3,
                  "kernel": kami.last_kernel()}))
