"""One small launch per kernel instantiation, for compute-sanitizer
(memcheck / racecheck / synccheck).

    compute-sanitizer --tool racecheck python tools/sanitize_cases.py

Every case runs with the grid capped at 2 CTAs, so each persistent CTA wraps
its rings (TMA stages, TMEM accumulators, A slots, C staging buffers) several
times -- the mbarrier / per-atom wait / TMEM handoffs are what the tools
check.  Results are compared with the oracle so a run that silently computes
garbage under the tool is also caught.  Prints one line per case.
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import kami_inputs as ki  # noqa: E402
import oracle  # noqa: E402
import paper_conf_sc_wangdltsl25_b200 as kami  # noqa: E402

CASES = [
    # (dtype, m, n, k, batch, algo, p)
    ("f16", 64, 64, 64, 24, "1d", 0),        # tc16 plain
    ("bf16", 128, 128, 64, 8, "1d", 0),      # tc16 per-atom split stores
    ("f16", 192, 64, 64, 7, "1d", 0),        # tc16 tail packing
    ("f16", 16, 256, 16, 9, "1d", 0),        # tc16 replicated thin m, per-warp stores
    ("f16", 32, 32, 32, 70, "1d", 0),        # tc16 U = 2 sub-tiles
    ("f16", 256, 256, 16, 4, "1d", 0),       # tc16 low-rank, 2 m-tiles
    ("tf32", 64, 64, 64, 16, "1d", 0),       # tc16 TF32 (B transposer warps)
    ("e4m3", 64, 64, 64, 16, "1d", 0),       # tc16 FP8
    ("f16", 64, 64, 64, 24, "1d_tmem", 0),   # TS 1D (A in TMEM)
    ("bf16", 128, 128, 128, 8, "3d_tmem", 0),  # TS 3D
    ("f16", 16, 16, 16, 64, "auto", 0),      # warp-level HMMA 1D
    ("f16", 64, 64, 64, 16, "3d", 0),        # warp-level 3D (layer reduction)
    ("f64", 32, 32, 32, 40, "2d", 0),        # warp-level DMMA 2D
    ("f64", 64, 64, 64, 16, "1d_tma", 0),    # FP64 TMA broadcast
    ("f64", 96, 40, 72, 12, "auto", 0),      # FP64 general (dmma_gen)
    ("bf16", 16, 128, 16, 40, "1d_xt", 0),   # transposed product, m = 16 (two epilogue warpgroups)
    ("f16", 32, 192, 32, 20, "1d_xt", 0),    # transposed product, m = 32, 64-column last tile
]


def run(dtype, m, n, k, batch, algo, p):
    A, B = ki.operands(m, n, k, batch, dtype, "int", seed=3)
    od = ki.OUT_DTYPE[dtype]
    C = torch.zeros(batch * m * n, dtype=ki.TORCH_DTYPES[od], device="cuda")
    kami.gemm_strided_batched(m, n, k, batch, dtype, "row", A.cuda(), B.cuda(), C, algo=algo, p=p)
    torch.cuda.synchronize()
    ref = oracle.round_to(oracle.gemm(m, n, k, batch, dtype, "row", ki.as_bits(A), ki.as_bits(B)), od)
    got = ki.as_bits(C.cpu()).reshape(-1)
    ok = np.array_equal(got.reshape(-1), np.asarray(ref).reshape(-1))
    return ok, kami.last_kernel()


def main():
    only = sys.argv[1:]
    bad = 0
    with kami.grid_cap(2):
        for case in CASES:
            if only and case[5] not in only:
                continue
            ok, kern = run(*case)
            bad += not ok
            print(f"{'OK ' if ok else 'BAD'} {kern:45s} {case}", flush=True)
    # pointer arrays (address-space TMA views) and variable sizes
    with kami.grid_cap(2):
        m = n = k = 64
        batch = 24
        A, B = ki.operands(m, n, k, batch, "f16", "int", seed=4)
        dA, dB = A.cuda().view(batch, -1), B.cuda().view(batch, -1)
        dC = torch.zeros(batch, m * n, dtype=torch.float16, device="cuda")
        pa = torch.tensor([dA[i].data_ptr() for i in range(batch)], dtype=torch.int64, device="cuda")
        pb = torch.tensor([dB[i].data_ptr() for i in range(batch)], dtype=torch.int64, device="cuda")
        pc = torch.tensor([dC[i].data_ptr() for i in range(batch)], dtype=torch.int64, device="cuda")
        kami.gemm_batched(m, n, k, batch, "f16", "row", pa, pb, pc)
        torch.cuda.synchronize()
        ref = oracle.round_to(oracle.gemm(m, n, k, batch, "f16", "row", ki.as_bits(A), ki.as_bits(B)), "f16")
        ok = np.array_equal(ki.as_bits(dC.cpu()).reshape(-1), ref.reshape(-1))
        bad += not ok
        print(f"{'OK ' if ok else 'BAD'} {kami.last_kernel():45s} pointer arrays 64^3 x 24", flush=True)
    # variable sizes, class-sorted (>= 256 entries: pre-pass + unit records)
    with kami.grid_cap(2):
        rng = np.random.default_rng(7)
        batch = 300
        sz = rng.choice(np.array([16, 32, 64]), size=(batch, 3))
        mats = [ki.operands(int(a), int(b), int(c), 1, "f16", "int", seed=100 + i) for i, (a, b, c) in enumerate(sz)]
        dA = [x[0].cuda() for x in mats]
        dB = [x[1].cuda() for x in mats]
        dC = [torch.zeros(int(a) * int(b), dtype=torch.float16, device="cuda") for a, b, _ in sz]
        ptr = lambda ts: torch.tensor([t.data_ptr() for t in ts], dtype=torch.int64, device="cuda")  # noqa: E731
        dm, dn, dk = (torch.tensor(sz[:, i], dtype=torch.int32, device="cuda") for i in range(3))
        kami.gemm_vbatched(batch, dm, dn, dk, 64, 64, 64, "f16", "row", ptr(dA), ptr(dB), ptr(dC))
        torch.cuda.synchronize()
        ok = True
        for i, (a, b, c) in enumerate(sz):
            A, B = mats[i]
            ref = oracle.round_to(oracle.gemm(int(a), int(b), int(c), 1, "f16", "row", ki.as_bits(A), ki.as_bits(B)),
                                  "f16")
            ok &= np.array_equal(ki.as_bits(dC[i].cpu()).reshape(-1), np.asarray(ref).reshape(-1))
        bad += not ok
        print(f"{'OK ' if ok else 'BAD'} {kami.last_kernel():45s} variable sizes {{16,32,64}}^3 x {batch}", flush=True)
    # SpMM (A blocks by TMA, absent blocks zeroed in shared memory)
    with kami.grid_cap(2):
        m, n, k, batch = 128, 96, 128, 12
        rp, cb, v, B = ki.bsr_operands(m, n, k, batch, "f16", density=0.5, dist="int", seed=8)
        C = torch.zeros(batch * m * n, dtype=torch.float16, device="cuda")
        kami.spmm_bsr_strided_batched(m, n, k, batch, "f16", rp.cuda(), cb.cuda(), v.cuda(), B.cuda(), C)
        torch.cuda.synchronize()
        ref = oracle.round_to(oracle.spmm_bsr(m, n, k, batch, "f16", rp.numpy(), cb.numpy(), ki.as_bits(v),
                                              ki.as_bits(B)), "f16")
        ok = np.array_equal(ki.as_bits(C.cpu()).reshape(-1), np.asarray(ref).reshape(-1))
        bad += not ok
        print(f"{'OK ' if ok else 'BAD'} {kami.last_kernel():45s} SpMM 128x96x128 x 12, 50 % blocks", flush=True)
    print("sanitize_cases:", "all OK" if not bad else f"{bad} BAD")
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
