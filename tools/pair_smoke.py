"""Smallest CTA-pair launch, checked against the oracle (first run of a new kernel)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import kami_inputs as ki, oracle
import paper_conf_sc_wangdltsl25_b200 as kami
for (m, n, k, batch) in [(256, 64, 16, 1), (256, 64, 16, 2), (256, 256, 256, 3), (224, 96, 40, 5)]:
    A, B = ki.operands(m, n, k, batch, "f16", "int", seed=1)
    C = torch.full((batch * m * n,), float("nan"), dtype=torch.float16, device="cuda")
    kami.gemm_strided_batched(m, n, k, batch, "f16", "row", A.cuda(), B.cuda(), C, algo="2d_pair")
    torch.cuda.synchronize()
    ref = oracle.round_to(oracle.gemm(m, n, k, batch, "f16", "row", ki.as_bits(A), ki.as_bits(B)), "f16")
    got = ki.as_bits(C.cpu()).reshape(-1)
    bad = np.flatnonzero(got != ref.reshape(-1))
    print((m, n, k, batch), kami.last_kernel(), "mismatches", bad.size, "first", bad[:5], flush=True)
