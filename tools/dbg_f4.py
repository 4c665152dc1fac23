"""Debug print for the TF32 path: one small entry, kernel vs oracle, with
idesc variants (KAMI_TC_IDESC_XOR) in subprocesses."""
import os
import subprocess
import sys
import numpy as np
import torch

if len(sys.argv) > 1:
    import kami_inputs as ki
    import oracle
    import paper_conf_sc_wangdltsl25_b200 as kami
    np.set_printoptions(linewidth=200, precision=3, suppress=True)
    m = n = k = 16
    batch = 2
    dtype = "tf32"
    A, B = ki.operands(m, n, k, batch, dtype, "int", seed=0)
    C0 = torch.ones(batch * m * n, dtype=torch.float32)
    dC = C0.cuda()
    kami.gemm_strided_batched_axpby(m, n, k, batch, dtype, "row", 1.0, A.cuda(), B.cuda(), 1.0, dC)
    torch.cuda.synchronize()
    got = dC.cpu().double().view(batch, m, n).numpy()
    ref = oracle.gemm(m, n, k, batch, dtype, "row", ki.as_bits(A), ki.as_bits(B)) + 1
    Ad = A.double().view(batch, m, k).numpy()
    Bd = B.double().view(batch, k, n).numpy()
    print("xor", os.environ.get("KAMI_TC_IDESC_XOR"), "mismatch", int((got != ref).sum()), "of", got.size,
          "nonone", int((got != 1).sum()), "hypAtB", int((got != Ad.transpose(0, 2, 1) @ Bd + 1).sum()),
          "hypABt", int((got != Ad @ Bd.transpose(0, 2, 1) + 1).sum()))
    print(got[0, :3, :6], ref[0, :3, :6])
else:
    for x in ["0", "0x80", "0x400", "0x480", "0x100", "0x10000", "0x8000", "0x18000", "0x300"]:
        env = dict(os.environ, KAMI_TC_IDESC_XOR=x, PYTHONPATH=".")
        r = subprocess.run([sys.executable, __file__, "go"], env=env, capture_output=True, text=True, timeout=120)
        print(r.stdout[-1500:], r.stderr[-600:])
