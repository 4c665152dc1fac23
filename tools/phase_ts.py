"""Run one tcgen05 launch per configuration after an L2 flush with the
phase-timing build (KAMI_LIB=.../libkami_ts.so, -DKAMI_PHASE_TIMING): CTA 0
prints clock64 deltas of its pipeline phases."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import kami_inputs as ki  # noqa: E402
import paper_conf_sc_wangdltsl25_b200 as kami  # noqa: E402

torch.cuda.set_device(0)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for (m, batch) in [(16, 8), (16, 1024), (32, 65536), (64, 8192)]:
    A, B = ki.operands(m, m, m, batch, "f16", "unif", seed=0, device="cuda")
    C = torch.empty(batch * m * m, dtype=torch.float16, device="cuda")
    for rep in range(4):
        flush.zero_()
        torch.cuda.synchronize()
        print(f"f16 {m}^3 x{batch} rep {rep}: ", end="", flush=True)
        kami.gemm_strided_batched(m, m, m, batch, "f16", "row", A, B, C)
        torch.cuda.synchronize()
