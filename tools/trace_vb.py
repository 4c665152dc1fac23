import ctypes, os, sys, torch, numpy as np
sys.path.insert(0, os.getcwd())
os.environ["KAMI_VB_DEBUG"] = "4"
import kami_inputs as ki, paper_conf_sc_wangdltsl25_b200 as kami
m = n = k = 64; batch = 32768
A, B = ki.operands(m, n, k, batch, "f16", "unif", device="cuda")
C = torch.empty(batch * m * n, dtype=A.dtype, device="cuda")
es = 2
idx = torch.arange(batch, device="cuda")
pa = (A.data_ptr() + idx * (m * k * es)).to(torch.int64); pb = (B.data_ptr() + idx * (k * n * es)).to(torch.int64); pc = (C.data_ptr() + idx * (m * n * es)).to(torch.int64)
for _ in range(3): kami.gemm_batched(m, n, k, batch, "f16", "row", pa, pb, pc)
torch.cuda.synchronize()
out = (ctypes.c_longlong * (8 * 1024))()
kami.lib().kami_debug_vb_trace(out)
t = np.array(out).reshape(8, 1024).astype(np.int64)
t0 = t[0, 0]
names = ["prod_empty_ok", "prod_issued", "mma_full_ok", "mma_commit_tfull", "epi_tfull_ok", "epi_done", "mma_tempty_ok"]
for i in range(0, 40, 1):
    print(i, " ".join(f"{names[e]}={t[e, i] - t0}" for e in range(7)))
