"""Reproducer for one pointer-array case: python tools/ptr_repro.py m n k batch dtype layout"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import kami_inputs as ki
import paper_conf_sc_wangdltsl25_b200 as kami
m, n, k, batch = (int(x) for x in sys.argv[1:5])
dtype, layout = sys.argv[5], sys.argv[6]
A, B = ki.operands(m, n, k, batch, dtype, "unif", seed=11)
dA, dB = A.cuda().view(batch, -1), B.cuda().view(batch, -1)
dC = torch.zeros(batch, m * n, dtype=A.dtype, device="cuda")
pa = torch.tensor([dA[i].data_ptr() for i in range(batch)], dtype=torch.int64, device="cuda")
pb = torch.tensor([dB[i].data_ptr() for i in range(batch)], dtype=torch.int64, device="cuda")
pc = torch.tensor([dC[i].data_ptr() for i in range(batch)], dtype=torch.int64, device="cuda")
print("A base", hex(dA.data_ptr()), "B", hex(dB.data_ptr()), "C", hex(dC.data_ptr()))
kami.gemm_batched(m, n, k, batch, dtype, layout, pa, pb, pc)
torch.cuda.synchronize()
print("ok", kami.last_kernel())
