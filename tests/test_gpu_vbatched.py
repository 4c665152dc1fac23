"""Pointer-array and variable-size batches (PAPER.md L523
"supports various matrix orders in a batch") on the LDG-fed tcgen05 kernel,
against the oracle entry by entry."""
import numpy as np
import pytest
import torch

import kami_inputs as ki
import oracle
import paper_conf_sc_wangdltsl25_b200 as kami

pytestmark = pytest.mark.gpu


def _tol(dtype, k):
    return {"f16": 2.0 ** -11, "bf16": 2.0 ** -8}[dtype] + k * 2.0 ** -23


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("shape", [(16, 16, 16), (32, 32, 32), (64, 64, 64), (48, 80, 40), (256, 256, 8), (192, 64, 256),
                                   (128, 256, 24), (32, 16, 256)])
def test_pointer_array_all_sizes(dtype, shape):
    m, n, k = shape
    batch = 23
    for dist, layout in (("unif", "row"), ("int", "col")):
        A, B = ki.operands(m, n, k, batch, dtype, dist, seed=11)
        dA, dB = A.cuda().view(batch, -1), B.cuda().view(batch, -1)
        dC = torch.zeros(batch, m * n, dtype=A.dtype, device="cuda")
        perm = torch.randperm(batch).tolist()
        pa = torch.tensor([dA[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
        pb = torch.tensor([dB[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
        pc = torch.tensor([dC[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
        kami.gemm_batched(m, n, k, batch, dtype, layout, pa, pb, pc)
        torch.cuda.synchronize()
        # square orders 16 / 32 go to the warp-level HMMA 1D (dispatch rule), the rest to tcgen05
        want = "kami_warp_ca_1d" if (m == n == k and m <= 32) else "kami_tc16_vb_kernel"
        assert kami.last_kernel().startswith(want), kami.last_kernel()
        Cref, S = oracle.gemm(m, n, k, batch, dtype, layout, ki.as_bits(A), ki.as_bits(B), with_scale=True)
        got_bits = oracle.to_row_major(ki.as_bits(dC.cpu()), batch, m, n, layout)
        if dist == "int":
            assert np.array_equal(got_bits, oracle.round_to(Cref, dtype).reshape(batch, m, n))
        else:
            got = oracle.decode(got_bits.reshape(-1), dtype).reshape(batch, m, n)
            assert oracle.normalised_error(got, Cref, S) <= _tol(dtype, k)


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("layout", ["row", "col"])
def test_vbatched_mixed_orders(dtype, layout):
    rng = np.random.default_rng(12)
    orders = [16, 32, 48, 64, 128, 192, 256]
    batch = 40
    sizes = [(int(rng.choice(orders)), int(rng.choice(orders)), int(rng.choice([8, 16, 24, 64, 136, 256])))
             for _ in range(batch)]
    sizes[0] = (256, 256, 256)
    sizes[1] = (16, 16, 8)
    bufs = []
    for e, (m, n, k) in enumerate(sizes):
        A, B = ki.operands(m, n, k, 1, dtype, "unif", seed=13, entry0=e)
        bufs.append((A, B, A.cuda(), B.cuda(), torch.zeros(m * n, dtype=A.dtype, device="cuda")))
    dm = torch.tensor([s[0] for s in sizes], dtype=torch.int32, device="cuda")
    dn = torch.tensor([s[1] for s in sizes], dtype=torch.int32, device="cuda")
    dk = torch.tensor([s[2] for s in sizes], dtype=torch.int32, device="cuda")
    pa = torch.tensor([b[2].data_ptr() for b in bufs], dtype=torch.int64, device="cuda")
    pb = torch.tensor([b[3].data_ptr() for b in bufs], dtype=torch.int64, device="cuda")
    pc = torch.tensor([b[4].data_ptr() for b in bufs], dtype=torch.int64, device="cuda")
    kami.gemm_vbatched(batch, dm, dn, dk, 256, 256, 256, dtype, layout, pa, pb, pc)
    torch.cuda.synchronize()
    for (m, n, k), (A, B, _, _, C) in zip(sizes, bufs):
        Cref, S = oracle.gemm(m, n, k, 1, dtype, layout, ki.as_bits(A), ki.as_bits(B), with_scale=True)
        got = oracle.decode(oracle.to_row_major(ki.as_bits(C.cpu()), 1, m, n, layout).reshape(-1), dtype)
        assert oracle.normalised_error(got.reshape(1, m, n), Cref, S) <= _tol(dtype, k), (m, n, k)


def test_vbatched_rejects():
    with pytest.raises(kami.KamiError):
        kami.gemm_vbatched(4, 16, 16, 16, 300, 16, 16, "f16", "row", 16, 16, 16)  # max_m off the grid
    with pytest.raises(kami.KamiError):
        kami.gemm_vbatched(4, 16, 16, 16, 64, 64, 64, "f64", "row", 16, 16, 16)  # fp64 not supported
