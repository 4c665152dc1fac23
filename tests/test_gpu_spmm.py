"""SpMM (Sec. 4.6): block-sparse A (BSR, 16x16
blocks, ~50% random block density as in Sec. 5.1) times dense B on the GPU
against the SpMM oracle."""
import numpy as np
import pytest
import torch

import kami_inputs as ki
import oracle
import paper_conf_sc_wangdltsl25_b200 as kami

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("shape", [(16, 16, 16), (64, 64, 64), (128, 128, 128), (192, 64, 256), (256, 256, 32),
                                   (48, 80, 112), (224, 96, 160), (32, 48, 256), (256, 16, 256)])
@pytest.mark.parametrize("density", [0.5, 1.0, 0.1, 0.0])
def test_spmm_vs_oracle(dtype, shape, density):
    m, n, k = shape
    batch = 19
    for dist in ("unif", "int"):
        rp, cb, v, B = ki.bsr_operands(m, n, k, batch, dtype, density=density, dist=dist, seed=5)
        C = torch.full((batch * m * n,), float("nan"), dtype=B.dtype, device="cuda")
        kami.spmm_bsr_strided_batched(m, n, k, batch, dtype, rp.cuda(), cb.cuda(), v.cuda(), B.cuda(), C)
        torch.cuda.synchronize()
        assert "spmm_bsr" in kami.last_kernel()
        Cref, S = oracle.spmm_bsr(m, n, k, batch, dtype, rp.numpy(), cb.numpy(), ki.as_bits(v), ki.as_bits(B),
                                  with_scale=True)
        got_bits = ki.as_bits(C.cpu()).reshape(batch, m, n)
        if dist == "int":
            assert np.array_equal(got_bits, oracle.round_to(Cref, dtype).reshape(batch, m, n))
        else:
            got = oracle.decode(got_bits.reshape(-1), dtype).reshape(batch, m, n)
            tol = {"f16": 2.0 ** -11, "bf16": 2.0 ** -8}[dtype] + k * 2.0 ** -23
            assert oracle.normalised_error(got, Cref, S) <= tol


def test_spmm_dense_equivalence():
    """All blocks present: identical bits to the dense strided GEMM path (integer data)."""
    m = n = k = 64
    batch = 33
    rp, cb, v, B = ki.bsr_operands(m, n, k, batch, "f16", density=1.0, dist="int", seed=6)
    C1 = torch.empty(batch * m * n, dtype=torch.float16, device="cuda")
    kami.spmm_bsr_strided_batched(m, n, k, batch, "f16", rp.cuda(), cb.cuda(), v.cuda(), B.cuda(), C1)
    # densify on the host (test-side) and run the dense path
    A = torch.zeros(batch, m, k, dtype=torch.float16)
    for b in range(batch):
        for i in range(m // 16):
            for j in range(int(rp[b, i]), int(rp[b, i + 1])):
                c = int(cb[b, j])
                A[b, i * 16:(i + 1) * 16, c * 16:(c + 1) * 16] = v[b, j]
    C2 = torch.empty_like(C1)
    kami.gemm_strided_batched(m, n, k, batch, "f16", "row", A.cuda(), B.cuda(), C2)
    torch.cuda.synchronize()
    assert torch.equal(C1.view(torch.int16), C2.view(torch.int16))


# ------------------------------------------- Z-Morton block storage (f3)
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("shape", [(16, 16, 16), (64, 64, 64), (128, 128, 128), (192, 64, 256), (256, 256, 32),
                                   (48, 80, 112), (256, 256, 256), (224, 96, 160), (144, 32, 48)])
@pytest.mark.parametrize("density", [0.5, 1.0, 0.1])
@pytest.mark.parametrize("algo", ["auto", "2d"])
def test_spmm_zmorton_vs_oracle(dtype, shape, density, algo):
    """A in multi-level Z-Morton block storage (Sec. 4.6), built
    by the ORACLE's encoder from the generator's block description, decoded by
    the kernel; against the Z-Morton oracle."""
    m, n, k = shape
    if algo == "2d" and m <= 128:
        pytest.skip("the 2D pair schedule needs m > 128")
    batch = 19
    for dist in ("unif", "int"):
        present, blocks = ki.block_sparse(m, k, batch, dtype, density=density, dist=dist, seed=6)
        _, B = ki.operands(m, n, k, batch, dtype, dist, seed=6)
        nnzb, zcode, zvals = oracle.zmorton_from_blocks(present.numpy(), ki.as_bits(blocks))
        zv = torch.from_numpy(zvals.view(np.int16)).view(ki.TORCH_DTYPES[dtype])
        C = torch.full((batch * m * n,), float("nan"), dtype=B.dtype, device="cuda")
        kami.spmm_zmorton_strided_batched(m, n, k, batch, dtype, torch.from_numpy(nnzb).cuda(),
                                          torch.from_numpy(zcode).cuda(), zv.cuda(), B.cuda(), C, algo=algo)
        torch.cuda.synchronize()
        assert "spmm_zmorton" in kami.last_kernel()
        want = "kami_tc16_pair_2d" if algo == "2d" else "kami_tc16_vb_kernel"
        assert kami.last_kernel().startswith(want), kami.last_kernel()
        Cref, S = oracle.spmm_zmorton(m, n, k, batch, dtype, nnzb, zcode, zvals, ki.as_bits(B), with_scale=True)
        got_bits = ki.as_bits(C.cpu()).reshape(batch, m, n)
        if dist == "int":
            assert np.array_equal(got_bits, oracle.round_to(Cref, dtype).reshape(batch, m, n))
        else:
            got = oracle.decode(got_bits.reshape(-1), dtype).reshape(batch, m, n)
            tol = {"f16": 2.0 ** -11, "bf16": 2.0 ** -8}[dtype] + k * 2.0 ** -23
            assert oracle.normalised_error(got, Cref, S) <= tol


def test_spmm_zmorton_equals_bsr_bitwise():
    """The same matrices in BSR and in Z-Morton storage: identical output bits."""
    m, n, k, batch = 128, 64, 256, 23
    rp, cb, v, B = ki.bsr_operands(m, n, k, batch, "bf16", density=0.5, dist="unif", seed=9)
    present, blocks = ki.block_sparse(m, k, batch, "bf16", density=0.5, dist="unif", seed=9)
    nnzb, zcode, zvals = oracle.zmorton_from_blocks(present.numpy(), ki.as_bits(blocks))
    zv = torch.from_numpy(zvals.view(np.int16)).view(torch.bfloat16)
    C1 = torch.empty(batch * m * n, dtype=torch.bfloat16, device="cuda")
    C2 = torch.empty_like(C1)
    kami.spmm_bsr_strided_batched(m, n, k, batch, "bf16", rp.cuda(), cb.cuda(), v.cuda(), B.cuda(), C1)
    with kami.grid_cap(3):  # and the steady state
        kami.spmm_zmorton_strided_batched(m, n, k, batch, "bf16", torch.from_numpy(nnzb).cuda(),
                                          torch.from_numpy(zcode).cuda(), zv.cuda(), B.cuda(), C2)
    torch.cuda.synchronize()
    assert torch.equal(C1.view(torch.int16), C2.view(torch.int16))
