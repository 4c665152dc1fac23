"""16-bit sizes off the 16-grid: m or n = 8 mod 16 ("multiples
of 8 in [8, 256]"), on the LDG-fed tcgen05 kernel with the
MMA's N rounded up to 16 (tc16_vb.cu), strided and pointer arrays, both
layouts, against the oracle (same bars as tests/test_gpu_parity.py)."""
import numpy as np
import pytest
import torch

import kami_inputs as ki
import oracle
import paper_conf_sc_wangdltsl25_b200 as kami
from test_gpu_parity import check

pytestmark = pytest.mark.gpu

SHAPES = [
    (24, 16, 16, 301),    # G = 5 entries per tile, N = 80
    (8, 8, 8, 1029),      # smallest order
    (40, 24, 56, 97),     # both m and n = 8 mod 16
    (16, 40, 32, 203),    # n = 8 mod 16 only
    (136, 200, 72, 11),   # two m-tiles, N = 200
    (8, 256, 8, 33),
    (256, 8, 256, 9),
    (120, 120, 120, 17),
    (72, 88, 104, 23),
    (248, 248, 248, 3),   # largest order off the 16-grid
]


@pytest.mark.parametrize("shape", SHAPES, ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_grid8_strided(shape, dtype):
    m, n, k, batch = shape
    for layout, dist, seed in (("row", "int", 1), ("col", "int", 2), ("row", "unif", 3), ("col", "unif", 4)):
        check(m, n, k, batch, dtype, layout, dist, seed=seed)
        assert kami.last_kernel().startswith("kami_tc16_vb_kernel") or kami.last_kernel().startswith(
            "kami_warp"), kami.last_kernel()


@pytest.mark.parametrize("shape", [(24, 16, 16, 301), (40, 24, 56, 97), (136, 200, 72, 11)],
                         ids=lambda s: "x".join(map(str, s)))
def test_grid8_steady_state(shape):
    m, n, k, batch = shape
    with kami.grid_cap(3):
        check(m, n, k, batch, "f16", "row", "int", seed=5)
        check(m, n, k, batch, "bf16", "col", "unif", seed=6)


@pytest.mark.parametrize("shape", [(24, 16, 16), (40, 24, 56), (136, 200, 72), (16, 40, 32)],
                         ids=lambda s: "x".join(map(str, s)))
def test_grid8_pointer_arrays(shape):
    m, n, k = shape
    batch = 37
    for dtype, layout, dist in (("f16", "row", "int"), ("bf16", "col", "unif")):
        A, B = ki.operands(m, n, k, batch, dtype, dist, seed=7)
        dA, dB = A.cuda().view(batch, -1), B.cuda().view(batch, -1)
        dC = torch.full((batch, m * n), float("nan"), dtype=A.dtype, device="cuda")
        perm = torch.randperm(batch, generator=torch.Generator().manual_seed(8)).tolist()
        pa = torch.tensor([dA[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
        pb = torch.tensor([dB[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
        pc = torch.tensor([dC[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
        kami.gemm_batched(m, n, k, batch, dtype, layout, pa, pb, pc)
        torch.cuda.synchronize()
        Cref, S = oracle.gemm(m, n, k, batch, dtype, layout, ki.as_bits(A), ki.as_bits(B), with_scale=True)
        got_bits = oracle.to_row_major(ki.as_bits(dC.cpu()), batch, m, n, layout)
        if dist == "int":
            assert np.array_equal(got_bits, oracle.round_to(Cref, dtype).reshape(batch, m, n))
        else:
            got = oracle.decode(got_bits.reshape(-1), dtype).reshape(batch, m, n)
            tol = {"f16": 2.0 ** -11, "bf16": 2.0 ** -8}[dtype] + k * 2.0 ** -23
            assert oracle.normalised_error(got, Cref, S) <= tol
