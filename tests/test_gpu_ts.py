"""GPU parity of the tcgen05 kernel with the local operand resident in TMEM
(tc16_ts.cu; KAMI_ALGO_1D_TMEM and KAMI_ALGO_3D_TMEM) against the oracle,
with the same bars as tests/test_gpu_parity.py.  Shapes cover the packing
classes (G = 1, 2, 4, 8 entries per tile, unused lanes), k tails (zero-filled
A columns), several k-chunks, and the steady state (grid capped so each
persistent CTA runs many units: the A-slot ring and both accumulators wrap)."""
import pytest
import torch

import kami_inputs as ki
import paper_conf_sc_wangdltsl25_b200 as kami
from test_gpu_parity import check

pytestmark = pytest.mark.gpu

TS_SHAPES = [
    (64, 64, 64, 257),    # G = 2 (headline shape)
    (32, 32, 32, 301),    # G = 4
    (16, 16, 16, 1029),   # G = 8
    (128, 128, 128, 33),  # G = 1, two k-chunks
    (48, 80, 40, 77),     # G = 1 (n = 80), 48 live lanes, k tail 40 -> 48 (16-wide chunks)
    (96, 32, 24, 41),     # G = 1, k tail, unused lanes 96..127
    (64, 128, 256, 19),   # G = 1, four k-chunks, N = 128
    (32, 64, 8, 63),      # k = 8 (zero-filled to K = 16)
    (128, 16, 192, 23),   # narrow N, three k-chunks
]
TS3D_SHAPES = [s for s in TS_SHAPES if s[2] % 32 == 0]


@pytest.mark.parametrize("shape", TS_SHAPES, ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_ts_1d(shape, dtype):
    m, n, k, batch = shape
    for layout, dist, seed in (("row", "int", 1), ("col", "int", 2), ("row", "unif", 3), ("col", "unif", 4)):
        if layout == "col" and (n > 128 or m > 128):
            continue
        check(m, n, k, batch, dtype, layout, dist, algo="1d_tmem", seed=seed)
        assert kami.last_kernel().startswith("kami_tc16_ts_1d"), kami.last_kernel()


@pytest.mark.parametrize("shape", TS3D_SHAPES, ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_ts_3d(shape, dtype):
    m, n, k, batch = shape
    for layout, dist, seed in (("row", "int", 5), ("col", "int", 6), ("row", "unif", 7)):
        check(m, n, k, batch, dtype, layout, dist, algo="3d_tmem", seed=seed)
        assert kami.last_kernel().startswith("kami_tc16_ts_3d"), kami.last_kernel()


@pytest.mark.parametrize("algo", ["1d_tmem", "3d_tmem"])
@pytest.mark.parametrize("shape", [(64, 64, 64, 193), (32, 32, 32, 401), (128, 128, 128, 29), (64, 128, 256, 31)],
                         ids=lambda s: "x".join(map(str, s)))
def test_ts_steady_state(algo, shape):
    m, n, k, batch = shape
    with kami.grid_cap(3):
        check(m, n, k, batch, "f16", "row", "int", algo=algo, seed=8)
        check(m, n, k, batch, "bf16", "col", "unif", algo=algo, seed=9)


def test_ts_matches_ss_bitwise_on_int():
    """A in TMEM (TS) and A in SMEM (SS, tc16) give identical bits on integer data."""
    for (m, n, k) in ((64, 64, 64), (32, 32, 32), (128, 128, 128)):
        A, B = ki.operands(m, n, k, 97, "f16", "int", seed=10, device="cuda")
        outs = []
        for algo in ("1d", "1d_tmem", "3d_tmem"):
            C = torch.full((97 * m * n,), float("nan"), dtype=torch.float16, device="cuda")
            kami.gemm_strided_batched(m, n, k, 97, "f16", "row", A, B, C, algo=algo)
            torch.cuda.synchronize()
            outs.append(C.view(torch.int16).cpu())
        assert torch.equal(outs[0], outs[1]) and torch.equal(outs[0], outs[2])


def test_ts_rejects_out_of_scope():
    A = torch.zeros(256 * 256, dtype=torch.float16, device="cuda")
    for (m, n, k, algo) in ((192, 64, 64, "1d_tmem"), (64, 192, 64, "1d_tmem"), (48, 80, 40, "3d_tmem")):
        with pytest.raises(kami.KamiError):
            kami.gemm_strided_batched(m, n, k, 1, "f16", "row", A, A, A, algo=algo)
    with pytest.raises(kami.KamiError):
        kami.gemm_strided_batched(16, 16, 16, 1, "f64", "row", A, A, A, algo="1d_tmem")
