"""tcgen05 1D on the transposed product C^T = B^T A^T for thin m (tc16_xt.cu;
KAMI_ALGO_1D_XT) against the oracle, with the bars of
tests/test_gpu_parity.py (integer data bit-exact, uniform data within the
normalised-error bound).  Shapes: every (m, n, k) the kernel takes, batches
that leave a partial last group of E entries, 64-column last tiles (n = 64,
192), column-major C (the row problem n x m: thin n), and the steady state
(grid capped so every CTA runs many units and both accumulators / staging
buffers are reused)."""
import pytest

import paper_conf_sc_wangdltsl25_b200 as kami
from test_gpu_parity import check

pytestmark = pytest.mark.gpu

XT_SHAPES = [(m, n, k) for m in (16, 32) for n in (64, 128, 192, 256) for k in (16, 32, 64)]


@pytest.mark.parametrize("shape", XT_SHAPES, ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_xt(shape, dtype):
    m, n, k = shape
    for dist, seed, batch in (("int", 1, 37), ("unif", 2, 21)):
        check(m, n, k, batch, dtype, "row", dist, algo="1d_xt", seed=seed)
        assert kami.last_kernel().startswith("kami_tc16_xt_kernel"), kami.last_kernel()


@pytest.mark.parametrize("shape", [(128, 16, 16), (192, 32, 32), (256, 16, 64)], ids=lambda s: "x".join(map(str, s)))
def test_xt_col_major(shape):
    """Column-major C = A B is the row problem (n, m): thin in n."""
    m, n, k = shape
    check(m, n, k, 29, "f16", "col", "int", algo="1d_xt", seed=3)
    assert kami.last_kernel().startswith("kami_tc16_xt_kernel"), kami.last_kernel()


@pytest.mark.parametrize("shape", [(16, 128, 16), (16, 192, 32), (32, 256, 64), (16, 64, 64)],
                         ids=lambda s: "x".join(map(str, s)))
def test_xt_steady_state(shape):
    m, n, k = shape
    with kami.grid_cap(3):
        check(m, n, k, 203, "bf16", "row", "int", algo="1d_xt", seed=4)
        check(m, n, k, 117, "f16", "row", "unif", algo="1d_xt", seed=5)


def test_xt_rejects_off_shapes():
    with pytest.raises(kami.KamiError):
        check(48, 128, 16, 4, "f16", "row", "int", algo="1d_xt", seed=6)
    with pytest.raises(kami.KamiError):
        check(16, 96, 16, 4, "f16", "row", "int", algo="1d_xt", seed=6)
