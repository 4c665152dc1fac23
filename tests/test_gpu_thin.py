"""Thin tiles (k <= 32 with n = 16 / 32, and 16 x 128 x 16) on the one-warp
register-resident HMMA 1D (warp_ca.cu, KAMI_THIN_CASES) -- the kernels the
planner picks for the BF16 sweep's slowest r1 points -- against the oracle,
both layouts, integer bit-exact and unif within the derived bound, steady state
included."""
import pytest

import paper_conf_sc_wangdltsl25_b200 as kami
from test_gpu_parity import check

pytestmark = pytest.mark.gpu

THIN = [(16, 128, 16), (16, 32, 16), (16, 16, 32), (32, 16, 16), (64, 16, 16), (128, 16, 16), (192, 16, 16),
        (256, 16, 16), (192, 16, 32), (128, 32, 16)]


@pytest.mark.parametrize("shape", THIN, ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_thin_warp_1d(shape, dtype):
    m, n, k = shape
    for layout, dist, seed, batch in (("row", "int", 1, 301), ("row", "unif", 2, 77)):
        check(m, n, k, batch, dtype, layout, dist, algo="1d", p=1, seed=seed)
        assert kami.last_kernel().startswith(f"kami_warp_ca_1d<{dtype},{m}x{n}x{k}>"), kami.last_kernel()
    # column-major runs the transposed problem n x m (a thin instantiation only if that one exists)
    if (n, m, k) in THIN:
        check(m, n, k, 33, dtype, "col", "int", algo="1d", p=1, seed=3)


@pytest.mark.parametrize("shape", THIN, ids=lambda s: "x".join(map(str, s)))
def test_thin_auto_parity(shape):
    """Whatever AUTO picks for the thin shapes (both layouts) is correct; the
    grid cap forces the steady state."""
    m, n, k = shape
    with kami.grid_cap(3):
        check(m, n, k, 203, "bf16", "row", "int", seed=4)
        check(m, n, k, 203, "f16", "col", "unif", seed=5)
