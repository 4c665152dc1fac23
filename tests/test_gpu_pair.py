"""KAMI-2D across a CTA pair (tcgen05 cta_group::2, tc16_pair.cu;
KAMI_ALGO_2D_PAIR) against the oracle: rows split 128 / 128 over the pair,
B's columns split n/2 / n/2 and broadcast through the pair's shared memory.
Same bars as tests/test_gpu_parity.py; shapes cover m < 256 (the second CTA's
rows partly past m), every atom width of the B halves and C, k tails and
several k-chunks, and the steady state (grid capped at two pairs)."""
import pytest

import paper_conf_sc_wangdltsl25_b200 as kami
from test_gpu_parity import check

pytestmark = pytest.mark.gpu

PAIR_SHAPES = [
    (256, 256, 256, 5),
    (256, 128, 64, 17),
    (224, 96, 40, 13),   # rows 224..255 of CTA 1 clipped, 48-column halves, k tail
    (208, 64, 16, 19),
    (256, 256, 8, 7),    # k = 8 zero-filled to K = 16
    (256, 32, 24, 21),   # 16-column halves
    (240, 160, 48, 9),
    (256, 192, 192, 4),
]


@pytest.mark.parametrize("shape", PAIR_SHAPES, ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_pair_2d(shape, dtype):
    m, n, k, batch = shape
    for layout, dist, seed in (("row", "int", 1), ("row", "unif", 2)):
        check(m, n, k, batch, dtype, layout, dist, algo="2d_pair", seed=seed)
        assert kami.last_kernel().startswith("kami_tc16_pair_2d"), kami.last_kernel()
    if n > 192:  # column-major runs the transposed problem (n x m), also in scope
        check(m, n, k, batch, dtype, "col", "int", algo="2d_pair", seed=3)


@pytest.mark.parametrize("shape", [(256, 256, 256, 9), (224, 96, 40, 41), (256, 64, 128, 33)],
                         ids=lambda s: "x".join(map(str, s)))
def test_pair_steady_state(shape):
    m, n, k, batch = shape
    with kami.grid_cap(4):
        check(m, n, k, batch, "f16", "row", "int", algo="2d_pair", seed=4)
        check(m, n, k, batch, "bf16", "row", "unif", algo="2d_pair", seed=5)


def test_pair_rejects_out_of_scope():
    import torch
    A = torch.zeros(256 * 256, dtype=torch.float16, device="cuda")
    for (m, n, k) in ((128, 128, 64), (256, 48, 64), (112, 64, 64)):
        with pytest.raises(kami.KamiError):
            kami.gemm_strided_batched(m, n, k, 1, "f16", "row", A, A, A, algo="2d_pair")
