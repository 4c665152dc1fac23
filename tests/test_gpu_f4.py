"""GPU parity for SURVEY f4: TF32 and FP8 (E4M3 / E5M2) inputs on the
tcgen05 path, and the C-update form C <- alpha A B + beta C (tcgen05 types and
FP64), against the FP64 oracle (oracle.gemm + oracle.axpby).

Bars (f4):
  * "int" inputs, alpha, beta powers of two: bit-exact;
  * "unif": max |C - C_ref| / S' <= u_out + k 2^-23 + 2^-22, S' = |alpha| S +
    |beta| |C_in|; u_out = 2^-24 (f32 out) / 2^-11 (f16 out).  TF32 inputs
    are drawn already at TF32 precision, so the tensor core reads them exactly.
"""
import numpy as np
import pytest
import torch

import kami_inputs as ki
import oracle
import paper_conf_sc_wangdltsl25_b200 as kami

pytestmark = pytest.mark.gpu

U_OUT = {"f32": 2.0 ** -24, "f16": 2.0 ** -11, "bf16": 2.0 ** -8, "f64": 2.0 ** -53}


def tol(dtype, k):
    if dtype == "f64":
        return 2 * k * 2.0 ** -52
    return U_OUT[ki.OUT_DTYPE[dtype]] + k * 2.0 ** -23 + 2.0 ** -22


def c_in(m, n, batch, dtype, dist, seed):
    """Initial C in the output type (int: small integers so the update stays exact)."""
    od = ki.OUT_DTYPE[dtype]
    R = 16 if dist == "int" else None
    return ki.draw(seed + 1, 0, 0, batch, m, n, od, dist, R)


def run(m, n, k, batch, dtype, layout, dist, alpha=1.0, beta=0.0, seed=0):
    A, B = ki.operands(m, n, k, batch, dtype, dist, seed=seed)
    od = ki.OUT_DTYPE[dtype]
    C0 = c_in(m, n, batch, dtype, dist, seed) if beta != 0.0 else None
    dC = (C0.cuda() if C0 is not None else
          torch.full((batch * m * n,), float("nan"), dtype=ki.TORCH_DTYPES[od], device="cuda"))
    if alpha == 1.0 and beta == 0.0:
        kami.gemm_strided_batched(m, n, k, batch, dtype, layout, A.cuda(), B.cuda(), dC)
    else:
        kami.gemm_strided_batched_axpby(m, n, k, batch, dtype, layout, alpha, A.cuda(), B.cuda(), beta, dC)
    torch.cuda.synchronize()
    Cref, S = oracle.gemm(m, n, k, batch, dtype, layout, ki.as_bits(A), ki.as_bits(B), with_scale=True)
    Cref = Cref.reshape(batch, m, n)
    if C0 is not None:
        cin = oracle.to_row_major(oracle.decode(ki.as_bits(C0), od), batch, m, n, layout).reshape(batch, m, n)
        Cref = oracle.axpby(Cref, cin, alpha, beta)
        S = abs(alpha) * S + abs(beta) * np.abs(cin)
    else:
        Cref = alpha * Cref
        S = abs(alpha) * S
    got_bits = oracle.to_row_major(ki.as_bits(dC.cpu()), batch, m, n, layout)
    if dist == "int":
        exp = oracle.round_to(Cref, od).reshape(batch, m, n)
        bad = np.argwhere(got_bits.reshape(batch, m, n) != exp)
        assert bad.size == 0, f"{len(bad)} mismatches, first at {bad[:3].tolist()}"
    else:
        got = oracle.decode(got_bits.reshape(-1), od).reshape(batch, m, n)
        assert np.isfinite(got).all()
        err = oracle.normalised_error(got, Cref, S)
        assert err <= tol(dtype, k), err


TF32_SHAPES = [(16, 16, 16, 1029), (32, 32, 32, 301), (64, 64, 64, 257), (128, 128, 128, 33),
               (48, 80, 40, 77), (256, 256, 12, 5), (256, 256, 256, 2), (16, 256, 64, 20)]
FP8_SHAPES = [(32, 32, 32, 301), (64, 64, 64, 257), (128, 128, 128, 33), (96, 160, 48, 41),
              (256, 256, 16, 5), (256, 256, 256, 2), (32, 256, 64, 20)]


@pytest.mark.parametrize("shape", TF32_SHAPES, ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("layout", ["row", "col"])
@pytest.mark.parametrize("dist", ["int", "unif"])
def test_tf32(shape, layout, dist):
    run(*shape, "tf32", layout, dist)
    assert kami.last_kernel().startswith("kami_tc16_1d_kernel")


@pytest.mark.parametrize("shape", FP8_SHAPES, ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype", ["e4m3", "e5m2"])
@pytest.mark.parametrize("layout", ["row", "col"])
@pytest.mark.parametrize("dist", ["int", "unif"])
def test_fp8(shape, dtype, layout, dist):
    run(*shape, dtype, layout, dist)


@pytest.mark.parametrize("shape", [(16, 16, 16, 1029), (64, 64, 64, 257), (128, 128, 128, 33),
                                   (48, 80, 40, 77), (256, 256, 256, 2)], ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype", ["f16", "bf16", "tf32", "e4m3"])
@pytest.mark.parametrize("ab", [(1.0, 1.0), (2.0, -1.0), (0.5, 0.0)])
def test_axpby_int_exact(shape, dtype, ab):
    m, n, k, batch = shape
    if dtype == "e4m3" and (m % 32 or n % 32):
        pytest.skip("fp8 needs m, n multiples of 32")
    run(m, n, k, batch, dtype, "row", "int", alpha=ab[0], beta=ab[1])


@pytest.mark.parametrize("shape", [(32, 32, 32, 301), (64, 64, 64, 257), (256, 256, 64, 3)],
                         ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype", ["f16", "bf16", "tf32", "e5m2"])
@pytest.mark.parametrize("layout", ["row", "col"])
def test_axpby_unif(shape, dtype, layout):
    run(*shape, dtype, layout, "unif", alpha=0.75, beta=-1.25)


@pytest.mark.parametrize("order,batch", [(16, 1001), (32, 257), (64, 65)])
@pytest.mark.parametrize("dist", ["int", "unif"])
def test_axpby_f64(order, batch, dist):
    run(order, order, order, batch, "f64", "row", dist, alpha=0.5 if dist == "unif" else 2.0,
        beta=1.5 if dist == "unif" else 1.0)
    assert kami.last_kernel().startswith("kami_dmma_tma")


def test_axpby_not_supported_on_warp_family():
    A = torch.zeros(64 * 8, dtype=torch.float64, device="cuda")
    with pytest.raises(RuntimeError):
        kami.gemm_strided_batched_axpby(8, 8, 8, 1, "f64", "row", 1.0, A, A, 1.0, A)
