"""Pins for the FP64 GEMM oracle (oracle/oracle.c) against things other than
itself: hand-computed products (tests/golden), identities and closed forms of
the GEMM definition, exact integer arithmetic, the transpose
identity (AB)^T = B^T A^T, and an independent library routine
(torch.matmul in float64 on CPU).  CPU only."""
import json
import os
from fractions import Fraction

import numpy as np
import pytest
import torch

import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _enc(M, dtype):
    """Encode an integer/float matrix list as the oracle's raw input."""
    a = np.asarray(M, dtype=np.float64)
    if dtype == "f64":
        return a.reshape(-1)
    if dtype == "f16":
        return a.astype(np.float16).view(np.uint16).reshape(-1)
    return torch.tensor(a).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16).reshape(-1)


def _pack(M, layout):
    M = np.asarray(M)
    return M if layout == "row" else M.T.copy()


@pytest.mark.parametrize("dtype", ["f16", "bf16", "f64"])
@pytest.mark.parametrize("layout", ["row", "col"])
def test_hand_cases(dtype, layout):
    cases = json.load(open(os.path.join(GOLD, "gemm_hand_cases.json")))["cases"]
    for c in cases:
        A = _enc(_pack(c["A"], layout), dtype)
        B = _enc(_pack(c["B"], layout), dtype)
        C = oracle.gemm(c["m"], c["n"], c["k"], 1, dtype, layout, A, B)
        np.testing.assert_array_equal(C[0], np.asarray(c["C"], dtype=np.float64))


def _rand_int(rng, shape, R):
    return rng.integers(-R, R + 1, size=shape).astype(np.float64)


@pytest.mark.parametrize("layout", ["row", "col"])
def test_identity_and_permutation(layout):
    rng = np.random.default_rng(1)
    m, k = 7, 5
    A = rng.standard_normal((m, k))
    I = np.eye(k)
    C = oracle.gemm(m, k, k, 1, "f64", layout, _pack(A, layout), _pack(I, layout))
    np.testing.assert_array_equal(C[0], A)  # A * I = A exactly
    Im = np.eye(m)
    C = oracle.gemm(m, k, m, 1, "f64", layout, _pack(Im, layout), _pack(A, layout))
    np.testing.assert_array_equal(C[0], A)  # I * A = A exactly
    perm = rng.permutation(m)
    P = np.eye(m)[perm]
    C = oracle.gemm(m, k, m, 1, "f64", layout, _pack(P, layout), _pack(A, layout))
    np.testing.assert_array_equal(C[0], A[perm])  # P * A permutes rows


@pytest.mark.parametrize("dtype", ["f16", "bf16", "f64"])
def test_all_ones_closed_form(dtype):
    m, n, k, batch = 5, 3, 9, 4
    A = _enc(np.ones((batch, m, k)), dtype)
    B = _enc(np.ones((batch, k, n)), dtype)
    C = oracle.gemm(m, n, k, batch, dtype, "row", A, B)
    assert np.all(C == k)


def test_rank_one_closed_form():
    # (u v^T)(w z^T) = (v . w) u z^T, integers so every value is exact
    rng = np.random.default_rng(2)
    m, n, k = 6, 4, 8
    u, v = rng.integers(-5, 6, m), rng.integers(-5, 6, k)
    w, z = rng.integers(-5, 6, k), rng.integers(-5, 6, n)
    A = np.outer(u, v).astype(np.float64)
    B = np.outer(w, z).astype(np.float64)
    C = oracle.gemm(m, n, k, 1, "f64", "row", A, B)
    np.testing.assert_array_equal(C[0], float(np.dot(v, w)) * np.outer(u, z))


@pytest.mark.parametrize("dtype", ["f16", "bf16", "f64"])
def test_transpose_identity(dtype):
    """(AB)^T = B^T A^T: the row-major buffers of (A, B), read col-major with
    A<->B and m<->n swapped, must give the transposed product bit for bit."""
    rng = np.random.default_rng(3)
    m, n, k, batch = 12, 7, 9, 3
    A = _enc(rng.uniform(-1, 1, (batch, m, k)), dtype)
    B = _enc(rng.uniform(-1, 1, (batch, k, n)), dtype)
    C = oracle.gemm(m, n, k, batch, dtype, "row", A, B)
    Ct = oracle.gemm(n, m, k, batch, dtype, "col", B, A)
    np.testing.assert_array_equal(Ct, C.transpose(0, 2, 1))


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_integer_exact_vs_bruteforce(dtype):
    """Integer-valued 16-bit inputs: oracle equals exact rational brute force."""
    rng = np.random.default_rng(4)
    m, n, k, batch = 4, 5, 16, 2
    R = 11 if dtype == "f16" else 4
    Ai = rng.integers(-R, R + 1, (batch, m, k))
    Bi = rng.integers(-R, R + 1, (batch, k, n))
    C = oracle.gemm(m, n, k, batch, dtype, "row", _enc(Ai, dtype), _enc(Bi, dtype))
    for b in range(batch):
        for i in range(m):
            for j in range(n):
                exact = sum(Fraction(int(Ai[b, i, l])) * int(Bi[b, l, j]) for l in range(k))
                assert C[b, i, j] == float(exact)


def test_bruteforce_fractions_tiny_f16():
    """Brute force with exact rationals on tiny non-integer fp16 inputs: the
    oracle's fp64 result must equal the exactly rounded rational sum (k <= 4
    products of fp16 values are exact in fp64; the sum's rounding error is
    bounded by 2^-52 relative to S)."""
    rng = np.random.default_rng(5)
    m, n, k = 3, 3, 4
    A16 = rng.uniform(-1, 1, (m, k)).astype(np.float16)
    B16 = rng.uniform(-1, 1, (k, n)).astype(np.float16)
    C = oracle.gemm(m, n, k, 1, "f16", "row", A16.view(np.uint16), B16.view(np.uint16))
    for i in range(m):
        for j in range(n):
            exact = sum(Fraction(float(A16[i, l])) * Fraction(float(B16[l, j])) for l in range(k))
            S = sum(abs(float(A16[i, l]) * float(B16[l, j])) for l in range(k))
            assert abs(Fraction(C[0, i, j]) - exact) <= Fraction(S) * Fraction(1, 2 ** 50)


@pytest.mark.parametrize("layout", ["row", "col"])
@pytest.mark.parametrize("dtype", ["f16", "bf16", "f64"])
def test_vs_torch_matmul_f64(dtype, layout):
    """Independent library routine: torch.matmul in float64 on CPU."""
    rng = np.random.default_rng(6)
    m, n, k, batch = 24, 40, 32, 5
    A = rng.uniform(-1, 1, (batch, m, k))
    B = rng.uniform(-1, 1, (batch, k, n))
    tdt = {"f16": torch.float16, "bf16": torch.bfloat16, "f64": torch.float64}[dtype]
    At = torch.tensor(A).to(tdt)
    Bt = torch.tensor(B).to(tdt)
    ref = torch.matmul(At.double(), Bt.double()).numpy()
    if layout == "row":
        Ar, Br = At.contiguous(), Bt.contiguous()
    else:
        Ar, Br = At.transpose(1, 2).contiguous(), Bt.transpose(1, 2).contiguous()
    raw = (lambda t: t.view(torch.int16).numpy().view(np.uint16)) if dtype != "f64" else (lambda t: t.numpy())
    C, S = oracle.gemm(m, n, k, batch, dtype, layout, raw(Ar), raw(Br), with_scale=True)
    assert np.max(np.abs(C - ref) / S) < 1e-14
    np.testing.assert_allclose(S, torch.matmul(At.double().abs(), Bt.double().abs()).numpy(), rtol=1e-14)


def test_scale_definition():
    A = np.array([[1.0, -2.0]])
    B = np.array([[3.0], [4.0]])
    C, S = oracle.gemm(1, 1, 2, 1, "f64", "row", A, B, with_scale=True)
    assert C[0, 0, 0] == -5.0 and S[0, 0, 0] == 11.0


def test_batch_independence_and_threads():
    rng = np.random.default_rng(7)
    m, n, k, batch = 8, 8, 8, 9
    A = rng.uniform(-1, 1, batch * m * k)
    B = rng.uniform(-1, 1, batch * k * n)
    C1 = oracle.gemm(m, n, k, batch, "f64", "row", A, B, nthreads=1)
    C4 = oracle.gemm(m, n, k, batch, "f64", "row", A, B, nthreads=4)
    np.testing.assert_array_equal(C1, C4)
    for b in range(batch):
        Cb = oracle.gemm(m, n, k, 1, "f64", "row", A[b * m * k:(b + 1) * m * k], B[b * k * n:(b + 1) * k * n])
        np.testing.assert_array_equal(Cb[0], C1[b])


def test_rejects_bad_args():
    with pytest.raises(ValueError):
        oracle.gemm(0, 1, 1, 1, "f64", "row", np.zeros(0), np.zeros(1))


# ---------------------------------------------------------------- converters

def test_f16_decode_exhaustive_vs_numpy():
    bits = np.arange(65536, dtype=np.uint16)
    ours = oracle.decode(bits, "f16")
    ref = bits.view(np.float16).astype(np.float64)
    nan = np.isnan(ref)
    assert np.array_equal(np.isnan(ours), nan)
    np.testing.assert_array_equal(ours[~nan], ref[~nan])


def test_bf16_decode_exhaustive_vs_torch():
    bits = np.arange(65536, dtype=np.uint16)
    ours = oracle.decode(bits, "bf16")
    ref = torch.from_numpy(bits.view(np.int16).copy()).view(torch.bfloat16).double().numpy()
    nan = np.isnan(ref)
    assert np.array_equal(np.isnan(ours), nan)
    np.testing.assert_array_equal(ours[~nan], ref[~nan])


def test_f16_rne_vs_numpy_random():
    rng = np.random.default_rng(8)
    x = np.concatenate([
        rng.uniform(-70000, 70000, 200000),
        rng.standard_normal(200000) * 1e-5,       # subnormal range
        rng.standard_normal(200000),
        np.ldexp(rng.integers(1, 2048, 10000).astype(np.float64), -25),  # ties in subnormals
    ])
    ours = oracle.round_to(x, "f16")
    ref = x.astype(np.float16).view(np.uint16)  # numpy rounds double->half directly, RNE
    np.testing.assert_array_equal(ours, ref)


def test_f16_rne_hand_cases():
    L = oracle.lib()
    cases = {
        1.0: 0x3C00, -2.0: 0xC000, 65504.0: 0x7BFF, 65519.99: 0x7BFF, 65520.0: 0x7C00,
        2.0 ** -24: 0x0001, 2.0 ** -25: 0x0000, 1.5 * 2.0 ** -24: 0x0002, 2.0 ** -14: 0x0400,
        1 + 2.0 ** -11: 0x3C00,          # tie -> even (0x3C00)
        1 + 3 * 2.0 ** -11: 0x3C02,      # tie -> even (0x3C02)
    }
    cases = list(cases.items()) + [(0.0, 0x0000), (-0.0, 0x8000)]  # 0.0 == -0.0 as dict keys
    for x, b in cases:
        assert L.oracle_f64_to_f16_rne(x) == b, (x, hex(L.oracle_f64_to_f16_rne(x)), hex(b))


def test_bf16_rne_vs_torch_f32_exact_inputs():
    # inputs exactly representable in fp32 -> torch's float->bf16 RNE is single rounding
    rng = np.random.default_rng(9)
    x = np.concatenate([rng.uniform(-1e4, 1e4, 100000), rng.standard_normal(100000) * 1e-39,
                        rng.standard_normal(100000)]).astype(np.float32).astype(np.float64)
    ours = oracle.round_to(x, "bf16")
    ref = torch.from_numpy(x.astype(np.float32)).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    np.testing.assert_array_equal(ours, ref)


def test_bf16_rne_hand_cases():
    L = oracle.lib()
    cases = {
        1.0: 0x3F80, 1 + 2.0 ** -8: 0x3F80,            # tie -> even
        1 + 3 * 2.0 ** -8: 0x3F82,                      # tie -> even (up)
        1 + 2.0 ** -8 + 2.0 ** -30: 0x3F81,             # just above the tie (double rounding via f32 would give 0x3F80)
        -256.0: 0xC380, 3.0e38: 0x7F62, 3.4e38: 0x7F80,
    }
    for x, b in cases.items():
        assert L.oracle_f64_to_bf16_rne(x) == b, (x, hex(L.oracle_f64_to_bf16_rne(x)), hex(b))
