"""Pins for the oracle's f4 extensions: FP8 decoders (exhaustive against torch
float8 dtypes), FP32/TF32 inputs against torch.matmul float64, and the
alpha*AB + beta*C update form against closed forms."""
import numpy as np
import pytest
import torch

import oracle


@pytest.mark.parametrize("dt,tdt", [("e4m3", torch.float8_e4m3fn), ("e5m2", torch.float8_e5m2)])
def test_fp8_decode_exhaustive_vs_torch(dt, tdt):
    bits = np.arange(256, dtype=np.uint8)
    ours = oracle.decode(bits, dt)
    ref = torch.from_numpy(bits.copy()).view(tdt).double().numpy()
    nan = np.isnan(ref)
    assert np.array_equal(np.isnan(ours), nan)
    np.testing.assert_array_equal(ours[~nan], ref[~nan])


@pytest.mark.parametrize("dt,tdt", [("e4m3", torch.float8_e4m3fn), ("e5m2", torch.float8_e5m2)])
def test_fp8_gemm_vs_torch(dt, tdt):
    rng = np.random.default_rng(0)
    m, n, k, b = 16, 32, 64, 3
    A = torch.tensor(rng.uniform(-2, 2, (b, m, k))).to(tdt)
    B = torch.tensor(rng.uniform(-2, 2, (b, k, n))).to(tdt)
    C, S = oracle.gemm(m, n, k, b, dt, "row", A.view(torch.uint8).numpy(), B.view(torch.uint8).numpy(),
                       with_scale=True)
    ref = torch.matmul(A.double(), B.double()).numpy()
    assert np.max(np.abs(C - ref) / np.where(S == 0, 1, S)) < 1e-14


def test_f32_gemm_vs_torch_and_transpose():
    rng = np.random.default_rng(1)
    m, n, k, b = 24, 16, 40, 2
    A = rng.uniform(-1, 1, (b, m, k)).astype(np.float32)
    B = rng.uniform(-1, 1, (b, k, n)).astype(np.float32)
    C, S = oracle.gemm(m, n, k, b, "f32", "row", A, B, with_scale=True)
    ref = np.matmul(A.astype(np.float64), B.astype(np.float64))
    assert np.max(np.abs(C - ref) / S) < 1e-14
    Ct = oracle.gemm(n, m, k, b, "f32", "col", B, A)
    np.testing.assert_array_equal(Ct, C.transpose(0, 2, 1))


def test_axpby_closed_forms():
    rng = np.random.default_rng(2)
    Cr = rng.uniform(-1, 1, (2, 4, 4))
    Ci = rng.uniform(-1, 1, (2, 4, 4))
    np.testing.assert_array_equal(oracle.axpby(Cr, Ci, 1.0, 0.0), Cr)
    np.testing.assert_array_equal(oracle.axpby(Cr, Ci, 0.0, 1.0), Ci)
    np.testing.assert_array_equal(oracle.axpby(Cr, Ci, 2.0, -1.0), 2.0 * Cr - Ci)
    # C += A B on integers: exact
    A = rng.integers(-3, 4, (1, 5, 6)).astype(np.float64)
    B = rng.integers(-3, 4, (1, 6, 7)).astype(np.float64)
    C0 = rng.integers(-9, 10, (1, 5, 7)).astype(np.float64)
    Cr = oracle.gemm(5, 7, 6, 1, "f64", "row", A, B)
    np.testing.assert_array_equal(oracle.axpby(Cr, C0, 1.0, 1.0), A @ B + C0)
