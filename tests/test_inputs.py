"""Tests of the shared seeded input generator (kami_inputs)."""
import numpy as np
import pytest
import torch

import kami_inputs as ki


def test_splitmix64_known_value():
    # SplitMix64 seeded with 0: first output is 0xE220A8397B1DCDAF (Steele/Vigna reference)
    assert ki.splitmix64_py(0) == 0xE220A8397B1DCDAF


def test_torch_matches_python_reference():
    xs = [0, 1, 2, 12345, (1 << 44) + 7, (3 << 44) + 99999, (1 << 62) + 5]
    t = ki.splitmix64(torch.tensor(xs, dtype=torch.int64))
    got = [int(v) & ki.MASK64 for v in t.tolist()]
    assert got == [ki.splitmix64_py(x) for x in xs]


@pytest.mark.parametrize("dtype", ["f16", "bf16", "f64"])
@pytest.mark.parametrize("dist", ["unif", "int"])
def test_shard_independence(dtype, dist):
    A, B = ki.operands(8, 16, 24, 10, dtype, dist, seed=3)
    A1, B1 = ki.operands(8, 16, 24, 4, dtype, dist, seed=3, entry0=0)
    A2, B2 = ki.operands(8, 16, 24, 6, dtype, dist, seed=3, entry0=4)
    assert torch.equal(torch.cat([A1, A2]), A) and torch.equal(torch.cat([B1, B2]), B)


def test_seeds_and_operands_differ():
    A0, B0 = ki.operands(16, 16, 16, 2, "f16", seed=0)
    A1, _ = ki.operands(16, 16, 16, 2, "f16", seed=1)
    assert not torch.equal(A0, A1) and not torch.equal(A0, B0)


def test_ranges():
    A, B = ki.operands(32, 32, 64, 50, "f64", "unif")
    assert A.min() >= -1 and A.max() < 1 and abs(float(A.mean())) < 0.02
    for k, dtype in [(16, "f16"), (64, "f16"), (256, "f16"), (16, "bf16"), (256, "bf16")]:
        R = ki.int_range(k, dtype)
        A, _ = ki.operands(16, 16, k, 20, dtype, "int")
        assert float(A.abs().max()) == R and torch.all(A == A.round())
        lim = 2048 if dtype == "f16" else 256
        assert R * R * k <= lim


def test_int_range_table():
    # DESIGN.md input recipe: fp16 R = 11/8/5/4/2 and bf16 R = 4/2/2/1/1 for k = 16/32/64/128/256
    assert [ki.int_range(k, "f16") for k in (16, 32, 64, 128, 256)] == [11, 8, 5, 4, 2]
    assert [ki.int_range(k, "bf16") for k in (16, 32, 64, 128, 256)] == [4, 2, 2, 1, 1]


def test_as_bits_roundtrip():
    A, _ = ki.operands(4, 4, 4, 1, "f16")
    bits = ki.as_bits(A)
    assert bits.dtype == np.uint16
    np.testing.assert_array_equal(bits.view(np.float16).astype(np.float64), A.double().numpy())
