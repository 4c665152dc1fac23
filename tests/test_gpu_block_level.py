"""Block-level (on-chip-resident) mode, Sec. 5.1 L468 / Sec. 5.2 /
Sec. 5.6.2: the CA schedule repeated `reps` times on chip must give
C = reps * A B (checked against the oracle: bit-exact on integer inputs,
normalised error otherwise), and the per-phase cycle counters must be
populated."""
import numpy as np
import pytest
import torch

import kami_inputs as ki
import oracle
import paper_conf_sc_wangdltsl25_b200 as kami

pytestmark = pytest.mark.gpu

CASES = [("f64", 16, "1d", 0), ("f64", 32, "1d", 0), ("f64", 32, "2d", 0), ("f64", 32, "3d", 0),
         ("f64", 64, "2d", 0), ("f64", 32, "nonca", 0), ("f16", 64, "1d", 4), ("f16", 64, "2d", 0),
         ("f16", 64, "3d", 0), ("f16", 64, "nonca", 0), ("bf16", 32, "1d", 2), ("f16", 128, "1d", 8)]


@pytest.mark.parametrize("dtype,s,algo,p", CASES, ids=lambda x: str(x))
def test_block_level_int_bit_exact(dtype, s, algo, p):
    batch, reps = 45, 3
    A, B = ki.operands(s, s, s, batch, dtype, "int", seed=8)
    C = torch.empty(batch * s * s, dtype=A.dtype, device="cuda")
    cyc = torch.zeros(2 * batch, dtype=torch.int64, device="cuda")
    kami.gemm_block_level(s, s, s, batch, dtype, "row", A.cuda(), B.cuda(), C, algo=algo, p=p, reps=reps, cycles=cyc)
    torch.cuda.synchronize()
    Cref = oracle.gemm(s, s, s, batch, dtype, "row", ki.as_bits(A), ki.as_bits(B))
    exp = oracle.round_to(reps * Cref, dtype)  # reps * exact integer, rounded once
    assert np.array_equal(ki.as_bits(C.cpu()).reshape(-1), exp)
    cy = cyc.view(batch, 2).cpu()
    assert bool((cy[:, 0] > 0).all()) and bool((cy[:, 1] > 0).all())


@pytest.mark.parametrize("dtype,s,algo", [("f64", 64, "2d"), ("f16", 64, "3d"), ("bf16", 64, "2d")])
def test_block_level_unif(dtype, s, algo):
    batch, reps = 37, 10
    A, B = ki.operands(s, s, s, batch, dtype, "unif", seed=9)
    C = torch.empty(batch * s * s, dtype=A.dtype, device="cuda")
    kami.gemm_block_level(s, s, s, batch, dtype, "col", A.cuda(), B.cuda(), C, algo=algo, reps=reps)
    torch.cuda.synchronize()
    Cref, S = oracle.gemm(s, s, s, batch, dtype, "col", ki.as_bits(A), ki.as_bits(B), with_scale=True)
    got = oracle.decode(oracle.to_row_major(ki.as_bits(C.cpu()), batch, s, s, "col").reshape(-1), dtype)
    err = oracle.normalised_error(got.reshape(batch, s, s), reps * Cref, reps * S)
    tol = {"f64": reps * s * 2.0 ** -52, "f16": 2.0 ** -11 + reps * s * 2.0 ** -23, "bf16": 2.0 ** -8 + reps * s * 2.0 ** -23}
    assert err <= tol[dtype], err


def test_block_level_rejects():
    with pytest.raises(kami.KamiError):
        kami.gemm_block_level(64, 64, 64, 4, "f16", "row", 16, 16, 16, algo="1d", reps=0)
