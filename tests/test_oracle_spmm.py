"""Pins for the SpMM oracle (oracle_spmm_bsr, Sec. 4.6): closed
forms (all blocks present = dense GEMM, no blocks = 0, identity blocks = B),
exact integer arithmetic, and an independent library route
(torch.sparse_bsr_tensor -> to_dense -> matmul in float64)."""
import numpy as np
import pytest
import torch

import kami_inputs as ki
import oracle


def _dense_A(m, k, row_ptr, col_blk, vals, blk=16):
    A = np.zeros((m, k))
    for i in range(m // blk):
        for j in range(row_ptr[i], row_ptr[i + 1]):
            c = col_blk[j]
            A[i * blk:(i + 1) * blk, c * blk:(c + 1) * blk] = vals[j]
    return A


@pytest.mark.parametrize("dtype", ["f16", "bf16", "f64"])
def test_full_density_is_dense_gemm(dtype):
    m, n, k, batch = 48, 32, 64, 3
    rp, cb, v, B = ki.bsr_operands(m, n, k, batch, dtype, density=1.0, seed=2)
    C = oracle.spmm_bsr(m, n, k, batch, dtype, rp.numpy(), cb.numpy(), ki.as_bits(v), ki.as_bits(B))
    vv = v.double().numpy()
    for b in range(batch):
        Ad = _dense_A(m, k, rp[b].numpy(), cb[b].numpy(), vv[b])
        Ab = oracle.round_to(Ad, dtype) if dtype != "f64" else Ad
        Cd = oracle.gemm(m, n, k, 1, dtype, "row", Ab, ki.as_bits(B)[b * k * n:(b + 1) * k * n])
        np.testing.assert_array_equal(C[b], Cd[0])


def test_empty_and_identity():
    m = n = k = 32
    rp = np.zeros((1, 3), np.int32)
    cb = -np.ones((1, 4), np.int32)
    v = np.zeros((1, 4, 16, 16))
    B = np.random.default_rng(0).uniform(-1, 1, k * n)
    assert np.all(oracle.spmm_bsr(m, n, k, 1, "f64", rp, cb, v, B) == 0)
    rp = np.array([[0, 1, 2]], np.int32)
    cb = np.array([[0, 1, -1, -1]], np.int32)
    v = np.zeros((1, 4, 16, 16))
    v[0, 0] = np.eye(16)
    v[0, 1] = np.eye(16)
    np.testing.assert_array_equal(oracle.spmm_bsr(m, n, k, 1, "f64", rp, cb, v, B)[0], B.reshape(k, n))


def test_integer_exact_hand_built():
    rng = np.random.default_rng(1)
    m, n, k = 32, 16, 48
    # block row 0: blocks at cols 0 and 2; block row 1: block at col 1
    rp = np.array([[0, 2, 3]], np.int32)
    cb = np.array([[0, 2, 1, -1, -1, -1]], np.int32)
    v = np.zeros((1, 6, 16, 16))
    v[0, :3] = rng.integers(-4, 5, (3, 16, 16))
    B = rng.integers(-4, 5, (k, n)).astype(np.float64)
    A = np.zeros((m, k))
    A[0:16, 0:16] = v[0, 0]
    A[0:16, 32:48] = v[0, 1]
    A[16:32, 16:32] = v[0, 2]
    np.testing.assert_array_equal(oracle.spmm_bsr(m, n, k, 1, "f64", rp, cb, v, B)[0], A @ B)


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_vs_torch_sparse_bsr(dtype):
    m, n, k, batch = 64, 48, 96, 4
    rp, cb, v, B = ki.bsr_operands(m, n, k, batch, dtype, density=0.5, seed=3)
    C, S = oracle.spmm_bsr(m, n, k, batch, dtype, rp.numpy(), cb.numpy(), ki.as_bits(v), ki.as_bits(B),
                           with_scale=True)
    for b in range(batch):
        nnz = int(rp[b, -1])
        At = torch.sparse_bsr_tensor(rp[b].long(), cb[b, :nnz].long(), v[b, :nnz].double(), size=(m, k))
        ref = At.to_dense() @ B.view(batch, k, n)[b].double()
        assert np.max(np.abs(C[b] - ref.numpy()) / np.where(S[b] == 0, 1, S[b])) < 1e-14


def test_generator_density_and_sorting():
    rp, cb, v, B = ki.bsr_operands(128, 16, 256, 50, "f16", density=0.5, seed=4)
    frac = float(rp[:, -1].sum()) / (50 * 8 * 16)
    assert 0.45 < frac < 0.55
    for b in range(5):
        for i in range(8):
            cols = cb[b, rp[b, i]:rp[b, i + 1]].tolist()
            assert cols == sorted(cols) and len(set(cols)) == len(cols)


# ------------------------------------------------ Z-Morton block storage (f3)
# PAPER.md Sec. 4.6, Fig. 7(b): "a multi-level Z-Morton order is
# implemented to facilitate efficient submatrix indexing" (R31).


def test_morton_order_of_a_4x4_block_grid():
    # the Z curve: quadrants TL, TR, BL, BR at every level, hand-written
    want = [(0, 0), (0, 1), (1, 0), (1, 1), (0, 2), (0, 3), (1, 2), (1, 3),
            (2, 0), (2, 1), (3, 0), (3, 1), (2, 2), (2, 3), (3, 2), (3, 3)]
    got = sorted(((oracle.morton_encode(i, j), (i, j)) for i in range(4) for j in range(4)))
    assert [ij for _, ij in got] == want
    assert [z for z, _ in got] == list(range(16))


def test_morton_round_trip_and_every_aligned_submatrix_is_one_range():
    for i in range(16):
        for j in range(16):
            assert oracle.morton_decode(oracle.morton_encode(i, j)) == (i, j)
    for L in range(5):  # 1x1 ... 16x16 aligned submatrices
        s = 1 << L
        for i0 in range(0, 16, s):
            for j0 in range(0, 16, s):
                codes = sorted(oracle.morton_encode(i, j) for i in range(i0, i0 + s) for j in range(j0, j0 + s))
                assert codes == list(range(codes[0], codes[0] + s * s))


@pytest.mark.parametrize("shape", [(64, 32, 48, 5), (128, 64, 256, 3), (16, 16, 16, 7), (192, 48, 96, 2)])
@pytest.mark.parametrize("density", [0.5, 1.0, 0.0])
def test_zmorton_spmm_equals_bsr_spmm(shape, density):
    """The same block-sparse matrices in two independent storage formats give
    bit-identical oracle products (and density 1 is the dense GEMM)."""
    import kami_inputs as ki
    m, n, k, batch = shape
    rp, cb, v, B = ki.bsr_operands(m, n, k, batch, "f16", density=density, dist="unif", seed=3)
    present, blocks = ki.block_sparse(m, k, batch, "f16", density=density, dist="unif", seed=3)
    nnzb, zcode, zvals = oracle.zmorton_from_blocks(present.numpy(), ki.as_bits(blocks))
    C1 = oracle.spmm_bsr(m, n, k, batch, "f16", rp.numpy(), cb.numpy(), ki.as_bits(v), ki.as_bits(B))
    C2 = oracle.spmm_zmorton(m, n, k, batch, "f16", nnzb, zcode, zvals, ki.as_bits(B))
    assert np.array_equal(C1, C2)
    assert (nnzb == present.reshape(batch, -1).sum(1).numpy()).all()
    if density == 1.0:
        A = blocks.permute(0, 1, 3, 2, 4).reshape(batch, m, k)
        Cd = oracle.gemm(m, n, k, batch, "f16", "row", ki.as_bits(A.contiguous()), ki.as_bits(B))
        assert np.array_equal(C2, Cd)
    if density == 0.0:
        assert not C2.any()
