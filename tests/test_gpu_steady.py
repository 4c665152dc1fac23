"""Steady-state parity: every kernel instantiation with each persistent CTA
running many work units.

The persistent kernels deal units round-robin over min(units, #SMs) CTAs,
so at the small batches the other parity tests use a CTA runs at most one
unit: the TMA ring never wraps, mbarrier phases never flip, TMEM
accumulators and C staging buffers are never reused.  Here the grid is
capped with ``kami.grid_cap`` (the C ABI's kami_set_grid_cap, a test knob
that changes nothing but the grid size) so each CTA runs >= 8 units: ring
slots, accumulator buffers and staging buffers are each reused several
times, and ragged last units are included.

Same bars as tests/test_gpu_parity.py: integer inputs bit-exact against
RNE(C_ref); "unif" within the north_star and the derived tolerance.
"""
import numpy as np
import pytest
import torch

import kami_inputs as ki
import oracle
import paper_conf_sc_wangdltsl25_b200 as kami
from test_gpu_parity import check, derived_tol

pytestmark = pytest.mark.gpu

CAP = 3  # odd: also coprime with m_tiles = 2 (units of one entry land on different CTAs)


@pytest.fixture(autouse=True)
def _capped():
    with kami.grid_cap(CAP):
        yield


# (m, n, k, batch, expected kernel-name prefix).  Batches give >= 8 units per
# CTA at CAP = 3 for the unit size each shape plans (G entries x U sub-tiles).
TC_STEADY = [
    (64, 64, 64, 97, "kami_tc16_1d_kernel<{dt}>"),            # plain, G = 2: 49 units
    (32, 32, 32, 401, "kami_tc16_1d_kernel<{dt}>"),           # G = 4, U = 2: 51 units
    (16, 64, 16, 403, "kami_tc16_1d_kernel<{dt}>"),           # thin m, 32-lane slots, U = 2
    (128, 16, 16, 101, "kami_tc16_1d_kernel<{dt}>"),          # narrow N, U = 4
    (48, 80, 40, 121, "kami_tc16_1d_kernel<{dt}>"),           # 96 live lanes, k tail
    (112, 32, 24, 61, "kami_tc16_1d_kernel<{dt}>"),           # m not dividing 128
    (128, 128, 64, 29, "kami_tc16_1d_kernel<{dt}>"),          # per-atom split stores
    (192, 192, 192, 13, "kami_tc16_1d_kernel<{dt}>"),         # split, 2 m-tiles, 3 k-chunks
    (256, 256, 16, 13, "kami_tc16_1d_kernel<{dt}>"),          # low-rank, whole-unit stores, 2 m-tiles
    (256, 256, 8, 13, "kami_tc16_1d_kernel<{dt}>"),           # low-rank k = 8 (zero-filled K)
    (192, 64, 64, 19, "kami_tc16_1d_kernel<{dt},tailpack>"),  # tail packing: 30 units, odd batch
    (144, 128, 24, 17, "kami_tc16_1d_kernel<{dt},tailpack>"),  # tail packing, N = 256, k tail
    (16, 256, 16, 29, "kami_tc16_1d_kernel<{dt},warpstore>"),  # replicated thin m, per-warp stores
    (32, 192, 16, 29, "kami_tc16_1d_kernel<{dt},warpstore>"),  # 3 slots
    (16, 144, 16, 31, "kami_tc16_1d_kernel<{dt}>"),           # replicated A, 16-column atoms
]


@pytest.mark.parametrize("case", TC_STEADY, ids=lambda c: "x".join(map(str, c[:4])))
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_tc16_steady(case, dtype):
    m, n, k, batch, name = case
    for layout, dist, seed in (("row", "int", 1), ("col", "int", 2), ("row", "unif", 3), ("col", "unif", 4)):
        check(m, n, k, batch, dtype, layout, dist, algo="1d", seed=seed)
        if layout == "row":  # (col-major runs the transposed problem, n x m: another instantiation)
            assert kami.last_kernel() == name.format(dt=dtype), kami.last_kernel()


def _ptr_run(m, n, k, batch, dtype, layout, dist, seed):
    A, B = ki.operands(m, n, k, batch, dtype, dist, seed=seed)
    dA, dB = A.cuda().view(batch, -1), B.cuda().view(batch, -1)
    dC = torch.full((batch, m * n), float("nan"), dtype=A.dtype, device="cuda")
    perm = torch.randperm(batch, generator=torch.Generator().manual_seed(seed)).tolist()
    pa = torch.tensor([dA[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
    pb = torch.tensor([dB[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
    pc = torch.tensor([dC[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
    kami.gemm_batched(m, n, k, batch, dtype, layout, pa, pb, pc)
    torch.cuda.synchronize()
    Cref, S = oracle.gemm(m, n, k, batch, dtype, layout, ki.as_bits(A), ki.as_bits(B), with_scale=True)
    got_bits = oracle.to_row_major(ki.as_bits(dC.cpu()), batch, m, n, layout)
    if dist == "int":
        assert np.array_equal(got_bits, oracle.round_to(Cref, dtype).reshape(batch, m, n))
    else:
        got = oracle.decode(got_bits.reshape(-1), dtype).reshape(batch, m, n)
        assert oracle.normalised_error(got, Cref, S) <= derived_tol(dtype, k)


PTR_STEADY = [
    (64, 64, 64, 97, "kami_tc16_1d_kernel<{dt},ptr>"),
    (32, 32, 32, 401, "kami_tc16_1d_kernel<{dt},ptr>"),
    (128, 128, 64, 29, "kami_tc16_1d_kernel<{dt},ptr>"),    # ptr + per-atom split stores
    (192, 128, 16, 17, "kami_tc16_1d_kernel<{dt},ptr>"),    # m tail, 2 atoms, whole-unit stores
    (160, 96, 32, 17, "kami_tc16_1d_kernel<{dt},ptr>"),     # m tail, 3 atoms of 32 columns
    (144, 48, 64, 17, "kami_tc16_1d_kernel<{dt},ptr>"),     # m tail, 3 atoms of 16 columns
    (64, 64, 40, 97, "kami_tc16_vb_kernel<{dt}>"),          # k = 8 mod 16: the LDG-fed kernel
    (16, 16, 16, 401, "kami_warp_ca_1d<{dt},16>"),          # order 16: warp-level HMMA
]


@pytest.mark.parametrize("case", PTR_STEADY, ids=lambda c: "x".join(map(str, c[:4])))
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_pointer_array_steady(case, dtype):
    m, n, k, batch, name = case
    for layout, dist, seed in (("row", "int", 5), ("col", "unif", 6)):
        _ptr_run(m, n, k, batch, dtype, layout, dist, seed)
        if layout == "row":
            assert kami.last_kernel().startswith(name.format(dt=dtype)), kami.last_kernel()


@pytest.mark.parametrize("s,batch", [(16, 401), (32, 401), (64, 97)])
def test_f64_pointer_array_steady(s, batch):
    for layout, dist, seed in (("row", "unif", 7), ("col", "int", 8)):
        _ptr_run(s, s, s, batch, "f64", layout, dist, seed)
        assert kami.last_kernel().startswith(f"kami_dmma_tma_1d<{s}"), kami.last_kernel()


@pytest.mark.parametrize("s,batch", [(16, 401), (32, 401), (64, 97)])
def test_f64_strided_steady(s, batch):
    for layout, dist, seed in (("row", "unif", 9), ("col", "int", 10)):
        check(s, s, s, batch, "f64", layout, dist, algo="1d_tma", seed=seed)
        assert kami.last_kernel().startswith(f"kami_dmma_tma_1d<{s}"), kami.last_kernel()


@pytest.mark.parametrize("dtype,s,algo,p", [("f64", 32, "1d", 0), ("f64", 32, "2d", 0), ("f64", 32, "3d", 0),
                                            ("f64", 64, "2d", 0), ("f64", 32, "nonca", 0), ("f16", 64, "1d", 4),
                                            ("f16", 64, "2d", 0), ("f16", 64, "3d", 0), ("bf16", 64, "nonca", 0),
                                            ("f16", 16, "1d", 1)])
def test_warp_ca_steady(dtype, s, algo, p):
    for layout, dist, seed in (("row", "int", 11), ("col", "unif", 12)):
        check(s, s, s, 301, dtype, layout, dist, algo=algo, p=p, seed=seed)
        assert "warp" in kami.last_kernel()


# ----------------------------------------------- f4: update form, TF32, FP8


def _f4():
    import test_gpu_f4

    return test_gpu_f4


@pytest.mark.parametrize("shape", [(64, 64, 64, 97), (32, 32, 32, 401), (128, 128, 64, 29), (256, 256, 64, 13)],
                         ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype", ["f16", "bf16", "tf32", "e4m3"])
def test_update_form_steady(shape, dtype):
    f4 = _f4()
    f4.run(*shape, dtype, "row", "int", alpha=2.0, beta=-1.0, seed=13)
    f4.run(*shape, dtype, "col", "unif", alpha=0.75, beta=1.25, seed=14)


@pytest.mark.parametrize("order,batch", [(16, 401), (32, 401), (64, 97)])
def test_update_form_f64_steady(order, batch):
    f4 = _f4()
    f4.run(order, order, order, batch, "f64", "row", "unif", alpha=0.5, beta=1.5, seed=15)
    f4.run(order, order, order, batch, "f64", "col", "int", alpha=2.0, beta=1.0, seed=16)
    assert kami.last_kernel().startswith("kami_dmma_tma")


@pytest.mark.parametrize("shape", [(64, 64, 64, 97), (32, 32, 32, 401), (128, 128, 128, 29), (256, 256, 16, 13)],
                         ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype", ["tf32", "e4m3", "e5m2"])
def test_tf32_fp8_steady(shape, dtype):
    f4 = _f4()
    f4.run(*shape, dtype, "row", "int", seed=17)
    f4.run(*shape, dtype, "col", "unif", seed=18)


# ------------------------------------------------ variable sizes and SpMM


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_vbatched_steady(dtype):
    import test_gpu_vbatched

    test_gpu_vbatched.test_vbatched_mixed_orders(dtype, "row")
    test_gpu_vbatched.test_vbatched_mixed_orders(dtype, "col")


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("shape", [(64, 64, 64), (128, 128, 128), (256, 256, 32), (48, 80, 112)])
def test_spmm_steady(dtype, shape):
    m, n, k = shape
    batch = 61
    for dist in ("unif", "int"):
        rp, cb, v, B = ki.bsr_operands(m, n, k, batch, dtype, density=0.5, dist=dist, seed=19)
        C = torch.full((batch * m * n,), float("nan"), dtype=B.dtype, device="cuda")
        kami.spmm_bsr_strided_batched(m, n, k, batch, dtype, rp.cuda(), cb.cuda(), v.cuda(), B.cuda(), C)
        torch.cuda.synchronize()
        Cref, S = oracle.spmm_bsr(m, n, k, batch, dtype, rp.numpy(), cb.numpy(), ki.as_bits(v), ki.as_bits(B),
                                  with_scale=True)
        got_bits = ki.as_bits(C.cpu()).reshape(batch, m, n)
        if dist == "int":
            assert np.array_equal(got_bits, oracle.round_to(Cref, dtype).reshape(batch, m, n))
        else:
            got = oracle.decode(got_bits.reshape(-1), dtype).reshape(batch, m, n)
            assert oracle.normalised_error(got, Cref, S) <= derived_tol(dtype, k)


def test_cap_changes_nothing_but_speed():
    """Same bits with and without the cap (the knob only resizes the grid)."""
    A, B = ki.operands(64, 64, 64, 301, "f16", "unif", seed=20, device="cuda")
    outs = []
    for cap in (0, 1, 2, CAP, 7):
        kami.set_grid_cap(cap)
        C = torch.full((301 * 64 * 64,), float("nan"), dtype=torch.float16, device="cuda")
        kami.gemm_strided_batched(64, 64, 64, 301, "f16", "row", A, B, C)
        torch.cuda.synchronize()
        outs.append(C.view(torch.int16).cpu())
    kami.set_grid_cap(CAP)
    for o in outs[1:]:
        assert torch.equal(o, outs[0])
