"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (same workload table, same device-side input generation, same entry
point).  The oracle recomputes sampled entries one by one (first/last entries,
the block-diagonal packing boundaries and a stride sample); the small configs
are checked in full.  Properties that hold at any size (finite outputs) are
checked on every element."""
import numpy as np
import pytest
import torch

import kami_inputs as ki
import oracle
import paper_conf_sc_wangdltsl25_b200 as kami
from bench import WORKLOADS, parse_workload

pytestmark = pytest.mark.gpu

TOL = {"f16": 2.0 ** -11, "bf16": 2.0 ** -8, "f64": 0.0}


def sample_entries(batch, n=192):
    idx = set(range(0, batch, max(1, batch // n)))
    idx |= {0, 1, 2, 3, 7, 8, batch - 1, batch - 2, batch - 3}
    return sorted(i for i in idx if 0 <= i < batch)


def run_and_sample(dtype, m, n, k, batch, dist="unif", algo="auto"):
    A, B = ki.operands(m, n, k, batch, dtype, dist, seed=0, device="cuda")
    C = torch.empty(batch * m * n, dtype=A.dtype, device="cuda")
    kami.gemm_strided_batched(m, n, k, batch, dtype, "row", A, B, C, algo=algo)
    torch.cuda.synchronize()
    Cv = C.view(batch, m * n)
    if dtype != "f64":
        assert bool(torch.isfinite(Cv.float()).all())
    else:
        assert bool(torch.isfinite(Cv).all())
    idx = sample_entries(batch)
    worst = 0.0
    for e in idx:
        Ae, Be = ki.operands(m, n, k, 1, dtype, dist, seed=0, entry0=e)  # same values, regenerated on CPU
        Cref, S = oracle.gemm(m, n, k, 1, dtype, "row", ki.as_bits(Ae), ki.as_bits(Be), with_scale=True)
        got = oracle.decode(ki.as_bits(Cv[e].cpu()).reshape(-1), dtype).reshape(1, m, n)
        if dist == "int":
            exp = oracle.round_to(Cref, dtype)
            assert np.array_equal(ki.as_bits(Cv[e].cpu()).reshape(-1), exp), e
        else:
            worst = max(worst, oracle.normalised_error(got, Cref, S))
    return worst, kami.last_kernel()


@pytest.mark.parametrize("wl", ["f16-16", "f16-32", "f16-64", "f16-128", "lr-8", "lr-16", "lr-32", "f64-16", "f64-32",
                                "f64-64"])
def test_fullsize_sampled(wl):
    dtype, m, n, k, batch, _ = WORKLOADS[wl]
    worst, kern = run_and_sample(dtype, m, n, k, batch)
    assert worst <= TOL[dtype] + k * 2.0 ** (-52 if dtype == "f64" else -23), (wl, worst, kern)


def test_config0_full_oracle_bit_exact():
    """BASELINE configs[0]: FP16 16^3 x 1024, integer inputs, every entry, bit-exact."""
    m = n = k = 16
    batch = 1024
    A, B = ki.operands(m, n, k, batch, "f16", "int", seed=0, device="cuda")
    C = torch.empty(batch * m * n, dtype=torch.float16, device="cuda")
    for layout in ("row", "col"):
        kami.gemm_strided_batched(m, n, k, batch, "f16", layout, A, B, C)
        torch.cuda.synchronize()
        Cref = oracle.gemm(m, n, k, batch, "f16", layout, ki.as_bits(A), ki.as_bits(B))
        got = oracle.to_row_major(ki.as_bits(C), batch, m, n, layout)
        assert np.array_equal(got, oracle.round_to(Cref, "f16").reshape(batch, m, n))


@pytest.mark.parametrize("spec", ["bf16-16x16x16:125000", "bf16-64x64x64:125000", "bf16-192x192x192:20000",
                                  "bf16-256x256x256:8000", "bf16-32x128x256:60000", "bf16-256x16x64:40000"])
def test_bf16_sweep_points_sampled(spec):
    dtype, m, n, k, batch, _ = parse_workload(spec)
    worst, _ = run_and_sample(dtype, m, n, k, batch)
    assert worst <= 2.0 ** -8 + k * 2.0 ** -23


def test_fullsize_int_bit_exact_headline():
    worst, _ = run_and_sample("f16", 64, 64, 64, 65536, dist="int")


# ------------------------------------------------ unsampled full-size parity
# (SURVEY.md 8(d) plans the full oracle for configs 1-4:
# every entry of the batch bench.py times, in the same launch configuration)


def run_full(dtype, m, n, k, batch, dist, layout="row", chunk_elems=1 << 27):
    """One launch over the whole batch on device-generated inputs (bench.py's
    path), then every entry against the oracle, in chunks of entries whose
    inputs are regenerated on the CPU (bit-identical generator)."""
    A, B = ki.operands(m, n, k, batch, dtype, dist, seed=0, device="cuda")
    C = torch.full((batch * m * n,), float("nan"), dtype=A.dtype, device="cuda")
    kami.gemm_strided_batched(m, n, k, batch, dtype, layout, A, B, C)
    torch.cuda.synchronize()
    kern = kami.last_kernel()
    del A, B
    Cv = C.view(batch, m * n)
    step = max(1, chunk_elems // (m * n))
    worst = 0.0
    for e0 in range(0, batch, step):
        nb = min(step, batch - e0)
        Ae, Be = ki.operands(m, n, k, nb, dtype, dist, seed=0, entry0=e0)
        Cref, S = oracle.gemm(m, n, k, nb, dtype, layout, ki.as_bits(Ae), ki.as_bits(Be), with_scale=True)
        got_bits = oracle.to_row_major(ki.as_bits(Cv[e0:e0 + nb].cpu()), nb, m, n, layout)
        if dist == "int":
            exp = oracle.round_to(Cref, dtype).reshape(nb, m, n)
            bad = np.argwhere(got_bits != exp)
            assert bad.size == 0, (kern, e0, bad[:3].tolist())
        else:
            got = oracle.decode(got_bits.reshape(-1), dtype).reshape(nb, m, n)
            worst = max(worst, oracle.normalised_error(got, Cref, S))
    return worst, kern


@pytest.mark.parametrize("dist,layout", [("int", "row"), ("unif", "row"), ("int", "col"), ("unif", "col")])
def test_headline_every_entry(dist, layout):
    """BASELINE configs[1] at 64^3 x 65 536 (bench.py's default workload), all
    268 M outputs: int bit-exact, unif within the derived bound; both layouts."""
    worst, kern = run_full("f16", 64, 64, 64, 65536, dist, layout)
    assert kern.startswith("kami_tc16_1d_kernel"), kern
    assert worst <= TOL["f16"] + 64 * 2.0 ** -23, worst


@pytest.mark.parametrize("wl", ["lr-8", "lr-16", "lr-32"])
def test_lowrank_every_entry(wl):
    """BASELINE configs[3]: FP16 256 x 256 x k, k in {8, 16, 32}, batch 16 384, every entry."""
    dtype, m, n, k, batch, _ = WORKLOADS[wl]
    for dist in ("unif", "int"):
        worst, kern = run_full(dtype, m, n, k, batch, dist)
        assert worst <= TOL[dtype] + k * 2.0 ** -23, (wl, worst, kern)


@pytest.mark.parametrize("wl", ["f16-32", "f16-128", "f64-16", "f64-32", "f64-64"])
def test_other_configs_every_entry(wl):
    """The rest of configs[1] and configs[2] at full batch, every entry (unif)."""
    dtype, m, n, k, batch, _ = WORKLOADS[wl]
    worst, kern = run_full(dtype, m, n, k, batch, "unif", chunk_elems=1 << 26)
    tol = k * 2.0 ** -52 if dtype == "f64" else TOL[dtype] + k * 2.0 ** -23
    assert worst <= tol, (wl, worst, kern)


def test_bf16_256cubed_operands_beyond_4GiB():
    """The BF16 sweep's 256^3 chunk (tools/bf16_sweep.py streams 10^6 / 8
    entries through chunks of up to 40 GB): 40 000 entries, so A, B and C are
    5.2 GB each and TMA coordinates / byte offsets cross 2^32.  Sampled entries
    on both sides of the 2^32-byte boundary (entry 32 768) and at the end."""
    m = n = k = 256
    batch = 40000
    A, B = ki.operands(m, n, k, batch, "bf16", "unif", seed=0, device="cuda")
    assert A.numel() * 2 > 2 ** 32
    C = torch.full((batch * m * n,), float("nan"), dtype=torch.bfloat16, device="cuda")
    kami.gemm_strided_batched(m, n, k, batch, "bf16", "row", A, B, C)
    torch.cuda.synchronize()
    del A, B
    Cv = C.view(batch, m * n)
    boundary = 2 ** 32 // (m * k * 2)  # first entry whose A starts at or past 2^32 bytes
    idx = sorted({0, 1, boundary - 2, boundary - 1, boundary, boundary + 1, batch - 2, batch - 1} |
                 set(range(97, batch, 2503)))
    worst = 0.0
    for e in idx:
        Ae, Be = ki.operands(m, n, k, 1, "bf16", "unif", seed=0, entry0=e)
        Cref, S = oracle.gemm(m, n, k, 1, "bf16", "row", ki.as_bits(Ae), ki.as_bits(Be), with_scale=True)
        got = oracle.decode(ki.as_bits(Cv[e].cpu()).reshape(-1), "bf16").reshape(1, m, n)
        worst = max(worst, oracle.normalised_error(got, Cref, S))
    assert worst <= TOL["bf16"] + k * 2.0 ** -23, worst


# ------------------------------------------------------------- edge values

EDGE_SHAPES = [(64, 64, 64, 37), (128, 128, 64, 9), (16, 16, 16, 41), (256, 256, 16, 3), (32, 192, 16, 7)]


def _edge_run(m, n, k, batch, dtype, A, B, layout="row"):
    dC = torch.full((batch * m * n,), float("nan"), dtype=A.dtype, device="cuda")
    kami.gemm_strided_batched(m, n, k, batch, dtype, layout, A.cuda(), B.cuda(), dC)
    torch.cuda.synchronize()
    Cref, S = oracle.gemm(m, n, k, batch, dtype, layout, ki.as_bits(A), ki.as_bits(B), with_scale=True)
    return oracle.to_row_major(ki.as_bits(dC.cpu()), batch, m, n, layout), Cref.reshape(batch, m, n), S


@pytest.mark.parametrize("shape", EDGE_SHAPES, ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_overflow_to_inf(shape, dtype):
    """Products whose exact sum exceeds the output type's range round to +-inf
    (RNE overflow), the rest stay exact: entries alternate between huge
    (+-2^8 for f16, +-2^64 for bf16, so k a b > 65504 resp. > 3.4e38) and
    small integers."""
    m, n, k, batch = shape
    big = 256.0 if dtype == "f16" else 2.0 ** 64
    A, B = ki.operands(m, n, k, batch, dtype, "int", seed=31)
    A = A.view(batch, m * k).clone()
    B = B.view(batch, k * n).clone()
    A[::2] = big
    B[::2] = big
    B[::4] = -big  # entries 0, 4, 8, ...: -inf
    got, Cref, _ = _edge_run(m, n, k, batch, dtype, A.reshape(-1), B.reshape(-1))
    exp = oracle.round_to(Cref, dtype).reshape(batch, m, n)
    assert np.isinf(Cref[0]).sum() == 0  # the oracle's sum is finite; only the rounding overflows
    assert np.array_equal(got, exp)
    inf_bits = 0x7C00 if dtype == "f16" else 0x7F80
    assert (got[2] == inf_bits).all() and (got[0] == (inf_bits | 0x8000)).all()


@pytest.mark.parametrize("shape", EDGE_SHAPES, ids=lambda s: "x".join(map(str, s)))
def test_fp16_subnormal_outputs(shape):
    """FP16 outputs in the subnormal range (< 2^-14): inputs are small integers
    times 2^-12 (normal fp16), products i j 2^-24, sums |sum i j| < 2048 exact
    in FP32 and exactly representable in fp16 (subnormal below 2^-14, quantum
    2^-24) -- bit-exact."""
    m, n, k, batch = shape
    A, B = ki.operands(m, n, k, batch, "f16", "int", seed=32)
    A = (A.double() * 2.0 ** -12).half()
    B = (B.double() * 2.0 ** -12).half()
    got, Cref, _ = _edge_run(m, n, k, batch, "f16", A, B)
    exp = oracle.round_to(Cref, "f16").reshape(batch, m, n)
    sub = (exp & 0x7C00) == 0
    assert sub.mean() > 0.5  # most outputs are subnormal (or zero)
    assert np.array_equal(got, exp)


@pytest.mark.parametrize("shape", EDGE_SHAPES, ids=lambda s: "x".join(map(str, s)))
@pytest.mark.parametrize("dtype", ["f16", "bf16", "f64"])
@pytest.mark.parametrize("layout", ["row", "col"])
def test_zero_scale_rows_and_columns(shape, dtype, layout):
    """Rows of A and columns of B that are all zero make S = 0 for whole rows /
    columns of C: those outputs must be exactly zero (north_star rule), the
    rest within tolerance."""
    m, n, k, batch = shape
    A, B = ki.operands(m, n, k, batch, dtype, "unif", seed=33)
    A3 = oracle.to_row_major(ki.as_bits(A), batch, m, k, layout).copy()
    B3 = oracle.to_row_major(ki.as_bits(B), batch, k, n, layout).copy()
    A3[:, 1::3, :] = 0  # rows 1, 4, 7, ... of every A
    B3[:, :, 2::5] = 0  # columns 2, 7, 12, ... of every B
    A3[-1] = 0          # the whole last entry
    def pack(X):
        X = X if layout == "row" else X.transpose(0, 2, 1)
        t = torch.from_numpy(np.ascontiguousarray(X).reshape(-1).copy())
        return t if dtype == "f64" else t.view(torch.int16).view(ki.TORCH_DTYPES[dtype])
    got_bits, Cref, S = _edge_run(m, n, k, batch, dtype, pack(A3), pack(B3), layout)
    got = oracle.decode(got_bits.reshape(-1), dtype).reshape(batch, m, n)
    assert (S[:, 1::3, :] == 0).all() and (S[:, :, 2::5] == 0).all()
    assert (got[:, 1::3, :] == 0).all() and (got[:, :, 2::5] == 0).all() and (got[-1] == 0).all()
    tol = k * 2.0 ** -52 if dtype == "f64" else TOL[dtype] + k * 2.0 ** -23
    assert oracle.normalised_error(got, Cref, S) <= tol
