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
