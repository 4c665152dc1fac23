"""C-ABI tests that need no GPU: libkami.so loads, exports every symbol
include/kami.h declares, rejects bad arguments before any launch, and its
host-side planner / paper cost model agree with the oracle's."""
import ctypes
import json
import os
import re

import pytest

import paper_conf_sc_wangdltsl25_b200 as kami
from oracle import cost_model

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "kami.h")

INVALID, UNSUP, MISAL = 1, 2, 3


def header_functions():
    txt = open(HDR).read()
    return sorted(set(re.findall(r"^\s*(?:kami_status_t|const char\s*\*|int)\s+(kami_\w+)\s*\(", txt, re.M)))


def test_loads_and_exports_every_declared_symbol():
    L = kami.lib()
    declared = header_functions()
    assert len(declared) >= 10
    for name in declared:
        assert hasattr(L, name), name
    assert sorted(kami.EXPORTS) == declared
    assert L.kami_version() == (0 << 16) | 1


def test_status_strings():
    L = kami.lib()
    for code, name in kami.STATUS.items():
        assert L.kami_status_string(code).decode() == name


FAKE = 0x10000  # never dereferenced: every case below fails validation first


@pytest.mark.parametrize("args,code", [
    ((0, 16, 16, 1, 0, 0), INVALID),       # m <= 0
    ((16, -1, 16, 1, 0, 0), INVALID),      # n <= 0
    ((16, 16, 0, 1, 0, 0), INVALID),       # k <= 0
    ((16, 16, 16, -1, 0, 0), INVALID),     # batch < 0
    ((16, 16, 16, 1, 7, 0), INVALID),      # unknown dtype
    ((16, 16, 16, 1, 0, 5), INVALID),      # unknown layout
    ((20, 16, 16, 1, 0, 0), UNSUP),        # 16-bit m not a multiple of 8
    ((16, 12, 16, 1, 1, 0), UNSUP),        # 16-bit n not a multiple of 8
    ((16, 16, 12, 1, 0, 0), UNSUP),        # 16-bit k not a multiple of 8
    ((272, 16, 16, 1, 0, 0), UNSUP),       # > 256
    ((44, 48, 48, 1, 2, 0), UNSUP),        # fp64 m not a multiple of 8
    ((48, 48, 20, 1, 2, 0), UNSUP),        # fp64 k not a multiple of 8
])
def test_rejects_before_launch(args, code):
    L = kami.lib()
    m, n, k, batch, dt, lay = args
    assert L.kami_gemm_strided_batched(m, n, k, batch, dt, lay, FAKE, FAKE, FAKE, None) == code


def test_null_misaligned_and_empty():
    L = kami.lib()
    assert L.kami_gemm_strided_batched(64, 64, 64, 4, 0, 0, None, FAKE, FAKE, None) == INVALID
    assert L.kami_gemm_strided_batched(64, 64, 64, 4, 0, 0, FAKE + 2, FAKE, FAKE, None) == MISAL
    assert L.kami_gemm_strided_batched(64, 64, 64, 4, 0, 0, FAKE, FAKE, FAKE + 8, None) == MISAL
    # batch == 0 is a no-op success even with null pointers
    assert L.kami_gemm_strided_batched(64, 64, 64, 0, 0, 0, None, None, None, None) == 0
    assert L.kami_gemm(64, 64, 64, 2, 0, 0, FAKE, FAKE, FAKE, None) == INVALID  # kami_gemm needs batch == 1
    assert L.kami_gemm_batched(64, 64, 64, 3, 0, 0, None, FAKE, FAKE, None) == INVALID
    assert L.kami_gemm_strided_batched_ex(64, 64, 64, 1, 0, 0, FAKE, FAKE, FAKE, 10, 0, None) == INVALID
    assert L.kami_gemm_strided_batched_ex(64, 64, 64, 1, 0, 0, FAKE, FAKE, FAKE, 1, -2, None) == INVALID
    assert L.kami_gemm_strided_batched_host(64, 64, 64, 0, 0, 0, None, None, None) == 0
    assert L.kami_gemm_strided_batched_host(64, 64, 64, 2, 0, 0, None, None, None) == INVALID


def test_spmm_zmorton_ex_host_checks():
    """Schedule selection of the Z-Morton SpMM entry point, decided before any
    launch: unknown schedules and the 2D pair on m <= 128 are NOT_SUPPORTED,
    an empty batch is a no-op, null arrays are INVALID."""
    L = kami.lib()
    f = L.kami_spmm_zmorton_strided_batched_ex
    for algo in (3, 4, 5, 6, 7):  # 3D, non-CA, TMA-1D, TMEM variants: no sparse form
        assert f(256, 64, 64, 4, 0, FAKE, FAKE, FAKE, 16, FAKE, FAKE, algo, None) == UNSUP
    assert f(128, 64, 64, 4, 0, FAKE, FAKE, FAKE, 16, FAKE, FAKE, 8, None) == UNSUP  # pair needs m > 128
    assert f(128, 64, 64, 4, 0, FAKE, FAKE, FAKE, 16, FAKE, FAKE, 2, None) == UNSUP
    for algo in (0, 1, 2, 8):
        assert f(256, 64, 64, 0, 0, None, None, None, 16, None, None, algo, None) == 0
        assert f(256, 64, 64, 4, 0, None, FAKE, FAKE, 16, FAKE, FAKE, algo, None) == INVALID
    assert f(256, 64, 64, 4, 2, FAKE, FAKE, FAKE, 16, FAKE, FAKE, 0, None) == UNSUP  # FP64: no sparse path
    assert f(256, 64, 64, 4, 0, FAKE, FAKE, FAKE, 65, FAKE, FAKE, 0, None) == INVALID  # max_nnzb > (m/16)(k/16)


def test_plan_host_logic():
    p = kami.plan(64, 64, 64, "f16")
    assert p["kernel"] == "tcgen05" and p["algo"] == "1d" and p["p"] == 4 and p["stages"] >= 2
    # entries in flight per CTA: G = 2 entries per 128-lane MMA tile x stages
    assert p["entries_per_cta"] == 2 * p["stages"]
    p = kami.plan(64, 64, 64, "f64")
    # FP64 AUTO: the measured-fastest schedule (1D with TMA-fed broadcast on DMMA)
    assert p["kernel"] == "dmma_tma" and p["algo"] == "1d_tma"
    q = kami.plan(8, 8, 8, "f64")
    assert q["kernel"] == "warp_ca" and q["algo"] == "1d"
    for algo in ("1d", "2d", "3d", "nonca"):
        q = kami.plan(32, 32, 32, "f64", algo=algo)
        assert q["algo"] == algo and q["kernel"] == "warp_ca"
    with pytest.raises(kami.KamiError):
        kami.plan(64, 64, 64, "f64", algo="2d", p=3)


def test_plan_covers_the_16bit_grid():
    """Every shape of the 16-bit grid has a plan; AUTO is the model's pick (a
    tcgen05 kernel or, for some thin tiles, the one-warp register-resident 1D),
    and 1D with p = 0 always names the tcgen05 kernel of the shape.  The
    transposed-product kernel is picked only where it runs (thin m, n a
    multiple of 64, k in {16, 32, 64})."""
    for m in (8, 16, 24, 32, 48, 64, 128, 192, 256):
        for n in (8, 16, 40, 64, 256):
            for k in (8, 16, 40, 64, 256):
                p = kami.plan(m, n, k, "bf16")
                assert p["kernel"] in ("tcgen05", "tcgen05_ts", "tcgen05_ldg", "warp_ca", "tcgen05_xt"), (m, n, k, p)
                if p["kernel"] == "tcgen05_xt":
                    assert m in (16, 32) and n % 64 == 0 and k in (16, 32, 64), (m, n, k, p)
                if p["kernel"] == "warp_ca":
                    assert p["algo"] == "1d" and p["p"] == 1, (m, n, k, p)
                q = kami.plan(m, n, k, "bf16", algo="1d")  # 1D with p = 0: the tcgen05 family
                want = "tcgen05" if m % 16 == 0 and n % 16 == 0 else "tcgen05_ldg"
                assert q["kernel"] == want and q["stages"] >= 2, (m, n, k, q)


def test_plan_ring_depth_rules():
    """tcgen05 ring depth (DESIGN.md 4.1 'Stages and bytes in flight'): ~96 KB of TMA loads in
    flight, at least 3 stages where shared memory allows, at most 4 for write-heavy units."""
    assert kami.plan(64, 64, 64, "f16")["stages"] == 3          # 32 KB stages under the 96 KB cap
    assert kami.plan(192, 192, 192, "bf16")["stages"] == 3      # 40 KB stages: raised from 2 to 3
    assert kami.plan(256, 256, 256, "bf16")["stages"] == 2      # 48 KB stages + 128 KB staging: 2 fit
    assert kami.plan(64, 64, 64, "e4m3")["stages"] == 4         # FP8 in / FP16 out: write-heavy cap
    assert kami.plan(256, 256, 16, "f16")["stages"] == 4        # low-rank: write-heavy cap (was 8)
    assert kami.plan(16, 16, 256, "bf16")["stages"] >= 3        # read-heavy small tiles keep a deep ring


GOLD = json.load(open(os.path.join(ROOT, "tests", "golden", "cost_model_examples.json")))


@pytest.mark.parametrize("case", GOLD["cases"], ids=lambda c: c["variant"])
def test_library_paper_cost_matches_worked_examples(case):
    c = GOLD["common"]
    V, Tcm, Tcp, Tall = kami.paper_cost(case["variant"], c["m"], c["n"], c["k"], case["p"], c["s_e"], c["L_sm"],
                                        c["B_sm"], c["theta_r"], c["theta_w"], c["O_tc"], c["n_tc"])
    assert (V, Tcm, Tall) == (case["V_cm"], case["T_cm"], case["T_all"])
    if case["T_cp"] is not None:
        assert Tcp == case["T_cp"]


@pytest.mark.parametrize("variant,p", [("1d", 4), ("1d", 8), ("2d", 4), ("2d", 16), ("3d", 8)])
def test_library_cost_model_matches_oracle_model(variant, p):
    args = (96, 64, 128, p, 2, 29, 128, 0.9, 0.7, 256, 4)
    ours = kami.paper_cost(variant, *args)
    ref = cost_model.paper_model(variant, *args)
    assert ours == pytest.approx((ref.V_cm, ref.T_cm, ref.T_cp, ref.T_all), rel=1e-12)


def test_product_and_oracle_share_no_code():
    """The oracle and the CUDA path are independent (task rule 3): no
    import/include crosses between oracle/ and the product package."""
    prod = os.path.join(ROOT, "paper_conf_sc_wangdltsl25_b200")
    for dirpath, _, files in os.walk(prod):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+(oracle|kami_inputs)\b|#include\s+\"[^\"]*oracle", txt,
                                     re.M), f
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c")):
            txt = open(os.path.join(ROOT, "oracle", f)).read()
            assert not re.search(r"^\s*(import|from)\s+(paper_conf_sc_wangdltsl25_b200|kami_inputs)\b|"
                                 r"#include\s+\"[^\"]*(kami|csrc)", txt, re.M), f


def test_xt_plan_host_rules():
    """The transposed-product kernel (kernel 7, KAMI_ALGO_1D_XT): the shapes it
    runs, its unit geometry, and the model picks measured on one B200
    (profiles/r2/xt_r2.md): XT for thin m with k = 16 and n >= 128 / the pair
    tiles of n = 64, the SS kernel where its single-entry tiles stream better."""
    for m, n, k in [(16, 128, 16), (16, 192, 16), (16, 64, 16), (32, 256, 64)]:
        p = kami.plan(m, n, k, "bf16", algo="1d_xt")
        assert p["kernel"] == "tcgen05_xt" and p["algo"] == "1d_xt", (m, n, k, p)
        assert p["stages"] >= 3 and p["entries_per_cta"] >= 3, p
    for m, n, k in [(48, 128, 16), (16, 96, 16), (16, 128, 48), (16, 128, 128), (8, 128, 16)]:
        with pytest.raises(kami.KamiError):
            kami.plan(m, n, k, "bf16", algo="1d_xt")
    with pytest.raises(kami.KamiError):
        kami.plan(16, 128, 16, "f64", algo="1d_xt")
    assert kami.plan(16, 128, 16, "bf16")["kernel"] == "tcgen05_xt"   # 0.88 vs 0.43 (SS)
    assert kami.plan(16, 192, 16, "bf16")["kernel"] == "tcgen05_xt"   # 0.87 vs 0.52
    assert kami.plan(16, 64, 16, "bf16")["kernel"] == "tcgen05_xt"    # 0.88 vs 0.65 (pair tiles)
    assert kami.plan(16, 192, 64, "bf16")["kernel"] == "tcgen05"      # 1.00 vs 0.96
    assert kami.plan(64, 64, 64, "f16")["kernel"] == "tcgen05"        # the headline stays on SS
    # column-major C is the row problem n x m: thin n runs the XT kernel
    assert kami.plan(128, 16, 16, "bf16", layout="col")["kernel"] == "tcgen05_xt"
