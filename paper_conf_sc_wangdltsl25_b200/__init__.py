"""paper_conf_sc_wangdltsl25_b200 -- B200-native KAMI batched small GEMM.

Thin Python binding of the C ABI in ``include/kami.h`` (libkami.so, built
in-tree by ``build.py``).  Argument marshalling only: every step of the GEMM
runs in the library's CUDA kernels.  There is no CPU fallback -- if the
shared library is missing or a call fails, a ``KamiError`` is raised.

PyTorch is used only for device memory and the current CUDA stream.
"""
from __future__ import annotations

import ctypes
import os

__all__ = [
    "KamiError", "lib", "gemm", "gemm_batched", "gemm_strided_batched", "gemm_strided_batched_host",
    "plan", "paper_cost", "last_kernel", "probe_dmma_peak", "set_grid_cap", "grid_cap", "DTYPE", "LAYOUT", "ALGO",
    "SO_PATH",
]

_HERE = os.path.dirname(os.path.abspath(__file__))
# KAMI_LIB may point at another build of the same library (A/B experiments)
SO_PATH = os.environ.get("KAMI_LIB") or os.path.join(_HERE, "libkami.so")

DTYPE = {"f16": 0, "bf16": 1, "f64": 2, "tf32": 3, "e4m3": 4, "e5m2": 5}
LAYOUT = {"row": 0, "col": 1}
ALGO = {"auto": 0, "1d": 1, "2d": 2, "3d": 3, "nonca": 4, "1d_tma": 5, "1d_tmem": 6, "3d_tmem": 7, "2d_pair": 8, "1d_xt": 9}
STATUS = {0: "KAMI_SUCCESS", 1: "KAMI_ERROR_INVALID_VALUE", 2: "KAMI_ERROR_NOT_SUPPORTED",
          3: "KAMI_ERROR_MISALIGNED", 4: "KAMI_ERROR_CUDA"}

# every symbol include/kami.h declares (checked by tests/test_abi.py)
EXPORTS = [
    "kami_gemm", "kami_gemm_batched", "kami_gemm_strided_batched", "kami_gemm_strided_batched_ex",
    "kami_gemm_strided_batched_host", "kami_release_workspace", "kami_plan", "kami_paper_cost",
    "kami_status_string", "kami_last_kernel", "kami_version", "kami_gemm_block_level", "kami_gemm_vbatched",
    "kami_spmm_bsr_strided_batched", "kami_gemm_strided_batched_axpby", "kami_probe_dmma_peak",
    "kami_set_grid_cap", "kami_plan_candidates", "kami_spmm_zmorton_strided_batched", "kami_last_cuda_error",
    "kami_spmm_zmorton_strided_batched_ex",
]


class KamiError(RuntimeError):
    def __init__(self, status: int, what: str = ""):
        self.status = status
        self.name = STATUS.get(status, f"status {status}")
        super().__init__(f"{what}: {self.name}" if what else self.name)


class KamiPlan(ctypes.Structure):
    _fields_ = [("algo", ctypes.c_int), ("p", ctypes.c_int), ("kernel", ctypes.c_int),
                ("entries_per_cta", ctypes.c_int), ("stages", ctypes.c_int), ("kslice_regs_pct", ctypes.c_int),
                ("t_all_cycles", ctypes.c_double)]


class KamiCandidate(ctypes.Structure):
    _fields_ = [("algo", ctypes.c_int), ("p", ctypes.c_int), ("kernel", ctypes.c_int),
                ("model_cycles_per_entry", ctypes.c_double), ("model_tflops", ctypes.c_double),
                ("bound", ctypes.c_int)]


BOUND = {0: "hbm", 1: "tensor", 2: "smem", 3: "tma", 4: "issue", 5: "latency"}
KERNEL = {0: "tcgen05", 1: "warp_ca", 2: "dmma_tma", 3: "tcgen05_ts", 4: "dmma_gen", 5: "tcgen05_ldg",
          6: "tcgen05_pair", 7: "tcgen05_xt"}

_lib = None


def lib() -> ctypes.CDLL:
    """Load libkami.so (fails loudly if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(SO_PATH):
        raise ImportError(f"{SO_PATH} is missing: run `python -m paper_conf_sc_wangdltsl25_b200.build` "
                          "(there is no CPU fallback)")
    L = ctypes.CDLL(SO_PATH)
    i, i64, vp, st = ctypes.c_int, ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p
    L.kami_gemm.argtypes = [i, i, i, i64, i, i, vp, vp, vp, st]
    L.kami_gemm_batched.argtypes = [i, i, i, i64, i, i, vp, vp, vp, st]
    L.kami_gemm_strided_batched.argtypes = [i, i, i, i64, i, i, vp, vp, vp, st]
    L.kami_gemm_strided_batched_ex.argtypes = [i, i, i, i64, i, i, vp, vp, vp, i, i, st]
    L.kami_gemm_strided_batched_host.argtypes = [i, i, i, i64, i, i, vp, vp, vp]
    L.kami_gemm_block_level.argtypes = [i, i, i, i64, i, i, i, i, i, vp, vp, vp, vp, st]
    L.kami_gemm_vbatched.argtypes = [i64, vp, vp, vp, i, i, i, i, i, vp, vp, vp, st]
    L.kami_spmm_bsr_strided_batched.argtypes = [i, i, i, i64, i, vp, vp, vp, i, vp, vp, st]
    L.kami_spmm_zmorton_strided_batched.argtypes = [i, i, i, i64, i, vp, vp, vp, i, vp, vp, st]
    L.kami_spmm_zmorton_strided_batched.restype = ctypes.c_int
    L.kami_spmm_zmorton_strided_batched_ex.argtypes = [i, i, i, i64, i, vp, vp, vp, i, vp, vp, i, st]
    L.kami_spmm_zmorton_strided_batched_ex.restype = ctypes.c_int
    L.kami_gemm_strided_batched_axpby.argtypes = [i, i, i, i64, i, i, ctypes.c_double, vp, vp, ctypes.c_double, vp,
                                                  st]
    L.kami_release_workspace.argtypes = []
    L.kami_probe_dmma_peak.argtypes = [ctypes.c_double, ctypes.POINTER(ctypes.c_double),
                                       ctypes.POINTER(ctypes.c_double), st]
    L.kami_probe_dmma_peak.restype = ctypes.c_int
    L.kami_plan_candidates.argtypes = [i, i, i, i, i, ctypes.POINTER(KamiCandidate), i, ctypes.POINTER(i)]
    L.kami_plan_candidates.restype = ctypes.c_int
    L.kami_set_grid_cap.argtypes = [i]
    L.kami_set_grid_cap.restype = ctypes.c_int
    L.kami_plan.argtypes = [i, i, i, i, i, i, i, ctypes.POINTER(KamiPlan)]
    d = ctypes.c_double
    L.kami_paper_cost.argtypes = [i, d, d, d, d, d, d, d, d, d, d, d, ctypes.POINTER(ctypes.c_double)]
    for f in ("kami_gemm", "kami_gemm_batched", "kami_gemm_strided_batched", "kami_gemm_strided_batched_ex",
              "kami_gemm_block_level", "kami_gemm_vbatched", "kami_spmm_bsr_strided_batched",
              "kami_gemm_strided_batched_axpby",
              "kami_gemm_strided_batched_host", "kami_release_workspace", "kami_plan", "kami_paper_cost"):
        getattr(L, f).restype = ctypes.c_int
    L.kami_status_string.restype = ctypes.c_char_p
    L.kami_status_string.argtypes = [ctypes.c_int]
    L.kami_last_kernel.restype = ctypes.c_char_p
    L.kami_last_kernel.argtypes = []
    L.kami_last_cuda_error.restype = ctypes.c_char_p
    L.kami_last_cuda_error.argtypes = []
    L.kami_version.restype = ctypes.c_int
    _lib = L
    return L


def _check(status: int, what: str):
    if status != 0:
        if status == 4:  # KAMI_ERROR_CUDA: append the runtime's message
            what = f"{what} ({lib().kami_last_cuda_error().decode()})"
        raise KamiError(status, what)


def _enum(table, v, what):
    if isinstance(v, int):
        return v
    try:
        return table[v.lower()]
    except KeyError:
        raise ValueError(f"unknown {what} {v!r}") from None


def _stream(stream):
    if stream is not None:
        return int(getattr(stream, "cuda_stream", stream))
    import torch

    return int(torch.cuda.current_stream().cuda_stream)


def _dtype_of(t):
    import torch

    return {torch.float16: "f16", torch.bfloat16: "bf16", torch.float64: "f64", torch.float32: "tf32",
            torch.float8_e4m3fn: "e4m3", torch.float8_e5m2: "e5m2"}[t.dtype]


def _ptr(x):
    return None if x is None else (x if isinstance(x, int) else x.data_ptr())


def gemm_strided_batched(m, n, k, batch, dtype, layout, A, B, C, algo="auto", p=0, stream=None):
    """C_b = A_b B_b for b < batch on device buffers (torch tensors or raw
    device addresses).  Entries are packed; ``layout`` applies to all three."""
    _check(lib().kami_gemm_strided_batched_ex(
        m, n, k, batch, _enum(DTYPE, dtype, "dtype"), _enum(LAYOUT, layout, "layout"),
        _ptr(A), _ptr(B), _ptr(C), _enum(ALGO, algo, "algo"), p, _stream(stream)), "kami_gemm_strided_batched")
    return C


def gemm_strided_batched_axpby(m, n, k, batch, dtype, layout, alpha, A, B, beta, C, stream=None):
    """C <- alpha A B + beta C per entry (C read iff beta != 0)."""
    _check(lib().kami_gemm_strided_batched_axpby(
        m, n, k, batch, _enum(DTYPE, dtype, "dtype"), _enum(LAYOUT, layout, "layout"), float(alpha), _ptr(A),
        _ptr(B), float(beta), _ptr(C), _stream(stream)), "kami_gemm_strided_batched_axpby")
    return C


def gemm(A, B, out=None, layout="row", algo="auto", p=0, stream=None):
    """Torch convenience: A [batch, m, k] (or [m, k]) times B -> C, on the GPU.

    For layout "row" the tensors are the usual row-major views; for "col"
    each matrix is stored column-major (pass the transposed storage)."""
    import torch

    single = A.dim() == 2
    A3 = A.unsqueeze(0) if single else A
    B3 = B.unsqueeze(0) if single else B
    if not (A3.is_cuda and B3.is_cuda and A3.is_contiguous() and B3.is_contiguous()):
        raise ValueError("A and B must be contiguous CUDA tensors")
    batch = A3.shape[0]
    if layout == "row":
        m, k = A3.shape[1], A3.shape[2]
        n = B3.shape[2]
        shape = (batch, m, n)
    else:
        k, m = A3.shape[1], A3.shape[2]
        n = B3.shape[1]
        shape = (batch, n, m)
    if out is None:
        out = torch.empty(shape, dtype=A3.dtype, device=A3.device)
    gemm_strided_batched(m, n, k, batch, _dtype_of(A3), layout, A3, B3, out, algo, p, stream)
    return out[0] if single else out


def gemm_batched(m, n, k, batch, dtype, layout, A_ptrs, B_ptrs, C_ptrs, stream=None):
    """Pointer-array form: A_ptrs/B_ptrs/C_ptrs are device int64 tensors of
    per-entry device addresses (cuBLAS *gemmBatched convention)."""
    _check(lib().kami_gemm_batched(m, n, k, batch, _enum(DTYPE, dtype, "dtype"), _enum(LAYOUT, layout, "layout"),
                                   _ptr(A_ptrs), _ptr(B_ptrs), _ptr(C_ptrs), _stream(stream)), "kami_gemm_batched")


def gemm_vbatched(batch, m_arr, n_arr, k_arr, max_m, max_n, max_k, dtype, layout, A_ptrs, B_ptrs, C_ptrs,
                  stream=None):
    """Variable-size batched GEMM: per-entry sizes and pointers in device int32 /
    int64 tensors (MAGMA vbatched convention)."""
    _check(lib().kami_gemm_vbatched(batch, _ptr(m_arr), _ptr(n_arr), _ptr(k_arr), max_m, max_n, max_k,
                                    _enum(DTYPE, dtype, "dtype"), _enum(LAYOUT, layout, "layout"), _ptr(A_ptrs),
                                    _ptr(B_ptrs), _ptr(C_ptrs), _stream(stream)), "kami_gemm_vbatched")


def spmm_bsr_strided_batched(m, n, k, batch, dtype, row_ptr, col_blk, vals, B, C, stream=None):
    """Block-sparse A (BSR, 16x16 blocks; Sec. 4.6) times dense B.
    row_ptr [batch, m/16+1] and col_blk [batch, max_nnzb] int32, vals
    [batch, max_nnzb, 16, 16], B/C packed row-major -- all device tensors."""
    max_nnzb = col_blk.shape[-1]
    _check(lib().kami_spmm_bsr_strided_batched(m, n, k, batch, _enum(DTYPE, dtype, "dtype"), _ptr(row_ptr),
                                               _ptr(col_blk), _ptr(vals), max_nnzb, _ptr(B), _ptr(C),
                                               _stream(stream)), "kami_spmm_bsr_strided_batched")
    return C


def spmm_zmorton_strided_batched(m, n, k, batch, dtype, nnzb, zcode, vals, B, C, stream=None, algo="auto"):
    """Block-sparse A in Z-Morton block storage (Sec. 4.6, Fig. 7(b))
    times dense B.  nnzb [batch] and zcode [batch, max_nnzb] int32, vals
    [batch, max_nnzb, 16, 16], B/C packed row-major -- all device tensors.
    algo: "auto" / "1d" (Morton-decoding 1D kernel) or "2d" / "2d_pair" (CTA pair)."""
    max_nnzb = zcode.shape[-1]
    _check(lib().kami_spmm_zmorton_strided_batched_ex(m, n, k, batch, _enum(DTYPE, dtype, "dtype"), _ptr(nnzb),
                                                      _ptr(zcode), _ptr(vals), max_nnzb, _ptr(B), _ptr(C),
                                                      _enum(ALGO, algo, "algo"), _stream(stream)),
           "kami_spmm_zmorton_strided_batched_ex")
    return C


def gemm_single(m, n, k, dtype, layout, A, B, C, stream=None):
    _check(lib().kami_gemm(m, n, k, 1, _enum(DTYPE, dtype, "dtype"), _enum(LAYOUT, layout, "layout"),
                           _ptr(A), _ptr(B), _ptr(C), _stream(stream)), "kami_gemm")


def gemm_strided_batched_host(m, n, k, batch, dtype, layout, A, B, C):
    """End-to-end entry point on HOST buffers (pinned recommended): the
    library pipelines host->device copies, kernels and device->host copies
    and returns when C is complete on the host."""
    _check(lib().kami_gemm_strided_batched_host(m, n, k, batch, _enum(DTYPE, dtype, "dtype"),
                                                _enum(LAYOUT, layout, "layout"), _ptr(A), _ptr(B), _ptr(C)),
           "kami_gemm_strided_batched_host")


def gemm_block_level(m, n, k, batch, dtype, layout, A, B, C, algo="1d", p=0, reps=1000, cycles=None,
                     stream=None):
    """Block-level (on-chip-resident) mode: C_b = reps * A_b B_b with the CA
    schedule repeated ``reps`` times on chip; ``cycles`` (device int64, 2*batch,
    zeroed) receives per-entry [communication, computation] clock64 sums."""
    _check(lib().kami_gemm_block_level(m, n, k, batch, _enum(DTYPE, dtype, "dtype"), _enum(LAYOUT, layout, "layout"),
                                       _enum(ALGO, algo, "algo"), p, reps, _ptr(A), _ptr(B), _ptr(C), _ptr(cycles),
                                       _stream(stream)), "kami_gemm_block_level")
    return C


def release_workspace():
    _check(lib().kami_release_workspace(), "kami_release_workspace")


def plan(m, n, k, dtype, layout="row", algo="auto", p=0) -> dict:
    out = KamiPlan()
    _check(lib().kami_plan(m, n, k, _enum(DTYPE, dtype, "dtype"), _enum(LAYOUT, layout, "layout"),
                           _enum(ALGO, algo, "algo"), p, ctypes.byref(out)), "kami_plan")
    inv = {v: k for k, v in ALGO.items()}
    return {"algo": inv[out.algo], "p": out.p, "kernel": KERNEL[out.kernel],
            "entries_per_cta": out.entries_per_cta, "stages": out.stages, "kslice_regs_pct": out.kslice_regs_pct,
            "t_all_cycles": out.t_all_cycles}


def plan_candidates(m, n, k, dtype, layout="row") -> list:
    """Every schedule the library can run for the shape, with the planner
    model's prediction (AUTO takes the smallest model_cycles_per_entry)."""
    buf = (KamiCandidate * 32)()
    cnt = ctypes.c_int(0)
    _check(lib().kami_plan_candidates(m, n, k, _enum(DTYPE, dtype, "dtype"), _enum(LAYOUT, layout, "layout"), buf, 32,
                                      ctypes.byref(cnt)), "kami_plan_candidates")
    inv = {v: k_ for k_, v in ALGO.items()}
    return [{"algo": inv[c.algo], "p": c.p, "kernel": KERNEL[c.kernel], "model_cycles_per_entry": c.model_cycles_per_entry,
             "model_tflops": c.model_tflops, "bound": BOUND[c.bound]} for c in buf[:min(cnt.value, 32)]]


def paper_cost(variant, m, n, k, p, s_e, L_sm, B_sm, theta_r, theta_w, O_tc, n_tc):
    """The library's paper-faithful cost model (Eqs. 1-12): (V_cm, T_cm, T_cp, T_all)."""
    out = (ctypes.c_double * 4)()
    _check(lib().kami_paper_cost(_enum(ALGO, variant, "variant"), m, n, k, p, s_e, L_sm, B_sm, theta_r, theta_w,
                                 O_tc, n_tc, out), "kami_paper_cost")
    return tuple(out)


def probe_dmma_peak(min_ms=200.0, stream=None):
    """FP64 DMMA peak measured on the current device: (burst, sustained) TFLOP/s."""
    b, s_ = ctypes.c_double(), ctypes.c_double()
    _check(lib().kami_probe_dmma_peak(float(min_ms), ctypes.byref(b), ctypes.byref(s_), _stream(stream)),
           "kami_probe_dmma_peak")
    return b.value, s_.value


def set_grid_cap(max_ctas: int):
    """Test knob: cap every persistent kernel's grid (0 = no cap)."""
    _check(lib().kami_set_grid_cap(int(max_ctas)), "kami_set_grid_cap")


class grid_cap:
    """Context manager: ``with kami.grid_cap(4): ...`` runs the enclosed calls
    with at most 4 CTAs per persistent kernel (steady-state parity tests)."""

    def __init__(self, max_ctas: int):
        self.max_ctas = max_ctas

    def __enter__(self):
        set_grid_cap(self.max_ctas)
        return self

    def __exit__(self, *exc):
        set_grid_cap(0)
        return False


def last_kernel() -> str:
    return lib().kami_last_kernel().decode()
