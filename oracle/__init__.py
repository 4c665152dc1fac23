"""KAMI oracle -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product package ``paper_conf_sc_wangdltsl25_b200`` never imports it and it
never imports the product package; the two share no code.  The only module
both sides use is ``kami_inputs`` (seeded input generation, no GEMM
arithmetic).

Contents
--------
``gemm``          -- ctypes front end of ``oracle.c``: the plain FP64 triple
                     loop C_ref[b,i,j] = sum_l A[b,i,l] B[b,l,j] (PAPER.md L62,
                     Sec. 2.1; batched: L69), plus the error scale
                     S[b,i,j] = sum_l |A||B| (BASELINE.json north_star).
``round_f16`` / ``round_bf16`` -- RNE double -> 16-bit encoders (bit-exact
                     expectation for integer-valued inputs).
``normalised_error`` -- max_e |C_gpu - C_ref| / S (north_star metric).
``cost_model``    -- the paper's cycle model, Eqs. (1)-(12), step by step.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")

DTYPES = {"f16": 0, "bf16": 1, "f64": 2, "f32": 3, "tf32": 3, "e4m3": 4, "e5m2": 5}
LAYOUTS = {"row": 0, "col": 1}


def build(force: bool = False) -> str:
    """Compile oracle.c into liboracle.so with gcc -O2 (no BLAS, no intrinsics)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(
            ["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-pthread", _SRC, "-o", _SO, "-lm"]
        )
    return _SO


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        L.oracle_gemm.restype = ctypes.c_int
        L.oracle_gemm.argtypes = [
            ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int64, ctypes.c_int, ctypes.c_int,
            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int,
        ]
        for name in ("oracle_round_f16", "oracle_round_bf16", "oracle_decode_f16", "oracle_decode_bf16"):
            getattr(L, name).restype = None
            getattr(L, name).argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64]
        L.oracle_f64_to_f16_rne.restype = ctypes.c_uint16
        L.oracle_f64_to_f16_rne.argtypes = [ctypes.c_double]
        L.oracle_f64_to_bf16_rne.restype = ctypes.c_uint16
        L.oracle_f64_to_bf16_rne.argtypes = [ctypes.c_double]
        L.oracle_f16_to_f64.restype = ctypes.c_double
        L.oracle_f16_to_f64.argtypes = [ctypes.c_uint16]
        L.oracle_bf16_to_f64.restype = ctypes.c_double
        L.oracle_bf16_to_f64.argtypes = [ctypes.c_uint16]
        _lib = L
    return _lib


def _raw(x: np.ndarray, dtype: str) -> np.ndarray:
    """Contiguous raw storage: uint16 bit patterns for 16-bit types, float64 for
    f64, float32 for f32/tf32, uint8 bit patterns for fp8."""
    if dtype == "f64":
        return np.ascontiguousarray(x, dtype=np.float64)
    if dtype in ("f32", "tf32"):
        return np.ascontiguousarray(x, dtype=np.float32)
    if dtype in ("e4m3", "e5m2"):
        return np.ascontiguousarray(np.asarray(x).view(np.uint8) if np.asarray(x).dtype != np.uint8 else x,
                                    dtype=np.uint8)
    if x.dtype == np.float16:
        x = x.view(np.uint16)
    return np.ascontiguousarray(x, dtype=np.uint16)


def default_threads() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


def gemm(m: int, n: int, k: int, batch: int, dtype: str, layout: str, A, B,
         with_scale: bool = False, nthreads: int | None = None):
    """C_ref (and S if ``with_scale``) as float64 arrays of shape [batch, m, n].

    ``A``/``B`` hold the packed operands in ``layout`` (see oracle.c) as
    uint16 bit patterns (f16/bf16; float16 arrays are accepted) or float64.
    """
    a = _raw(np.asarray(A).reshape(-1), dtype)
    b = _raw(np.asarray(B).reshape(-1), dtype)
    assert a.size == batch * m * k and b.size == batch * k * n, "operand sizes"
    C = np.empty((batch, m, n), dtype=np.float64)
    S = np.empty((batch, m, n), dtype=np.float64) if with_scale else None
    rc = lib().oracle_gemm(
        m, n, k, batch, DTYPES[dtype], LAYOUTS[layout],
        a.ctypes.data, b.ctypes.data, C.ctypes.data,
        S.ctypes.data if S is not None else None,
        nthreads or default_threads(),
    )
    if rc != 0:
        raise ValueError("oracle_gemm rejected its arguments")
    return (C, S) if with_scale else C


def round_to(x: np.ndarray, dtype: str) -> np.ndarray:
    """RNE of float64 values to ``dtype``; uint16 bits for 16-bit, float64 for f64."""
    x = np.ascontiguousarray(x, dtype=np.float64).reshape(-1)
    if dtype == "f64":
        return x.copy()
    if dtype in ("f32", "tf32"):  # binary32 output (f4): IEEE cast, RNE
        return x.astype(np.float32)
    out = np.empty(x.size, dtype=np.uint16)
    fn = lib().oracle_round_f16 if dtype == "f16" else lib().oracle_round_bf16
    fn(x.ctypes.data, out.ctypes.data, x.size)
    return out


def decode(bits: np.ndarray, dtype: str) -> np.ndarray:
    """Exact decode of uint16 fp16/bf16 bit patterns, uint8 fp8 bit patterns,
    float32 or float64 to float64."""
    if dtype == "f64":
        return np.asarray(bits, dtype=np.float64).reshape(-1)
    if dtype in ("f32", "tf32"):
        return np.asarray(bits, dtype=np.float32).astype(np.float64).reshape(-1)
    if dtype in ("e4m3", "e5m2"):
        b = np.ascontiguousarray(np.asarray(bits).reshape(-1), dtype=np.uint8)
        out = np.empty(b.size, dtype=np.float64)
        L = lib()
        L.oracle_decode_fp8.restype = None
        L.oracle_decode_fp8.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int]
        L.oracle_decode_fp8(b.ctypes.data, out.ctypes.data, b.size, 1 if dtype == "e5m2" else 0)
        return out
    b = _raw(np.asarray(bits).reshape(-1), dtype)
    out = np.empty(b.size, dtype=np.float64)
    fn = lib().oracle_decode_f16 if dtype == "f16" else lib().oracle_decode_bf16
    fn(b.ctypes.data, out.ctypes.data, b.size)
    return out


def to_row_major(X: np.ndarray, batch: int, R: int, C: int, layout: str) -> np.ndarray:
    """View packed [batch] R-by-C matrices stored in ``layout`` as [batch, R, C]."""
    X = np.asarray(X).reshape(batch, -1)
    if layout == "row":
        return X.reshape(batch, R, C)
    return X.reshape(batch, C, R).transpose(0, 2, 1)


def normalised_error(c_gpu: np.ndarray, c_ref: np.ndarray, s: np.ndarray) -> float:
    """max |C_gpu - C_ref| / S with S = sum_l |a||b| (north_star).  Where S == 0
    the GPU value must be exactly 0, otherwise the error is reported as inf; a
    NaN anywhere in C_gpu is reported as inf.  Pinned by
    tests/test_oracle_checker.py."""
    c_gpu = np.asarray(c_gpu, dtype=np.float64)
    if np.any(np.isnan(c_gpu)):  # a NaN is never within any tolerance (max() would drop it)
        return float("inf")
    diff = np.abs(c_gpu - c_ref)
    zero = s == 0
    if np.any(zero & (c_gpu != 0)):
        return float("inf")
    with np.errstate(divide="ignore", invalid="ignore"):
        e = np.where(zero, 0.0, diff / np.where(zero, 1.0, s))
    return float(e.max()) if e.size else 0.0


def spmm_bsr(m: int, n: int, k: int, batch: int, dtype: str, row_ptr, col_blk, vals, B, blk: int = 16,
             with_scale: bool = False):
    """C_ref = A B for block-sparse A (BSR, Sec. 4.6): A densified
    (absent blocks = 0), then the plain GEMM definition.  Returns [batch, m, n]."""
    L = lib()
    if not hasattr(L, "_spmm_set"):
        L.oracle_spmm_bsr.restype = ctypes.c_int
        L.oracle_spmm_bsr.argtypes = [ctypes.c_int] * 4 + [ctypes.c_int64, ctypes.c_int] + [ctypes.c_void_p] * 3 + \
            [ctypes.c_int] + [ctypes.c_void_p] * 3 + [ctypes.c_int]
        L._spmm_set = True
    rp = np.ascontiguousarray(np.asarray(row_ptr), dtype=np.int32).reshape(-1)
    cb = np.ascontiguousarray(np.asarray(col_blk), dtype=np.int32).reshape(batch, -1)
    max_nnzb = cb.shape[1]
    v = _raw(np.asarray(vals).reshape(-1), dtype)
    b = _raw(np.asarray(B).reshape(-1), dtype)
    C = np.empty((batch, m, n), dtype=np.float64)
    S = np.empty((batch, m, n), dtype=np.float64) if with_scale else None
    rc = L.oracle_spmm_bsr(m, n, k, blk, batch, DTYPES[dtype], rp.ctypes.data, cb.ctypes.data, v.ctypes.data,
                           max_nnzb, b.ctypes.data, C.ctypes.data, S.ctypes.data if S is not None else None, 1)
    if rc != 0:
        raise ValueError(f"oracle_spmm_bsr rejected its arguments ({rc})")
    return (C, S) if with_scale else C


def morton_encode(i: int, j: int) -> int:
    """Z-Morton code of block (row i, column j) (oracle.c, Sec. 4.6)."""
    L = lib()
    L.oracle_morton_encode.restype = ctypes.c_int
    L.oracle_morton_encode.argtypes = [ctypes.c_int, ctypes.c_int]
    return int(L.oracle_morton_encode(i, j))


def morton_decode(z: int) -> tuple:
    L = lib()
    L.oracle_morton_decode.restype = None
    L.oracle_morton_decode.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_int), ctypes.POINTER(ctypes.c_int)]
    a, b = ctypes.c_int(), ctypes.c_int()
    L.oracle_morton_decode(z, ctypes.byref(a), ctypes.byref(b))
    return a.value, b.value


def zmorton_from_blocks(present: np.ndarray, blocks: np.ndarray):
    """Z-Morton block storage of a batch of block-sparse matrices, built from
    the dense block description: present [batch, mb, kb] bool, blocks [batch,
    mb, kb, 16, 16] (any dtype).  Returns (nnzb [batch] int32, zcode [batch,
    max_nnzb] int32 ascending, -1 padded, vals [batch, max_nnzb, 16, 16]) with
    max_nnzb = mb kb.  Plain loops: the oracle's encoder, independent of the
    library's decoder."""
    present = np.asarray(present, dtype=bool)
    batch, mb, kb = present.shape
    nnzb = np.zeros(batch, dtype=np.int32)
    zcode = np.full((batch, mb * kb), -1, dtype=np.int32)
    vals = np.zeros((batch, mb * kb) + blocks.shape[3:], dtype=blocks.dtype)
    for b in range(batch):
        items = sorted((morton_encode(i, j), i, j) for i in range(mb) for j in range(kb) if present[b, i, j])
        nnzb[b] = len(items)
        for s, (z, i, j) in enumerate(items):
            zcode[b, s] = z
            vals[b, s] = blocks[b, i, j]
    return nnzb, zcode, vals


def spmm_zmorton(m: int, n: int, k: int, batch: int, dtype: str, nnzb, zcode, vals, B, blk: int = 16,
                 with_scale: bool = False):
    """C_ref = A B for A in Z-Morton block storage (decoded block by block,
    densified, then the plain GEMM definition).  Returns [batch, m, n]."""
    L = lib()
    L.oracle_spmm_zmorton.restype = ctypes.c_int
    L.oracle_spmm_zmorton.argtypes = [ctypes.c_int] * 4 + [ctypes.c_int64, ctypes.c_int] + [ctypes.c_void_p] * 3 + \
        [ctypes.c_int] + [ctypes.c_void_p] * 3
    nz = np.ascontiguousarray(np.asarray(nnzb), dtype=np.int32).reshape(-1)
    zc = np.ascontiguousarray(np.asarray(zcode), dtype=np.int32).reshape(batch, -1)
    v = _raw(np.asarray(vals).reshape(-1), dtype)
    b = _raw(np.asarray(B).reshape(-1), dtype)
    C = np.empty((batch, m, n), dtype=np.float64)
    S = np.empty((batch, m, n), dtype=np.float64) if with_scale else None
    rc = L.oracle_spmm_zmorton(m, n, k, blk, batch, DTYPES[dtype], nz.ctypes.data, zc.ctypes.data, v.ctypes.data,
                               zc.shape[1], b.ctypes.data, C.ctypes.data, S.ctypes.data if S is not None else None)
    if rc != 0:
        raise ValueError(f"oracle_spmm_zmorton rejected its arguments ({rc})")
    return (C, S) if with_scale else C


def axpby(C_ref: np.ndarray, C_in: np.ndarray, alpha: float, beta: float) -> np.ndarray:
    """alpha * C_ref + beta * C_in in binary64 (the C-update form, DESIGN.md f4)."""
    out = np.ascontiguousarray(C_ref, dtype=np.float64).copy()
    cin = np.ascontiguousarray(C_in, dtype=np.float64).reshape(out.shape)
    L = lib()
    L.oracle_axpby.restype = None
    L.oracle_axpby.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_double, ctypes.c_double, ctypes.c_int64]
    L.oracle_axpby(out.ctypes.data, cin.ctypes.data, alpha, beta, out.size)
    return out
