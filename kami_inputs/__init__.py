"""Seeded synthetic inputs for KAMI batched GEMM -- shared by the oracle side
(tests, cpu baseline) and the CUDA side (tests, bench).

This module holds NO GEMM arithmetic: it only draws operand values.  Every
value is a pure function of (seed, operand, global entry index, element
index) through a counter-based SplitMix64 hash, so

  * entry e is identical whatever the batch chunking or GPU count
    (multi-GPU shards generate only their own entries);
  * the same torch code runs on CPU (oracle inputs) and on CUDA (bench inputs,
    no host->device copy of gigabytes) and yields bit-identical values
    (checked on the GPU by tests/test_gpu_parity.py::test_gpu_generator_matches_cpu).

Value recipes (the paper never states its value
distribution, Sec. 5.1 -- reading R17):
  "unif": uniform in [-1, 1) from 53 random bits, rounded RNE to the dtype;
  "int" : uniform integer in [-R, R]; R chosen (``int_range``) so that
          R^2 k <= 2048 (fp16) / 256 (bf16) / 2^40 (fp64): every product and
          partial sum is an integer exactly representable in FP32 and every
          result exactly representable in the output dtype, so any summation
          order gives the same bits (bit-exact parity, north_star).
"""
from __future__ import annotations

import torch

MASK64 = (1 << 64) - 1
_GOLDEN = 0x9E3779B97F4A7C15
_M1 = 0xBF58476D1CE4E5B9
_M2 = 0x94D049BB133111EB

OPERAND_A = 0
OPERAND_B = 1

TORCH_DTYPES = {"f16": torch.float16, "bf16": torch.bfloat16, "f64": torch.float64, "f32": torch.float32,
                "tf32": torch.float32, "e4m3": torch.float8_e4m3fn, "e5m2": torch.float8_e5m2}
# output (C) storage type of each input type (DESIGN.md f4)
OUT_DTYPE = {"f16": "f16", "bf16": "bf16", "f64": "f64", "tf32": "f32", "e4m3": "f16", "e5m2": "f16"}


def _to_tf32(x: torch.Tensor) -> torch.Tensor:
    """RNE of float64 values to TF32 precision (8-bit exponent, 10-bit
    fraction), stored as float32 -- the values a kind::tf32 MMA reads exactly."""
    u = x.to(torch.float32).view(torch.int32)
    u = (u + 0xFFF + ((u >> 13) & 1)) & ~0x1FFF
    return u.view(torch.float32)


def _s64(u: int) -> int:
    """uint64 constant -> the int64 with the same bits."""
    u &= MASK64
    return u - (1 << 64) if u >= (1 << 63) else u


def _lshr(x: torch.Tensor, s: int) -> torch.Tensor:
    """Logical right shift of int64 bit patterns."""
    return (x >> s) & ((1 << (64 - s)) - 1)


def splitmix64(x: torch.Tensor) -> torch.Tensor:
    """SplitMix64 finaliser of (x + golden) on int64 tensors (two's complement wrap)."""
    z = x + _s64(_GOLDEN)
    z = (z ^ _lshr(z, 30)) * _s64(_M1)
    z = (z ^ _lshr(z, 27)) * _s64(_M2)
    return z ^ _lshr(z, 31)


def splitmix64_py(x: int) -> int:
    """Pure-Python reference of the same function (used to pin the torch version)."""
    z = (x + _GOLDEN) & MASK64
    z = ((z ^ (z >> 30)) * _M1) & MASK64
    z = ((z ^ (z >> 27)) * _M2) & MASK64
    return z ^ (z >> 31)


def int_range(k: int, dtype: str) -> int:
    """Largest R with R^2 * k <= limit (fp16/fp8->fp16 2048, bf16 256, fp64 2^40,
    tf32->fp32 2^24) and R exactly representable in the input type, R >= 1."""
    limit = {"f16": 2048, "bf16": 256, "f64": 1 << 40, "tf32": 1 << 24, "f32": 1 << 24, "e4m3": 2048,
             "e5m2": 2048}[dtype]
    rmax = {"e4m3": 16, "e5m2": 8, "tf32": 2048, "f32": 2048}.get(dtype, 1 << 20)
    r = 1
    while (r + 1) * (r + 1) * k <= limit and r + 1 <= rmax:
        r += 1
    return r


def counters(seed: int, operand: int, entry0: int, n_entries: int, elems: int,
             device="cpu") -> torch.Tensor:
    """int64 counters (seed, operand) * 2^44 + global element index."""
    assert 0 <= seed < (1 << 17) and operand in (0, 1)
    base = ((seed * 2 + operand) << 44) + entry0 * elems
    return torch.arange(n_entries * elems, dtype=torch.int64, device=device) + base


def draw(seed: int, operand: int, entry0: int, n_entries: int, rows: int, cols: int,
         dtype: str, dist: str = "unif", R: int | None = None, device="cpu") -> torch.Tensor:
    """Operand values for entries [entry0, entry0 + n_entries), packed, as a 1-D
    tensor of ``dtype`` with n_entries * rows * cols elements.  The element
    index is the storage index inside the entry, so the values do not depend
    on the layout flag (the layout only says how they are interpreted)."""
    elems = rows * cols
    out = torch.empty(n_entries * elems, dtype=TORCH_DTYPES[dtype], device=device)
    chunk = 1 << 24
    total = n_entries * elems
    base = ((seed * 2 + operand) << 44) + entry0 * elems
    for s in range(0, total, chunk):
        e = min(total, s + chunk)
        z = splitmix64(torch.arange(s, e, dtype=torch.int64, device=device) + base)
        if dist == "unif":
            u = _lshr(z, 11).to(torch.float64) * (2.0 ** -52) - 1.0  # [-1, 1), exact
        elif dist == "int":
            assert R is not None and R >= 1
            u = (torch.remainder(_lshr(z, 33), 2 * R + 1) - R).to(torch.float64)
        else:
            raise ValueError(dist)
        out[s:e] = _to_tf32(u) if dtype == "tf32" else u.to(TORCH_DTYPES[dtype])
    return out


def operands(m: int, n: int, k: int, batch: int, dtype: str, dist: str = "unif",
             seed: int = 0, entry0: int = 0, device="cpu"):
    """(A, B) packed operands for entries [entry0, entry0+batch).  A has m*k
    and B k*n elements per entry (layout-agnostic storage order)."""
    R = int_range(k, dtype) if dist == "int" else None
    A = draw(seed, OPERAND_A, entry0, batch, m, k, dtype, dist, R, device)
    B = draw(seed, OPERAND_B, entry0, batch, k, n, dtype, dist, R, device)
    return A, B


def as_bits(x: torch.Tensor):
    """numpy view usable by the oracle: uint16 bits for 16-bit dtypes, uint8
    bits for fp8, float32 / float64 otherwise."""
    x = x.detach().cpu().contiguous()
    if x.dtype in (torch.float16, torch.bfloat16):
        return x.view(torch.int16).numpy().view("uint16")
    if x.dtype in (torch.float8_e4m3fn, torch.float8_e5m2):
        return x.view(torch.uint8).numpy()
    return x.numpy()


# ------------------------------------------------- block-sparse A (SpMM, f3)
BLK = 16  # dense block order (Sec. 4.6: user-configurable, default 16 x 16)


def _key(seed: int, op: int, idx: torch.Tensor) -> torch.Tensor:
    # a counter space disjoint from draw(): bit 62 set
    assert 0 <= seed < (1 << 13) and 0 <= op < 16
    return splitmix64(idx + ((1 << 62) + (seed << 48) + (op << 44)))


def bsr_operands(m: int, n: int, k: int, batch: int, dtype: str, density: float = 0.5, dist: str = "unif",
                 seed: int = 0, entry0: int = 0, device="cpu"):
    """Batched block-sparse A (BSR, 16 x 16 dense blocks, block-row order --
    the 1D storage of PAPER.md Fig. 7(a)) and dense B.

    Block (i, j) of entry e is present iff a counter-based draw keyed by
    (seed, e, i, j) falls below ``density`` (the paper's "50 % random
    sparsity", Sec. 5.1); its values are keyed by (seed, e, i, j, element) so
    they do not depend on the sparsity of other blocks.  Layout, per entry
    (max_nnzb = (m/16) (k/16), unused tail slots zero / -1):
      row_ptr [batch, m/16 + 1] int32, col_blk [batch, max_nnzb] int32 (sorted
      within a block row), vals [batch, max_nnzb, 16, 16] (row-major blocks),
      B [batch * k * n] packed row-major."""
    assert m % BLK == 0 and k % BLK == 0
    mb, kb = m // BLK, k // BLK
    nb = mb * kb
    ids = torch.arange(batch * nb, dtype=torch.int64, device=device) + entry0 * nb
    z = _key(seed, 0, ids)
    u = _lshr(z, 11).to(torch.float64) * (2.0 ** -53)
    present = (u < density).view(batch, mb, kb)
    counts = present.sum(2, dtype=torch.int32)                       # [batch, mb]
    row_ptr = torch.zeros(batch, mb + 1, dtype=torch.int32, device=device)
    row_ptr[:, 1:] = torch.cumsum(counts, 1)
    # col_blk: present columns of each row, in order, packed per entry
    cols = torch.arange(kb, dtype=torch.int32, device=device).expand(batch, mb, kb)
    order = torch.argsort((~present).to(torch.int8), dim=2, stable=True)  # present first, ascending col
    sorted_cols = torch.gather(cols, 2, order)
    col_blk = torch.full((batch, nb), -1, dtype=torch.int32, device=device)
    vals = torch.zeros(batch, nb, BLK, BLK, dtype=TORCH_DTYPES[dtype], device=device)
    R = int_range(k, dtype) if dist == "int" else None
    # vectorised scatter: slot of block (e, i, j-th present) = row_ptr[e, i] + j
    jpos = torch.arange(kb, device=device).expand(batch, mb, kb)
    valid = jpos < counts.unsqueeze(2)
    slot = (row_ptr[:, :mb].unsqueeze(2) + jpos).masked_select(valid)
    eidx = torch.arange(batch, device=device).view(batch, 1, 1).expand(batch, mb, kb).masked_select(valid)
    bi = torch.arange(mb, device=device).view(1, mb, 1).expand(batch, mb, kb).masked_select(valid)
    bj = sorted_cols.masked_select(valid).to(torch.int64)
    col_blk[eidx, slot.to(torch.int64)] = bj.to(torch.int32)
    # block values keyed by (entry, block row, block col, element)
    bid = ((eidx + entry0) * nb + bi * kb + bj)                       # [nnz_total]
    el = torch.arange(BLK * BLK, dtype=torch.int64, device=device)
    zz = _key(seed, 1, bid.unsqueeze(1) * (BLK * BLK) + el.unsqueeze(0))
    if dist == "unif":
        v = _lshr(zz, 11).to(torch.float64) * (2.0 ** -52) - 1.0
    else:
        v = (torch.remainder(_lshr(zz, 33), 2 * R + 1) - R).to(torch.float64)
    vals[eidx, slot.to(torch.int64)] = v.view(-1, BLK, BLK).to(TORCH_DTYPES[dtype])
    _, B = operands(m, n, k, batch, dtype, dist, seed=seed, entry0=entry0, device=device)
    return row_ptr, col_blk, vals, B


def block_sparse(m: int, k: int, batch: int, dtype: str, density: float = 0.5, dist: str = "unif", seed: int = 0,
                 entry0: int = 0):
    """The block-sparse matrices of bsr_operands as a dense block description
    (no storage format): present [batch, m/16, k/16] bool and blocks [batch,
    m/16, k/16, 16, 16] of ``dtype`` (zero where absent), drawn with the same
    keys, so bsr_operands(...) and any other storage built from these hold
    the same matrices.  CPU only."""
    assert m % BLK == 0 and k % BLK == 0
    mb, kb = m // BLK, k // BLK
    nb = mb * kb
    ids = torch.arange(batch * nb, dtype=torch.int64) + entry0 * nb
    u = _lshr(_key(seed, 0, ids), 11).to(torch.float64) * (2.0 ** -53)
    present = (u < density).view(batch, mb, kb)
    el = torch.arange(BLK * BLK, dtype=torch.int64)
    zz = _key(seed, 1, ids.unsqueeze(1) * (BLK * BLK) + el.unsqueeze(0))
    if dist == "unif":
        v = _lshr(zz, 11).to(torch.float64) * (2.0 ** -52) - 1.0
    else:
        R = int_range(k, dtype)
        v = (torch.remainder(_lshr(zz, 33), 2 * R + 1) - R).to(torch.float64)
    blocks = v.view(batch, mb, kb, BLK, BLK).to(TORCH_DTYPES[dtype])
    blocks[~present] = 0
    return present, blocks
