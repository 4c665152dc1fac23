"""Pointer-array batches (kami_gemm_batched: the TMA tcgen05 kernel over
address-space views) and variable-size batches (PAPER.md L523
"supports various matrix orders in a batch": the LDG-fed tcgen05 kernel),
against the oracle entry by entry."""
import numpy as np
import pytest
import torch

import kami_inputs as ki
import oracle
import paper_conf_sc_wangdltsl25_b200 as kami

pytestmark = pytest.mark.gpu


def _ptr_kernel(dtype, k):
    # k = 8 mod 16 (a K tail inside the MMA's 16-element step) goes to the LDG-fed kernel,
    # which zero-fills it; everything else to the TMA kernel over address-space views
    return f"kami_tc16_vb_kernel<{dtype}>" if k % 16 else f"kami_tc16_1d_kernel<{dtype},ptr>"


def _tol(dtype, k):
    return {"f16": 2.0 ** -11, "bf16": 2.0 ** -8}[dtype] + k * 2.0 ** -23


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("shape", [(16, 16, 16), (32, 32, 32), (64, 64, 64), (48, 80, 40), (256, 256, 8), (192, 64, 256),
                                   (128, 256, 24), (32, 16, 256)])
def test_pointer_array_all_sizes(dtype, shape):
    m, n, k = shape
    batch = 23
    for dist, layout in (("unif", "row"), ("int", "col")):
        A, B = ki.operands(m, n, k, batch, dtype, dist, seed=11)
        dA, dB = A.cuda().view(batch, -1), B.cuda().view(batch, -1)
        dC = torch.zeros(batch, m * n, dtype=A.dtype, device="cuda")
        perm = torch.randperm(batch).tolist()
        pa = torch.tensor([dA[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
        pb = torch.tensor([dB[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
        pc = torch.tensor([dC[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
        kami.gemm_batched(m, n, k, batch, dtype, layout, pa, pb, pc)
        torch.cuda.synchronize()
        # square order 16 goes to the warp-level HMMA 1D (dispatch rule), the rest to the
        # TMA tcgen05 kernel over address-space views
        want = "kami_warp_ca_1d" if (m == n == k and m <= 16) else _ptr_kernel(dtype, k)
        assert kami.last_kernel().startswith(want), kami.last_kernel()
        Cref, S = oracle.gemm(m, n, k, batch, dtype, layout, ki.as_bits(A), ki.as_bits(B), with_scale=True)
        got_bits = oracle.to_row_major(ki.as_bits(dC.cpu()), batch, m, n, layout)
        if dist == "int":
            assert np.array_equal(got_bits, oracle.round_to(Cref, dtype).reshape(batch, m, n))
        else:
            got = oracle.decode(got_bits.reshape(-1), dtype).reshape(batch, m, n)
            assert oracle.normalised_error(got, Cref, S) <= _tol(dtype, k)


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("shape", [(64, 64, 64), (48, 80, 40), (256, 256, 16), (192, 128, 64), (16, 192, 16),
                                   (64, 64, 8), (64, 64, 40), (128, 128, 200), (32, 64, 24),
                                   (192, 32, 16), (144, 16, 32),  # m-tails with U > 1 sub-tiles
                                   (192, 128, 16), (160, 96, 32), (144, 48, 64)])  # multi-atom m-tails
def test_pointer_array_scattered_addresses(dtype, shape):
    """Entries at arbitrary 16-byte-aligned addresses: inside one buffer at offsets that are
    not multiples of the entry size, and in separate allocations more than 2^28 bytes apart
    (both coordinates of the address-space view), pointers shuffled, ragged last unit."""
    m, n, k = shape
    batch = 37
    es = 2
    A, B = ki.operands(m, n, k, batch, dtype, "int", seed=21)
    g = torch.Generator().manual_seed(5)
    # A: one buffer, entry i at a random 16-byte-aligned offset (non-overlapping)
    gaps = (torch.randint(0, 9, (batch,), generator=g) * 16).tolist()
    a_off, pos = [], 0
    for i in range(batch):
        pos += gaps[i]
        a_off.append(pos)
        pos += m * k * es
    bufA = torch.zeros(pos // es + 8, dtype=A.dtype, device="cuda")
    Av = A.view(batch, -1)
    for i in range(batch):
        bufA[a_off[i] // es: a_off[i] // es + m * k] = Av[i].cuda()
    # B and C: separate allocations with a > 2^28-byte spacer between the halves
    Bv = B.view(batch, -1)
    dB = [Bv[i].cuda().clone() for i in range(batch // 2)]
    dC = [torch.zeros(m * n, dtype=A.dtype, device="cuda") for _ in range(batch // 2)]
    spacer = torch.empty(300 << 20, dtype=torch.uint8, device="cuda")
    dB += [Bv[i].cuda().clone() for i in range(batch // 2, batch)]
    dC += [torch.zeros(m * n, dtype=A.dtype, device="cuda") for _ in range(batch // 2, batch)]
    perm = torch.randperm(batch, generator=g).tolist()
    pa = torch.tensor([bufA.data_ptr() + a_off[i] for i in perm], dtype=torch.int64, device="cuda")
    pb = torch.tensor([dB[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
    pc = torch.tensor([dC[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
    kami.gemm_batched(m, n, k, batch, dtype, "row", pa, pb, pc)
    torch.cuda.synchronize()
    assert kami.last_kernel() == _ptr_kernel(dtype, k), kami.last_kernel()
    del spacer
    Cref = oracle.gemm(m, n, k, batch, dtype, "row", ki.as_bits(A), ki.as_bits(B))
    want = oracle.round_to(Cref, dtype).reshape(batch, m, n)
    got = np.stack([ki.as_bits(c.cpu()).reshape(m, n) for c in dC])
    assert np.array_equal(got, want)


@pytest.mark.parametrize("s", [16, 32, 64])
@pytest.mark.parametrize("layout", ["row", "col"])
def test_pointer_array_f64_tma_view(s, layout):
    """FP64 pointer arrays on the DMMA kernel with TMA-fed broadcast operand (address-space
    view of each entry's A): scattered, shuffled entries in two allocations > 2^28 B apart,
    a batch that leaves teams with unequal entry counts; within the FP64 tolerance."""
    batch = 203
    A, B = ki.operands(s, s, s, batch, "f64", "unif", seed=22)
    Av, Bv = A.view(batch, -1), B.view(batch, -1)
    half = batch // 2
    dA = [Av[i].cuda().clone() for i in range(half)]
    dB = [Bv[i].cuda().clone() for i in range(half)]
    dC = [torch.zeros(s * s, dtype=torch.float64, device="cuda") for _ in range(half)]
    spacer = torch.empty(300 << 20, dtype=torch.uint8, device="cuda")
    dA += [Av[i].cuda().clone() for i in range(half, batch)]
    dB += [Bv[i].cuda().clone() for i in range(half, batch)]
    dC += [torch.zeros(s * s, dtype=torch.float64, device="cuda") for _ in range(half, batch)]
    perm = torch.randperm(batch, generator=torch.Generator().manual_seed(3)).tolist()
    pa = torch.tensor([dA[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
    pb = torch.tensor([dB[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
    pc = torch.tensor([dC[i].data_ptr() for i in perm], dtype=torch.int64, device="cuda")
    kami.gemm_batched(s, s, s, batch, "f64", layout, pa, pb, pc)
    torch.cuda.synchronize()
    assert kami.last_kernel() == f"kami_dmma_tma_1d<{s},ptr>", kami.last_kernel()
    del spacer
    Cref, S = oracle.gemm(s, s, s, batch, "f64", layout, A.numpy(), B.numpy(), with_scale=True)
    got = oracle.to_row_major(np.stack([c.cpu().numpy() for c in dC]).reshape(-1), batch, s, s, layout)
    assert oracle.normalised_error(got.reshape(batch, s, s), Cref, S) <= s * 2.0 ** -52


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("layout", ["row", "col"])
def test_vbatched_mixed_orders(dtype, layout):
    rng = np.random.default_rng(12)
    orders = [16, 32, 48, 64, 128, 192, 256]
    batch = 40
    sizes = [(int(rng.choice(orders)), int(rng.choice(orders)), int(rng.choice([8, 16, 24, 64, 136, 256])))
             for _ in range(batch)]
    sizes[0] = (256, 256, 256)
    sizes[1] = (16, 16, 8)
    bufs = []
    for e, (m, n, k) in enumerate(sizes):
        A, B = ki.operands(m, n, k, 1, dtype, "unif", seed=13, entry0=e)
        bufs.append((A, B, A.cuda(), B.cuda(), torch.zeros(m * n, dtype=A.dtype, device="cuda")))
    dm = torch.tensor([s[0] for s in sizes], dtype=torch.int32, device="cuda")
    dn = torch.tensor([s[1] for s in sizes], dtype=torch.int32, device="cuda")
    dk = torch.tensor([s[2] for s in sizes], dtype=torch.int32, device="cuda")
    pa = torch.tensor([b[2].data_ptr() for b in bufs], dtype=torch.int64, device="cuda")
    pb = torch.tensor([b[3].data_ptr() for b in bufs], dtype=torch.int64, device="cuda")
    pc = torch.tensor([b[4].data_ptr() for b in bufs], dtype=torch.int64, device="cuda")
    kami.gemm_vbatched(batch, dm, dn, dk, 256, 256, 256, dtype, layout, pa, pb, pc)
    torch.cuda.synchronize()
    for (m, n, k), (A, B, _, _, C) in zip(sizes, bufs):
        Cref, S = oracle.gemm(m, n, k, 1, dtype, layout, ki.as_bits(A), ki.as_bits(B), with_scale=True)
        got = oracle.decode(oracle.to_row_major(ki.as_bits(C.cpu()), 1, m, n, layout).reshape(-1), dtype)
        assert oracle.normalised_error(got.reshape(1, m, n), Cref, S) <= _tol(dtype, k), (m, n, k)


def test_vbatched_rejects():
    with pytest.raises(kami.KamiError):
        kami.gemm_vbatched(4, 16, 16, 16, 300, 16, 16, "f16", "row", 16, 16, 16)  # max_m off the grid
    with pytest.raises(kami.KamiError):
        kami.gemm_vbatched(4, 16, 16, 16, 64, 64, 64, "tf32", "row", 16, 16, 16)  # tf32: no variable-size path


@pytest.mark.gpu
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_vbatched_many_units_ring_wraps(dtype):
    """Mixed orders at a batch large enough that every persistent CTA runs
    tens of units: the stage ring wraps many times and every TMEM accumulator
    and C staging buffer is reused, with view (TMA) and copy units interleaved."""
    rng = np.random.default_rng(21)
    orders = np.array([16, 32, 48, 64, 128, 192, 256])
    batch = 1200
    sizes = [(int(rng.choice(orders)), int(rng.choice(orders)), int(rng.choice([8, 16, 40, 64, 136, 256])))
             for _ in range(batch)]
    ops = [ki.operands(m, n, k, 1, dtype, "unif", seed=22, entry0=e) for e, (m, n, k) in enumerate(sizes)]
    offA = np.concatenate([[0], np.cumsum([a.numel() for a, _ in ops])])
    offB = np.concatenate([[0], np.cumsum([b.numel() for _, b in ops])])
    offC = np.concatenate([[0], np.cumsum([m * n for m, n, _ in sizes])])
    dA = torch.cat([a for a, _ in ops]).cuda()
    dB = torch.cat([b for _, b in ops]).cuda()
    dC = torch.full((int(offC[-1]),), float("nan"), dtype=dA.dtype, device="cuda")
    es = dA.element_size()
    dm, dn, dk = (torch.tensor([s[i] for s in sizes], dtype=torch.int32, device="cuda") for i in range(3))
    pa = torch.tensor(dA.data_ptr() + offA[:-1] * es, dtype=torch.int64, device="cuda")
    pb = torch.tensor(dB.data_ptr() + offB[:-1] * es, dtype=torch.int64, device="cuda")
    pc = torch.tensor(dC.data_ptr() + offC[:-1] * es, dtype=torch.int64, device="cuda")
    kami.gemm_vbatched(batch, dm, dn, dk, 256, 256, 256, dtype, "row", pa, pb, pc)
    torch.cuda.synchronize()
    assert kami.last_kernel().startswith("kami_tc16_vb_kernel")
    Cb = ki.as_bits(dC.cpu())
    for e, ((m, n, k), (A, B)) in enumerate(zip(sizes, ops)):
        Cref, S = oracle.gemm(m, n, k, 1, dtype, "row", ki.as_bits(A), ki.as_bits(B), with_scale=True)
        got = oracle.decode(Cb[offC[e]:offC[e + 1]], dtype)
        assert oracle.normalised_error(got.reshape(1, m, n), Cref, S) <= _tol(dtype, k), (e, m, n, k)


def _mixed_batch(sizes, dtype, seed):
    ops = [ki.operands(m, n, k, 1, dtype, "unif", seed=seed, entry0=e) for e, (m, n, k) in enumerate(sizes)]
    offA = np.concatenate([[0], np.cumsum([a.numel() for a, _ in ops])])
    offB = np.concatenate([[0], np.cumsum([b.numel() for _, b in ops])])
    offC = np.concatenate([[0], np.cumsum([m * n for m, n, _ in sizes])])
    dA = torch.cat([a for a, _ in ops]).cuda()
    dB = torch.cat([b for _, b in ops]).cuda()
    es = dA.element_size()
    dm, dn, dk = (torch.tensor([s[i] for s in sizes], dtype=torch.int32, device="cuda") for i in range(3))
    pa = torch.tensor(dA.data_ptr() + offA[:-1] * es, dtype=torch.int64, device="cuda")
    pb = torch.tensor(dB.data_ptr() + offB[:-1] * es, dtype=torch.int64, device="cuda")

    def run(keep=(dA, dB)):  # the closure keeps the operands alive
        dC = torch.full((int(offC[-1]),), float("nan"), dtype=dA.dtype, device="cuda")
        pc = torch.tensor(dC.data_ptr() + offC[:-1] * es, dtype=torch.int64, device="cuda")
        kami.gemm_vbatched(len(sizes), dm, dn, dk, 256, 256, 256, dtype, "row", pa, pb, pc)
        torch.cuda.synchronize()
        return dC
    return ops, offC, run


@pytest.mark.gpu
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_vbatched_view_classes(dtype, monkeypatch):
    """Every TMA-view class of tc16_vb.cu (k and n in {16, 32} with 32 / 64-byte
    swizzles, multiples of 64 with 128-byte ones), the copy path beside them
    (k or n 8, 48), and m-tiles of 8..128 live rows (m 8, 72, 200), one entry
    per tile and class-sorted packed tiles (KAMI_VB_SORT): against the oracle,
    and the four (sort, views) modes bit-identical (KAMI_VB_VIEWS=0: the
    cp.async path for every entry)."""
    sizes = [(m, n, k) for m in (8, 72, 128, 200, 256) for n in (16, 32, 48, 64, 192, 256)
             for k in (8, 16, 32, 48, 64, 128, 192, 256)]
    rng = np.random.default_rng(31)
    sizes = [sizes[i] for i in rng.permutation(len(sizes))]
    ops, offC, run = _mixed_batch(sizes, dtype, seed=32)
    outs = {}
    for srt in ("0", "1"):
        for views in ("0", "1"):
            monkeypatch.setenv("KAMI_VB_SORT", srt)
            monkeypatch.setenv("KAMI_VB_VIEWS", views)
            outs[srt + views] = ki.as_bits(run().cpu())
            assert kami.last_kernel().endswith("sorted>") == (srt == "1")
    C0, C1 = outs["00"], outs["11"]
    for key in ("01", "10"):
        assert np.array_equal(outs[key], C0), key
    bad = {0: [], 1: []}
    for e, ((m, n, k), (A, B)) in enumerate(zip(sizes, ops)):
        Cref, S = oracle.gemm(m, n, k, 1, dtype, "row", ki.as_bits(A), ki.as_bits(B), with_scale=True)
        for v, Cv in ((0, C0), (1, C1)):
            got = oracle.decode(Cv[offC[e]:offC[e + 1]], dtype)
            if not oracle.normalised_error(got.reshape(1, m, n), Cref, S) <= _tol(dtype, k):
                bad[v].append((m, n, k))
    assert not bad[0] and not bad[1], bad
    assert np.array_equal(C0, C1)


@pytest.mark.gpu
@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_vbatched_sorted_many_classes(dtype, monkeypatch):
    """Class-sorted mode at scale: 3000 entries over the BF16-sweep orders and
    thin / odd sizes, so buckets hold partial tiles (ng < G), every CTA runs
    many units and packed tiles of every G (1..8) occur; parity with the
    oracle and bit-identity with the unsorted path."""
    rng = np.random.default_rng(41)
    orders = [8, 16, 24, 32, 48, 64, 96, 128, 192, 256]
    sizes = [tuple(int(x) for x in rng.choice(orders, 3)) for _ in range(3000)]
    ops, offC, run = _mixed_batch(sizes, dtype, seed=42)
    monkeypatch.setenv("KAMI_VB_SORT", "1")
    Cs = ki.as_bits(run().cpu())
    assert kami.last_kernel().endswith("sorted>")
    monkeypatch.setenv("KAMI_VB_SORT", "0")
    Cu = ki.as_bits(run().cpu())
    diff = [e for e in range(len(sizes)) if not np.array_equal(Cs[offC[e]:offC[e + 1]], Cu[offC[e]:offC[e + 1]])]
    check = sorted(set(range(0, len(sizes), 7)) | set(diff[:20]))
    bad = []
    for e in check:
        (m, n, k), (A, B) = sizes[e], ops[e]
        Cref, S = oracle.gemm(m, n, k, 1, dtype, "row", ki.as_bits(A), ki.as_bits(B), with_scale=True)
        for name, Cv in (("sorted", Cs), ("unsorted", Cu)):
            got = oracle.decode(Cv[offC[e]:offC[e + 1]], dtype)
            if not oracle.normalised_error(got.reshape(1, m, n), Cref, S) <= _tol(dtype, k):
                bad.append((name, e, m, n, k))
    assert not bad and not diff, (bad[:20], [(e,) + sizes[e] for e in diff[:20]], len(diff))


@pytest.mark.gpu
@pytest.mark.parametrize("layout", ["row", "col"])
@pytest.mark.parametrize("cap", [0, 3])
def test_vbatched_f64_mixed_orders(layout, cap):
    """FP64 variable sizes on the k-sliced DMMA kernel with
    per-entry sizes: every entry against the oracle (FP64 bound), entries of
    the whole FP64 grid (non-square, k not a multiple of 16, n past one
    64-column block, m past one 32-row block), with and without a grid cap
    (steady state: every team walks many units and skips dead ones)."""
    rng = np.random.default_rng(21)
    orders = [8, 16, 24, 40, 64, 72, 128, 136, 200, 256]
    batch = 37
    sizes = [(int(rng.choice(orders)), int(rng.choice(orders)), int(rng.choice(orders))) for _ in range(batch)]
    sizes[0] = (256, 256, 256)
    sizes[1] = (8, 8, 8)
    bufs = []
    for e, (m, n, k) in enumerate(sizes):
        A, B = ki.operands(m, n, k, 1, "f64", "unif", seed=23, entry0=e)
        bufs.append((A, B, A.cuda(), B.cuda(), torch.full((m * n,), float("nan"), dtype=torch.float64, device="cuda")))
    dm = torch.tensor([s[0] for s in sizes], dtype=torch.int32, device="cuda")
    dn = torch.tensor([s[1] for s in sizes], dtype=torch.int32, device="cuda")
    dk = torch.tensor([s[2] for s in sizes], dtype=torch.int32, device="cuda")
    pa = torch.tensor([b[2].data_ptr() for b in bufs], dtype=torch.int64, device="cuda")
    pb = torch.tensor([b[3].data_ptr() for b in bufs], dtype=torch.int64, device="cuda")
    pc = torch.tensor([b[4].data_ptr() for b in bufs], dtype=torch.int64, device="cuda")
    with kami.grid_cap(cap):
        kami.gemm_vbatched(batch, dm, dn, dk, 256, 256, 256, "f64", layout, pa, pb, pc)
    torch.cuda.synchronize()
    assert kami.last_kernel().startswith("kami_dmma_gen"), kami.last_kernel()
    for (m, n, k), (A, B, _, _, C) in zip(sizes, bufs):
        Cref, S = oracle.gemm(m, n, k, 1, "f64", layout, ki.as_bits(A), ki.as_bits(B), with_scale=True)
        got = oracle.decode(oracle.to_row_major(ki.as_bits(C.cpu()), 1, m, n, layout).reshape(-1), "f64")
        assert oracle.normalised_error(got.reshape(1, m, n), Cref, S) <= k * 2.0 ** -52, (m, n, k)
