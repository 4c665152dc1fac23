// tc16_vb.cu -- FP16/BF16 batched GEMM on tcgen05 for POINTER-ARRAY and
// VARIABLE-SIZE batches ("supports various matrix orders in
// a batch") and for SpMM with block-sparse A (f3, Sec. 4.6).
//
// Same KAMI-1D mapping as tc16.cu (4 sub-partition tensor cores, C_i in TMEM,
// B broadcast through shared memory, G = min(128/m, 256/n) same-size entries
// packed block-diagonally per 128-lane MMA tile), but the operands cannot be
// described by one TMA tensor map (every entry has its own pointer, possibly
// its own m, n, k, or a sparse A), so a producer warpgroup performs the
// paper's GMem2Reg + Reg2SMem itself: coalesced 16-byte cp.async (LDGSTS)
// copies of A and B rows straight into the UMMA canonical layouts (128-byte
// swizzle, K-major A, N-major B), zero-filling k beyond the entry's order
// (SpMM: absent 16x16 blocks of A are zero-filled -- A is densified on load,
// only its nonzero blocks cross HBM).  Once a stage's copy group has landed, a
// generic->async proxy fence and an mbarrier arrive hand it to the MMA warp.
//
// Warps: 0-3 producer, 4 MMA issuer + TMEM allocator, 5-12 epilogue (two
// warpgroups on alternate units; tcgen05.ld -> cvt.rn -> padded SMEM staging
// -> coalesced 16-byte st.global).  A unit is G entries x one 128-row m-tile.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <numeric>

#include "kernels.h"
#include "ptx.cuh"
#include "sched.cuh"

namespace kami {
namespace {

constexpr int kVbThreads = 416;  // 13 warps
constexpr int kMaxStages = 8;
constexpr int kMaxAcc = 4;
constexpr uint32_t kAReg = 128 * 128;                 // 128 rows x 64 k (128 B)
constexpr uint32_t kCRow = 128 * 2 + 16;              // padded staging row (128 columns)
constexpr uint32_t kCBuf = 128 * kCRow;               // one warpgroup's C staging (34 KB)
constexpr int kSmemLimit = 232448;

struct alignas(64) VbParams {
  // SpMM with n % 64 == 0: dense B arrives by TMA (4-D (64, k, n/64, batch), box
  // (64, 64, n/64, G), 128-byte swizzle = the N-major atoms the copies build)
  // and the producer warpgroup copies only the sparse A
  CUtensorMap tmB;
  // SpMM: A's nonzero 16 x 16 blocks by TMA, one box per block, from the
  // block array viewed as (16, 16, batch max_nnzb) with the 32-byte swizzle
  CUtensorMap tmA;
  int b_tma;
  uint32_t b_tx;
  int b_wb;  // SpMM: B atom row bytes (2 Wn, Wn = 64, 32 or 16 columns)
  const void* const* A;
  const void* const* B;
  void* const* C;
  const int* dm;  // per-entry sizes (device) or nullptr -> uniform m, n, k
  const int* dn;
  const int* dk;
  int m, n, k;
  int G;       // entries per unit (block-diagonal packing; 1 for mixed sizes)
  int mtiles;  // m-tiles per unit slot
  long long batch, units;
  int stages;
  uint32_t stage_bytes, c_off, bar_off;
  int acc_cols, acc_bufs;
  // SpMM (Sec. 4.6): A block-sparse in BSR with 16 x 16 dense blocks
  // (block-row order, the 1D storage of Fig. 7(a)); B, C dense and strided.
  int bsr, max_nnzb;
  const int* rowptr;
  const int* colblk;
  // Z-Morton block storage (Sec. 4.6, Fig. 7(b); R31):
  // colblk holds each stored block's Morton code (ascending), rowptr the
  // per-entry block counts nnzb[batch]; a block's (row, column) is decoded
  // from its code, so no row pointer walk is needed
  int zorder;
  const uint16_t* vals;
  const uint16_t* Bs;
  uint16_t* Cs;
  int dbg;  // experiments only (env KAMI_VB_DEBUG): 1 = skip C stores, 2 = skip A/B copies
  // strided batches whose m or n is 8 mod 16 (no TMA tile for them; R5):
  // entry e at As + e m k, Bs + e k n, Cs + e m n
  int strided;
  const uint16_t* As;
  // TMA views (non-SpMM modes with one entry per tile): an entry
  // whose k is 16, 32 or a multiple of 64 has its A chunk (Wk = min(k, 64)
  // columns x the tile's live rows) loaded by one TMA box through an
  // address-space view (sched.cuh), and if n is 16, 32 or a multiple of 64
  // too, its B chunk (Wn = min(n, 64) columns x Wk k-rows x n / Wn atoms).
  // Boxes use the 2 Wk- / 2 Wn-byte swizzle, so the MMA descriptors follow the
  // unit's (Wk, Wn) (vb_layout); other entries keep the cp.async path and its
  // 128-byte layouts.  vmap[vidx(k) * 16 + rows / 8 - 1]: A views,
  // vmap[96 + vidx(n) * 6 + vidx(k)]: B views, vidx: 16, 32, 64, 128, 192, 256 -> 0..5
  const CUtensorMap* vmap;
  int vsmall;  // 0: views only for multiples of 64 (A/B experiments, KAMI_VB_VIEWS=2)
  int vprefetch;
  int early;  // release the accumulator before the copy-out (KAMI_VB_EARLY, A/B experiments)
  // Variable-size batches, class-sorted: a pre-pass buckets the
  // entries by (m, n, k) and packs each bucket's entries G(m, n) to a tile like
  // a uniform batch.  Unit u's record is rec[16 u .. 16 u + 15]: slot g < 8 =
  // {A_g, B_g} (entry pointers), slot 8 + g = {C_g, hdr, 0} with hdr = ng |
  // mt << 4 | G << 8 | class << 12 in every slot.  Every role reads a unit
  // with ONE load per thread (no table -> pointer chain), a unit ahead;
  // *nunits = live unit count.
  int sorted;
  const int4* rec;
  const int* nunits;  // prefetch the next unit's maps (KAMI_VB_PREFETCH=0 disables, A/B experiments)
};

// TMA-view class of a size (16, 32 or a multiple of 64 up to 256), else -1
__host__ __device__ __forceinline__ int vidx(int x) {
  return x == 16 ? 0 : x == 32 ? 1 : ((x & 63) == 0 && x <= 256) ? 1 + (x >> 6) : -1;
}
// Shared-memory layout of one unit's stage: A rows of wa bytes (K-major,
// wa-byte swizzle), B atoms of wb-byte rows x kr k-rows (N-major, wb-byte
// swizzle).  The copies build (128, 128, 64); view units (min(k, 64) 2,
// min(n, 64) 2, min(k, 64)).
// SpMM (slab): A as four 4 KB k-step slabs per stage (128 rows x 32 bytes,
// K-major, 32-byte swizzle -- the layout a 16 x 16 block box lands in), B as
// N-major atoms of b_wb-byte rows.
struct VbLayout {
  bool va, vb, slab;
  uint32_t wa, wb, kr;
};
__device__ __forceinline__ VbLayout vb_layout(const VbParams& p, int n, int k) {
  VbLayout L;
  if (p.bsr) {
    L.va = L.vb = false;
    L.slab = true;
    L.wa = 32u;
    L.wb = (uint32_t)p.b_wb;
    L.kr = 64u;
    return L;
  }
  L.slab = false;
  L.va = p.vmap != nullptr && vidx(k) >= (p.vsmall ? 0 : 2);
  L.vb = L.va && vidx(n) >= (p.vsmall ? 0 : 2);
  L.wa = L.va ? (uint32_t)min(k, 64) * 2u : 128u;
  L.wb = L.vb ? (uint32_t)min(n, 64) * 2u : 128u;
  L.kr = L.vb ? (uint32_t)min(k, 64) : 64u;
  return L;
}

__device__ __forceinline__ const uint16_t* entry_B(const VbParams& p, long long e, int k, int n) {
  return (p.bsr || p.strided) ? p.Bs + e * (long long)k * n : reinterpret_cast<const uint16_t*>(p.B[e]);
}
__device__ __forceinline__ uint16_t* entry_C(const VbParams& p, long long e, int m, int n) {
  return (p.bsr || p.strided) ? p.Cs + e * (long long)m * n : reinterpret_cast<uint16_t*>(p.C[e]);
}
__device__ __forceinline__ void entry_dims(const VbParams& p, long long e, int& m, int& n, int& k) {
  if (p.dm) {
    m = __ldg(p.dm + e);
    n = __ldg(p.dn + e);
    k = __ldg(p.dk + e);
  } else {
    m = p.m;
    n = p.n;
    k = p.k;
  }
}
// unit -> first entry, m-tile, live entries, sizes
struct Unit {
  long long e0;
  int mt, ng, m, n, k, G;
};
// Fills U for (entry group grp, m-tile mt).  The size loads (variable-size
// batches) are consumed one unit later by the callers, so their latency hides
// behind the current unit's work.  A unit is live iff mt * 128 < m (mixed
// sizes: an entry may have fewer m-tiles than the widest one).
__device__ __forceinline__ void unit_fill(const VbParams& p, long long grp, int mt, Unit& U) {
  U.mt = mt;
  U.e0 = grp * p.G;
  const long long left = p.batch - U.e0;
  U.ng = left < p.G ? (int)left : p.G;
  U.G = p.G;
  entry_dims(p, U.e0, U.m, U.n, U.k);
}
// class key of a size triple (multiples of 8 in [8, 256]): 5 bits each
__host__ __device__ __forceinline__ int vb_class(int m, int n, int k) {
  return (((m >> 3) - 1) << 10) | (((n >> 3) - 1) << 5) | ((k >> 3) - 1);
}
// entries per tile (block-diagonal packing), capped at the 8-entry tables
__host__ __device__ __forceinline__ int vb_pack(int m, int n) {
  if (m > 128) return 1;
  const int g1 = 128 / m, g2 = 256 / n;
  const int g = g1 < g2 ? g1 : g2;
  return g < 1 ? 1 : (g > 8 ? 8 : g);
}
// sorted mode: slot q of unit u's record.  Loaded a unit (or two) before it
// is decoded (unit_decode): decoding right after the load would stall the
// role for a global-memory round trip per unit (ncu).
__device__ __forceinline__ int4 rec_slot(const VbParams& p, long long u, int q) {
  return __ldg(p.rec + u * 16 + q);
}
__device__ __forceinline__ int vb_hdr(int ng, int mt, int G, int c) { return ng | (mt << 4) | (G << 8) | (c << 12); }
__device__ __forceinline__ void unit_decode(const int hdr, Unit& U) {
  U.e0 = 0;  // (sorted mode: pointers come from the record)
  U.ng = hdr & 15;
  U.mt = (hdr >> 4) & 15;
  U.G = (hdr >> 8) & 15;
  const int c = hdr >> 12;
  U.m = ((c >> 10) + 1) << 3;
  U.n = (((c >> 5) & 31) + 1) << 3;
  U.k = ((c & 31) + 1) << 3;
}
__device__ __forceinline__ const uint16_t* rec_ptr(int lo, int hi) {
  return reinterpret_cast<const uint16_t*>((unsigned long long)(unsigned)lo | ((unsigned long long)(unsigned)hi << 32));
}
// entry index of slot g of a unit (sorted mode: its position in bucket order)
__device__ __forceinline__ long long unit_entry(const VbParams&, const Unit& U, int g) { return U.e0 + g; }

__device__ __forceinline__ void cp_async_wait_n(int n) {
  switch (n) {
    case 0: ptx::cp_async_wait<0>(); break;
    case 1: ptx::cp_async_wait<1>(); break;
    case 2: ptx::cp_async_wait<2>(); break;
    case 3: ptx::cp_async_wait<3>(); break;
    case 4: ptx::cp_async_wait<4>(); break;
    case 5: ptx::cp_async_wait<5>(); break;
    default: ptx::cp_async_wait<6>(); break;
  }
}

// debug trace (KAMI_VB_DEBUG bit 4): clock64 of role events of CTA 0
__device__ long long g_vb_trace[8][1024];
__device__ __forceinline__ void trace(int ev, uint32_t i) {
  if (blockIdx.x == 0 && (threadIdx.x & 31) == 0 && i < 1024) g_vb_trace[ev][i] = clock64();
}

template <bool kBF16>
// 13 warps: the SM sub-partition holding four of them has 16 K registers, so
// 128 per thread is the ceiling (a 150-register build fails to launch)
__global__ void __launch_bounds__(kVbThreads, 1) kami_tc16_vb_kernel
    (const __grid_constant__ VbParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1024-byte aligned base; pointer arithmetic on the __shared__ array keeps
  // the address space, so table reads compile to LDS rather than generic loads
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + p.bar_off);
  uint64_t* empty = full + kMaxStages;
  uint64_t* tfull = empty + kMaxStages;
  uint64_t* tempty = tfull + kMaxAcc;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + kMaxAcc);
  int* blk_tab = reinterpret_cast<int*>(tmem_slot + 4);  // SpMM: [8 tile block rows][16 block cols]
  // per-unit entry pointer tables (loaded once per unit, not once per copy)
  const uint16_t** a_tab = reinterpret_cast<const uint16_t**>(blk_tab + 128);
  const uint16_t** b_tab = a_tab + 8;
  uint16_t** c_tab = reinterpret_cast<uint16_t**>(const_cast<uint16_t**>(b_tab + 8));  // [2 warpgroups][8]
  int* rp_tab = reinterpret_cast<int*>(c_tab + 16);  // (unused since the SpMM row pointers live in lanes)
  // SpMM: the block table is double-buffered by unit parity (blk_tab, blk_tab2)
  // and tagged with the unit, so it needs neither a reset nor a barrier before
  // it is rebuilt: a buffer was last read two units ago, before every producer
  // thread passed the previous unit's publish barrier
  int* blk_tab2 = rp_tab + 32;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < p.stages; ++s) {
      // SpMM: the 128 producer threads' arrivals (after their A boxes'
      // expect_tx and zero stores) + the B TMA's arrive.expect_tx.
      // Otherwise one regular arrival by producer thread 0 per stage (after
      // the TMA issue, or after every copy thread raised the pending count
      // with its cp.async arrival and a named barrier).
      ptx::mbar_init(&full[s], p.bsr ? 128 + (p.b_tma ? 1 : 0) : 4);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < p.acc_bufs; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], 4);
    }
    ptx::fence_mbar_init();
  }
  if (warp == 4) ptx::tmem_alloc(tmem_slot, p.acc_cols * p.acc_bufs);
  // SpMM block tables: tag 0 (never written) -- shared memory keeps an earlier
  // launch's tags otherwise
  for (int i = threadIdx.x; i < 128; i += blockDim.x) blk_tab[i] = blk_tab2[i] = 0;
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  const uint32_t smem_base = ptx::smem_u32(smem);
  const long long units = p.sorted ? (long long)*p.nunits : p.units;

  if (warp < 4) {
    // ------------------------------------------------ producer warpgroup
    // cp.async straight into the swizzled stage buffers; a stage is handed to
    // the MMA warp once its copy group has landed, `lag` stages later, so
    // several stages stream concurrently without register staging.
    const int tid = threadIdx.x;  // 0..127
    RingPos rs;
    uint32_t it = 0;     // stages issued (trace index)
    uint32_t nunit = 0;  // units issued (SpMM table buffer / tag)
    UnitIter ui(blockIdx.x, gridDim.x, p.mtiles);
    // The sizes and entry pointers of a unit are fetched TWO units ahead into
    // alternating register slots: their global-load latency (the pointer and
    // size arrays live in HBM; ~1.5-2k cycles under load, more than one small
    // unit's copy issue -- tools/trace_vb.py mix) hides behind two units of
    // copy issue.  The loop body is instantiated once per slot so a slot whose
    // loads are in flight is never copied.
    // With one entry per unit (G == 1, no SpMM) every thread loads the entry's
    // pointers itself (one broadcast address per warp), so no shared table or
    // table barrier is needed.
    const bool one = p.G == 1 && !p.bsr && !p.sorted;
    // SpMM: the next unit's block structure is fetched ahead too, without the
    // row_ptr -> col_blk dependency: every col_blk slot of the unit's entries
    // (<= 2 per thread: G mb kb <= 256) and every row_ptr value (<= 17)
    const int mbk = p.bsr ? p.m / 16 : 0, rpn = p.zorder ? 1 : mbk + 1;
    struct PSlot {
      Unit U;
      const uint16_t *pa, *pb;
      int cb[2], rp;
    };
    // sorted mode: R = this lane's record slot (lane & 15) of the unit,
    // loaded one fetch earlier: lanes g < ng of every producer warp hold
    // entry g's A and B pointers, lane 8's slot the header
    auto fetch = [&](PSlot& S, const int4 R) {
      S.pa = S.pb = nullptr;
      S.cb[0] = S.cb[1] = -1;
      S.rp = 0;
      if (p.sorted) {
        unit_decode(__shfl_sync(0xffffffffu, R.z, 8), S.U);
        if ((tid & 31) < S.U.ng) {
          S.pa = rec_ptr(R.x, R.y);
          S.pb = rec_ptr(R.z, R.w);
        }
        return;
      }
      unit_fill(p, ui.grp, ui.mt, S.U);
      if (one || (tid & 31) < S.U.ng) {
        const long long e = one ? S.U.e0 : unit_entry(p, S.U, tid & 31);
        S.pa = p.bsr ? nullptr
               : p.strided ? p.As + e * (long long)p.m * p.k
                           : reinterpret_cast<const uint16_t*>(p.A[e]);
        S.pb = (p.bsr || p.strided) ? p.Bs + e * (long long)p.k * p.n : reinterpret_cast<const uint16_t*>(p.B[e]);
      }
      if (p.bsr) {
#pragma unroll
        for (int q = 0; q < 2; ++q) {
          const int idx = tid + 128 * q;
          S.cb[q] = idx < S.U.ng * p.max_nnzb ? __ldg(p.colblk + S.U.e0 * (long long)p.max_nnzb + idx) : -1;
        }
        // every warp holds the unit's <= 32 row pointers in its lanes (shuffled below)
        if ((tid & 31) < S.U.ng * rpn) S.rp = __ldg(p.rowptr + S.U.e0 * (long long)rpn + (tid & 31));
      }
      ui.next();
    };
    auto body = [&](const PSlot& S) {
      const Unit& U = S.U;
      const uint16_t *pa = S.pa, *pb = S.pb;
      const int cb0 = S.cb[0], cb1 = S.cb[1], rpv = S.rp;
      if (U.mt * 128 >= U.m) return;
      const int m = U.m, n = U.n, k = U.k, G = U.G;
      const int kchunks = (k + 63) / 64;
      const int rows = G > 1 ? U.ng * m : min(128, m - U.mt * 128);  // live tile rows
      // ---- all-TMA unit (A and B through views): lane g of every producer
      // warp holds entry g's pointers; warp w issues the boxes of entries
      // g = w, w + 4, ... (the TMA issue of a packed unit is ~50 instructions
      // per entry, one warp's serial issue was the bound for small entries)
      // and makes one of the stage's four arrivals with its own byte count.
      const VbLayout lay = vb_layout(p, n, k);
      if (!p.bsr && lay.va && lay.vb && !(p.dbg & 2)) {
        const int w = tid >> 5, ln = tid & 31;
        const int rows_e = G > 1 ? m : rows;
        const uint32_t a_e = (uint32_t)rows_e * lay.wa, b_e = lay.kr * (uint32_t)n * 2u;
        const int mine = U.ng > w ? (U.ng - w + 3) >> 2 : 0;  // entries this warp issues
        const uint32_t tx = (uint32_t)mine * (a_e + b_e);
        const CUtensorMap* ma = p.vmap + vidx(k) * 16 + (rows_e >> 3) - 1;
        const CUtensorMap* mb = p.vmap + 96 + vidx(n) * 6 + vidx(k);
        const int arow = G > 1 ? 0 : U.mt * 128;
        int alo = 0, ahi = 0, blo = 0, bhi = 0;
        if (one || ln < U.ng) {
          view_coords(pa, alo, ahi);
          view_coords(pb, blo, bhi);
        }
        for (int kc = 0; kc < kchunks; ++kc, rs.next(p.stages), ++it) {
          const uint32_t s = rs.s;
          ptx::mbar_wait(&empty[s], rs.ph ^ 1);
          if (p.dbg & 4) trace(0, it);
          uint8_t* st = smem + s * p.stage_bytes;
          if (ln == 0) ptx::mbar_arrive_expect_tx(&full[s], tx);
#pragma unroll 1
          for (int g = w; g < U.ng; g += 4) {
            const int xa = __shfl_sync(0xffffffffu, alo, g), ya = __shfl_sync(0xffffffffu, ahi, g);
            const int xb = __shfl_sync(0xffffffffu, blo, g), yb = __shfl_sync(0xffffffffu, bhi, g);
            if (ln == 0) {
              ptx::tma_load_4d(st + g * a_e, ma, &full[s], kc * 64, arow, xa, ya);
              ptx::tma_load_5d(st + kAReg + g * b_e, mb, &full[s], 0, kc * 64, 0, xb, yb);
            }
          }
          if (p.dbg & 4) trace(1, it);
        }
        return;
      }
      if (one && !p.bsr && p.vmap) {
        ptx::named_bar_sync(3, 128);  // warp 0 has issued every earlier TMA unit (see above)
      }
      if (!one && !p.bsr) {
        ptx::named_bar_sync(3, 128);  // previous unit's items issued: tables reusable
        if (tid < U.ng) {
          a_tab[tid] = pa;
          b_tab[tid] = pb;
        }
        ptx::named_bar_sync(3, 128);
      }
      // SpMM table entry: tag << 11 | g << 8 | j (tag = unit + 1 mod 2^21; 0 = never written)
      const uint32_t btag = ((nunit & 0x1FFFFFu) + 1u) << 11;
      int* const bt = (nunit & 1u) ? blk_tab2 : blk_tab;
      ++nunit;
      if (p.bsr) {
        // block lookup table of this tile: tile block row -> global block slot.
        // Slot idx = g max_nnzb + j of entry g lies in block row br with
        // rp[br] <= j < rp[br + 1]; only rows [br0, br1) belong to this m-tile.
        const int br0 = U.mt * 8, br1 = min(br0 + 8, mbk);
#pragma unroll
        for (int q = 0; q < 2; ++q) {
          const int idx = tid + 128 * q;
          const int col = q ? cb1 : cb0;
          const int g = idx / p.max_nnzb, j = idx - g * p.max_nnzb;
          // row pointers of entry g from the lanes (every lane shuffles, valid or not)
          const int gl = (col >= 0 && g < U.ng) ? g * rpn : 0;
          int br;
          if (p.zorder) {  // (row, column) from the Morton code: odd bits row, even bits column
            const int cnt = __shfl_sync(0xffffffffu, rpv, gl);
            if (col < 0 || j >= cnt) continue;  // past the entry's nnzb
            const uint32_t z = (uint32_t)col;
            uint32_t r = 0, c = 0;
#pragma unroll
            for (int t = 0; t < 5; ++t) {
              c |= ((z >> (2 * t)) & 1u) << t;
              r |= ((z >> (2 * t + 1)) & 1u) << t;
            }
            br = (int)r;
            if (br < br0 || br >= br1) continue;
            bt[(g * mbk + br - br0) * 16 + (int)c] = (int)(btag | ((uint32_t)g << 8) | (uint32_t)j);  // g < 8, j < 256
            continue;
          }
          const int last = __shfl_sync(0xffffffffu, rpv, gl + mbk);
          // block row of slot j: the last br with rp[br] <= j (binary search
          // over the <= 17 row pointers, shuffled from the lanes)
          br = 0;
#pragma unroll
          for (int step = 8; step > 0; step >>= 1) {
            const int cand = br + step;
            const int v = __shfl_sync(0xffffffffu, rpv, gl + min(cand, mbk - 1));
            if (cand <= mbk - 1 && v <= j) br = cand;
          }
          if (col < 0 || j >= last) continue;  // unused tail slot
          if (br < br0 || br >= br1) continue;
          bt[(g * mbk + br - br0) * 16 + col] = (int)(btag | ((uint32_t)g << 8) | (uint32_t)j);
        }
        ptx::named_bar_sync(3, 128);
      }
      const int nc8 = n / 8;  // 16-byte chunks per B row of one entry
      const int nc8_shift = (nc8 & (nc8 - 1)) == 0 ? __ffs(nc8) - 1 : -1;  // power-of-two fast path
      for (int kc = 0; kc < kchunks; ++kc, rs.next(p.stages), ++it) {
        const uint32_t s = rs.s;
        ptx::mbar_wait(&empty[s], rs.ph ^ 1);
        if (p.dbg & 4) trace(0, it);
        const uint32_t sa = smem_base + s * p.stage_bytes, sb = sa + kAReg;
        if (!(p.dbg & 2)) {
        // Only the K columns the MMA reads in this chunk are written (kpad_c,
        // a multiple of 16; zero-filled past k): for k < 64 the copy issue --
        // the producer's bottleneck (tools/trace_vb.py) -- shrinks with k.
        const int kpad_c = min(64, ((k + 15) & ~15) - kc * 64);
        // A through views, B copied (n off the view classes): thread 0 raises
        // the stage's transaction count and issues one A box per entry
        const bool va = lay.va, vb = false;
        if (va && tid == 0) {
          const int rows_e = G > 1 ? m : rows;
          ptx::mbar_expect_tx(&full[s], (uint32_t)U.ng * (uint32_t)rows_e * lay.wa);
          const CUtensorMap* ma = p.vmap + vidx(k) * 16 + (rows_e >> 3) - 1;
          for (int g = 0; g < U.ng; ++g) {
            int lo, hi;
            view_coords(one ? pa : a_tab[g], lo, hi);
            ptx::tma_load_4d(smem + s * p.stage_bytes + g * rows_e * lay.wa, ma, &full[s], kc * 64,
                             G > 1 ? 0 : U.mt * 128, lo, hi);
          }
        }
        // A: thread = (16-byte chunk j, row r0 + rstep q): the chunks of a row
        // are spread over 2^cshift threads, the swizzle phase (r & 7) is fixed
        // per thread (rstep is a multiple of 8) and addresses advance by
        // constant strides.
        if (p.bsr) {
          // SpMM A (Sec. 4.6): one TMA box per nonzero
          // 16 x 16 block, straight from the block array into its k-step slab
          // (block row ib of the tile at ib * 512 in slab ks); the absent
          // blocks of the tile are zeroed in shared memory -- A is densified
          // on chip, only its nonzero blocks cross HBM.  Thread quad
          // (ib, ks) = tid / 4 owns one block position of the stage.
          const int nib = rows >> 4, nks = kpad_c >> 4;
          const int slot = tid >> 2, part = tid & 3, ib = slot >> 2, ks = slot & 3;
          if (ib < nib && ks < nks) {
            const int v = bt[ib * 16 + kc * 4 + ks];
            const uint32_t off = s * p.stage_bytes + (uint32_t)ks * 4096u + (uint32_t)ib * 512u;
            if (((uint32_t)v & 0xFFFFF800u) == btag) {  // present in this unit's table
              const int idx = (int)((U.e0 + ((v >> 8) & 0x7)) * p.max_nnzb + (v & 0xFF));
              if (part == 0) {
                ptx::mbar_expect_tx(&full[s], 512u);
                ptx::tma_load_3d(smem + off, &p.tmA, &full[s], 0, 0, idx);
              }
            } else {
#pragma unroll
              for (int q = 0; q < 8; ++q) ptx::st_shared_v4(smem_base + off + (uint32_t)(q * 4 + part) * 16u, 0u, 0u, 0u, 0u);
            }
          }
        } else if (!va) {
          const int cpa = kpad_c >> 3;  // live chunks per row: 2, 4, 6 or 8
          const int cshift = cpa <= 2 ? 1 : cpa <= 4 ? 2 : 3;
          const int j = tid & ((1 << cshift) - 1), r0 = tid >> cshift, rstep = 128 >> cshift;
          const int gc = kc * 64 + j * 8;
          const bool col_ok = gc < k;
          const uint32_t dst0 = sa + r0 * 128 + ((j ^ (r0 & 7)) << 4);
          for (int g = 0; g < U.ng && j < cpa; ++g) {
            const int tbase = G > 1 ? g * m : 0;                 // first tile row of the entry
            const int ebase = G > 1 ? 0 : U.mt * 128;            // first entry row in the tile
            const int cnt = G > 1 ? m : rows;                    // entry rows in the tile
            {
              const uint16_t* A = one ? pa : a_tab[g];
              const uint16_t* src = A + (long long)(ebase + r0) * k + gc;
              const long long step = (long long)rstep * k;
              for (int q = r0; q < cnt; q += rstep, src += step)
                ptx::cp_async_16(dst0 + (tbase + q - r0) * 128, col_ok ? src : A, col_ok ? 16 : 0);
            }
          }
        }
        // B: per entry 64 k-rows x n/8 chunks at columns [g n, g n + n) of the
        // N-major tile (atoms of 64 columns x 64 k-rows)
        if (vb) {
          // (view TMA issued above)
        } else if (p.b_tma) {  // one TMA box: G entries x 64 k-rows x n (zero-filled past k / batch)
          if (tid == 0) {
            ptx::mbar_arrive_expect_tx(&full[s], p.b_tx);
            ptx::tma_load_4d(smem + s * p.stage_bytes + kAReg, &p.tmB, &full[s], 0, kc * 64, 0, (int)U.e0);
          }
        } else if (nc8_shift >= 0 && nc8 <= 128) {
          const int j = tid & (nc8 - 1), kr0 = tid >> nc8_shift, kstep = 128 >> nc8_shift;
          for (int g = 0; g < U.ng; ++g) {
            const uint16_t* B = one ? pb : b_tab[g];
            const int cc = g * nc8 + j;  // 16-byte chunk column in the tile
            const uint32_t dcol = sb + (cc >> 3) * 8192;
            const uint16_t* src = B + (long long)(kc * 64 + kr0) * n + j * 8;
            const long long step = (long long)kstep * n;
            for (int kr = kr0; kr < kpad_c; kr += kstep, src += step) {
              const bool ok = kc * 64 + kr < k;
              ptx::cp_async_16(dcol + kr * 128 + (((cc & 7) ^ (kr & 7)) << 4), ok ? src : B, ok ? 16 : 0);
            }
          }
        } else {
          const int per = kpad_c * nc8;
          for (int i = tid; i < U.ng * per; i += 128) {
            const int g = i / per, rem = i - g * per;
            const int kr = rem / nc8, j = rem - kr * nc8;
            const int gk = kc * 64 + kr;
            const bool ok = gk < k;
            const uint16_t* B = one ? pb : b_tab[g];
            const uint16_t* src = ok ? B + (long long)gk * n + j * 8 : B;
            const int cc = g * nc8 + j;
            ptx::cp_async_16(sb + (cc >> 3) * 8192 + kr * 128 + (((cc & 7) ^ (kr & 7)) << 4), src, ok ? 16 : 0);
          }
        }
        }  // dbg & 2
        // full[s] completes when all 128 threads' copies of this stage landed;
        // the MMA warp fences generic->async proxy before reading the stage
        if (p.bsr) {
          // the zero stores (generic proxy) become visible to the tensor core
          // (async proxy) before the arrival releases the stage
          ptx::fence_proxy_async_smem();
          ptx::mbar_arrive(&full[s]);
        } else {
          ptx::cp_async_mbar_arrive(&full[s]);  // pending count raised until the copies land
          ptx::named_bar_sync(3, 128);          // every thread's raise precedes the arrival
          if (tid == 0) ptx::mbar_arrive_cnt(&full[s], 4);  // the four producer warps' share
        }
        if (p.dbg & 4) trace(1, it);
      }
    };
    // the next unit's view maps are prefetched into the TMA descriptor cache
    // while the current unit issues (a cold map costs a global-memory round
    // trip inside the TMA issue)
    auto prefetch_maps = [&](const PSlot& S) {
      const Unit& V = S.U;
      if (tid != 0 || V.mt * 128 >= V.m) return;
      const VbLayout lay = vb_layout(p, V.n, V.k);
      if (!lay.va) return;
      const int rows = min(128, V.m - V.mt * 128);
      ptx::prefetch_tmap(p.vmap + vidx(V.k) * 16 + (rows >> 3) - 1);
      if (lay.vb) ptx::prefetch_tmap(p.vmap + 96 + vidx(V.n) * 6 + vidx(V.k));
    };
    const long long g1 = gridDim.x, g2 = 2 * g1;
    long long u = blockIdx.x;
    if (p.sorted) {
      // class-sorted units: the slots are the raw record slots (4 registers
      // each, loaded two units ahead), decoded right before the unit's body
      // (PSlot state two units deep spilled, and a spilled load result is a
      // stall on that load)
      int4 R0 = make_int4(0, 0, 0, 0), R1 = R0;
      if (u < units) R0 = rec_slot(p, u, tid & 15);
      if (u + g1 < units) R1 = rec_slot(p, u + g1, tid & 15);
      while (u < units) {
        {
          const int4 c = R0;
          if (u + g2 < units) R0 = rec_slot(p, u + g2, tid & 15);
          PSlot S;
          fetch(S, c);
          body(S);
        }
        if ((u += g1) >= units) break;
        {
          const int4 c = R1;
          if (u + g2 < units) R1 = rec_slot(p, u + g2, tid & 15);
          PSlot S;
          fetch(S, c);
          body(S);
        }
        u += g1;
      }
    } else {
      // slots S0 / S1 = units u and u + g1 (pointers in flight or landed)
      const int4 z = make_int4(0, 0, 0, 0);
      PSlot S0, S1;
      if (u < units) fetch(S0, z);
      if (u + g1 < units) fetch(S1, z);
      while (u < units) {
        {
          const PSlot c = S0;
          if (u + g2 < units) fetch(S0, z);
          if (p.vprefetch && p.vmap && u + g1 < units) prefetch_maps(S1);
          body(c);
        }
        if ((u += g1) >= units) break;
        {
          const PSlot c = S1;
          if (u + g2 < units) fetch(S1, z);
          if (p.vprefetch && p.vmap && u + g1 < units) prefetch_maps(S0);
          body(c);
        }
        u += g1;
      }
    }
    ptx::cp_async_wait<0>();  // nothing may be in flight when the CTA exits
  } else if (warp == 4) {
    // ------------------------------------------------------------- MMA
    RingPos rs, ra;
    uint32_t it = 0, acc_it = 0;  // trace indices
    UnitIter ui(blockIdx.x, gridDim.x, p.mtiles);
    Unit Un;
    // sorted mode: hn = the next unit's header, decoded one unit later
    int hn = 0;
    if (!p.sorted && (long long)blockIdx.x < units) unit_fill(p, ui.grp, ui.mt, Un);
    if (p.sorted && (long long)blockIdx.x < units) hn = __ldg(&p.rec[(long long)blockIdx.x * 16 + 8].z);
    for (long long u = blockIdx.x; u < units; u += gridDim.x) {
      if (p.sorted) unit_decode(hn, Un);
      const Unit U = Un;
      ui.next();
      if (u + gridDim.x < units) {
        if (p.sorted) hn = __ldg(&p.rec[(u + gridDim.x) * 16 + 8].z);
        else unit_fill(p, ui.grp, ui.mt, Un);
      }
      if (U.mt * 128 >= U.m) continue;
      const uint32_t a = ra.s;
      ptx::mbar_wait(&tempty[a], ra.ph ^ 1);
      if (p.dbg & 4) trace(6, acc_it);
      ptx::tc_fence_after();
      const uint32_t d_tmem = tmem_base + a * p.acc_cols;
      // N of the MMA: the tile's G n live columns rounded up to the M = 128 granule of
      // 16 (n = 8 mod 16: the pad columns' products are never stored)
      const uint32_t idesc = ptx::make_idesc_f16(kBF16 ? 1 : 0, 128, (U.G * U.n + 15) & ~15, 0, 1);
      const int kpad = (U.k + 15) / 16 * 16;
      const int kchunks = (U.k + 63) / 64;
      const VbLayout lay = vb_layout(p, U.n, U.k);
      for (int kc = 0; kc < kchunks; ++kc, rs.next(p.stages), ++it) {
        const uint32_t s = rs.s;
        ptx::mbar_wait(&full[s], rs.ph);
        if (p.dbg & 4) trace(2, it);
        ptx::fence_proxy_async_smem();  // cp.async (generic proxy) writes -> tensor-core reads
        ptx::tc_fence_after();
        if (lane == 0) {
          const uint32_t sa = smem_base + s * p.stage_bytes, sb = sa + kAReg;
          const int nsteps = (kpad - kc * 64) >= 64 ? 4 : (kpad - kc * 64) / 16;
          for (int ks = 0; ks < nsteps; ++ks) {
            // A: K-major, a K step is 32 bytes along the row; B: N-major, a K
            // step is 16 k-rows, atoms kr k-rows apart
            const uint64_t adesc =
                lay.slab ? ptx::make_smem_desc(sa + ks * 4096, 16, 256, ptx::umma_layout_code(32))
                         : ptx::make_smem_desc(sa + ks * 32, 16, 8 * lay.wa, ptx::umma_layout_code(lay.wa));
            const uint64_t bdesc = ptx::make_smem_desc(sb + ks * 16 * lay.wb, lay.kr * lay.wb, 8 * lay.wb,
                                                       ptx::umma_layout_code(lay.wb));
            ptx::umma_f16_ss(d_tmem, adesc, bdesc, idesc, (kc | ks) != 0);
          }
          ptx::umma_commit(&empty[s]);
        }
        __syncwarp();
      }
      if (lane == 0) ptx::umma_commit(&tfull[a]);
      if (p.dbg & 4) trace(3, acc_it);
      __syncwarp();
      ra.next(p.acc_bufs);
      ++acc_it;
    }
  } else {
    // -------------------------------------------------------- epilogue
    const int wg = (warp - 5) >> 2;
    const int sp = warp & 3;
    const int L = sp * 32 + lane;
    const uint32_t cst = smem_base + p.c_off + wg * kCBuf;
    RingPos ra;
    uint32_t live = 0;  // live units seen (the warpgroups take alternate live units)
    UnitIter ui(blockIdx.x, gridDim.x, p.mtiles);
    Unit Un;
    uint16_t* pc_n = nullptr;
    // sorted mode: Rn = this thread's record slot 8 + (L & 7) of the next
    // unit ({C pointer, header}), decoded one unit later
    int4 Rn = make_int4(0, 0, 0, 0);
    auto fetch = [&]() {
      if (p.sorted) {
        // the header from lane 0's slot 8 (slots 8 + g, g >= ng, are never written)
        unit_decode(__shfl_sync(0xffffffffu, Rn.z, 0), Un);
        if (L < Un.ng) pc_n = const_cast<uint16_t*>(rec_ptr(Rn.x, Rn.y));
      } else {
        unit_fill(p, ui.grp, ui.mt, Un);
        if (L < Un.ng) pc_n = entry_C(p, unit_entry(p, Un, L), Un.m, Un.n);
      }
    };
    if ((long long)blockIdx.x < units) {
      if (p.sorted) Rn = rec_slot(p, blockIdx.x, 8 + (L & 7));
      fetch();
      if (p.sorted && (long long)blockIdx.x + gridDim.x < units) Rn = rec_slot(p, blockIdx.x + gridDim.x, 8 + (L & 7));
    }
    for (long long u = blockIdx.x; u < units; u += gridDim.x) {
      const Unit U = Un;
      uint16_t* const pc = pc_n;
      ui.next();
      if (u + gridDim.x < units) {
        fetch();
        if (p.sorted && u + 2ll * gridDim.x < units) Rn = rec_slot(p, u + 2ll * gridDim.x, 8 + (L & 7));
      }
      if (U.mt * 128 >= U.m) continue;
      const uint32_t a = ra.s;
      const uint32_t aph = ra.ph;
      ra.next(p.acc_bufs);
      const bool mine = (int)(live & 1) == wg;
      ++live;
      if (!mine) continue;
      const int m = U.m, n = U.n, G = U.G;
      const int rows = G > 1 ? U.ng * m : min(128, m - U.mt * 128);
      // lanes -> (entry g, row); the warp's lanes may span several entries
      const int g = G > 1 ? L / m : 0;
      const bool row_ok = L < rows;
      const int glo = G > 1 ? (sp * 32) / m : 0;
      const int ghi = G > 1 ? min(U.ng - 1, (sp * 32 + 31) / m) : 0;
      const bool warp_live = sp * 32 < rows;
      if (L < U.ng) c_tab[wg * 8 + L] = pc;  // read after the staging barrier
      ptx::mbar_wait(&tfull[a], aph);
      if (p.dbg & 4) trace(4, live);
      ptx::tc_fence_after();
      const uint32_t t_row = tmem_base + (uint32_t(sp * 32) << 16) + a * p.acc_cols;
      for (int h0 = 0; h0 < n; h0 += 128) {
        const int hw = min(128, n - h0);
        if (warp_live) {
          for (int gg = glo; gg <= ghi; ++gg) {  // warp-uniform
            for (int c0 = 0; c0 < hw; c0 += 32) {
              uint32_t v[32];
              const uint32_t col = (uint32_t)(gg * n + h0 + c0);
              const int rem = hw - c0;  // multiple of 8
              if (rem >= 32) {
                ptx::tmem_ld_32x32b_x32(t_row + col, v);
              } else if (rem >= 16) {
                ptx::tmem_ld_32x32b_x16(t_row + col, *reinterpret_cast<uint32_t(*)[16]>(&v[0]));
                if (rem >= 24) ptx::tmem_ld_32x32b_x8(t_row + col + 16, &v[16]);
              } else {
                ptx::tmem_ld_32x32b_x8(t_row + col, &v[0]);
              }
              ptx::tmem_wait_ld();
              if (row_ok && g == gg) {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                  if (c0 + 8 * q < hw) {
                    uint32_t w0, w1, w2, w3;
                    if (kBF16) {
                      w0 = ptx::pack_bf16x2(__uint_as_float(v[8 * q + 0]), __uint_as_float(v[8 * q + 1]));
                      w1 = ptx::pack_bf16x2(__uint_as_float(v[8 * q + 2]), __uint_as_float(v[8 * q + 3]));
                      w2 = ptx::pack_bf16x2(__uint_as_float(v[8 * q + 4]), __uint_as_float(v[8 * q + 5]));
                      w3 = ptx::pack_bf16x2(__uint_as_float(v[8 * q + 6]), __uint_as_float(v[8 * q + 7]));
                    } else {
                      w0 = ptx::pack_f16x2(__uint_as_float(v[8 * q + 0]), __uint_as_float(v[8 * q + 1]));
                      w1 = ptx::pack_f16x2(__uint_as_float(v[8 * q + 2]), __uint_as_float(v[8 * q + 3]));
                      w2 = ptx::pack_f16x2(__uint_as_float(v[8 * q + 4]), __uint_as_float(v[8 * q + 5]));
                      w3 = ptx::pack_f16x2(__uint_as_float(v[8 * q + 6]), __uint_as_float(v[8 * q + 7]));
                    }
                    ptx::st_shared_v4(cst + L * kCRow + (c0 + 8 * q) * 2, w0, w1, w2, w3);
                  }
                }
              }
            }
          }
        }
        if (p.early && h0 + 128 >= n) {
          // every accumulator column is in registers / staging: release the
          // accumulator before the copy-out, so the MMA of the unit after next
          // overlaps this unit's stores
          ptx::tc_fence_before();
          __syncwarp();
          if (lane == 0) ptx::mbar_arrive(&tempty[a]);
        }
        ptx::named_bar_sync(1 + wg, 128);
        // copy-out: chunk index i -> (tile row i / cpr, 16-byte chunk i % cpr)
        const int cpr = hw / 8;
        const int cpr_shift = (cpr & (cpr - 1)) == 0 ? __ffs(cpr) - 1 : -1;
        const uint32_t inv_m = (65536u + m - 1) / m;  // r / m == (r inv_m) >> 16 for r < 256
        if (cpr_shift >= 0 && !(p.dbg & 1)) {
          // power-of-two chunks per row (hw = 8 .. 128): this thread's chunk
          // column is fixed and its rows step by 128 / cpr, so shared and
          // global addresses advance by constants -- ~4 instructions per 16
          // bytes instead of ~12 (the general loop below bound the
          // write-heavy classes, ncu r2)
          const int c = L & (cpr - 1), rstep = 128 >> cpr_shift;
          int r = L >> cpr_shift;
          uint32_t sa = cst + (uint32_t)r * kCRow + (uint32_t)c * 16u;
          const uint32_t sstep = (uint32_t)rstep * kCRow;
          if (G == 1) {
            uint16_t* ga = c_tab[wg * 8] + (long long)(U.mt * 128 + r) * n + h0 + c * 8;
            const long long gstep = (long long)rstep * n;
#pragma unroll 4
            for (; r < rows; r += rstep, sa += sstep, ga += gstep) {
              uint32_t x0, x1, x2, x3;
              ptx::ld_shared_v4(sa, x0, x1, x2, x3);
              ptx::st_global_v4(ga, make_uint4(x0, x1, x2, x3));
            }
          } else {
#pragma unroll 2
            for (; r < rows; r += rstep, sa += sstep) {
              const int ge = (int)(((uint32_t)r * inv_m) >> 16), er = r - ge * m;
              uint32_t x0, x1, x2, x3;
              ptx::ld_shared_v4(sa, x0, x1, x2, x3);
              ptx::st_global_v4(c_tab[wg * 8 + ge] + (long long)er * n + h0 + c * 8, make_uint4(x0, x1, x2, x3));
            }
          }
          ptx::named_bar_sync(1 + wg, 128);  // staging buffer reusable
          continue;
        }
        for (int i = L; i < rows * cpr; i += 128) {
          const int r = cpr_shift >= 0 ? i >> cpr_shift : i / cpr, c = i - r * cpr;
          const int ge = G > 1 ? (int)(((uint32_t)r * inv_m) >> 16) : 0;
          const int er = G > 1 ? r - ge * m : U.mt * 128 + r;
          if (p.dbg & 1) continue;
          uint32_t x0, x1, x2, x3;
          ptx::ld_shared_v4(cst + r * kCRow + c * 16, x0, x1, x2, x3);
          ptx::st_global_v4(c_tab[wg * 8 + ge] + (long long)er * n + h0 + c * 8, make_uint4(x0, x1, x2, x3));
        }
        ptx::named_bar_sync(1 + wg, 128);  // staging buffer reusable
      }
      if (!p.early) {
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(&tempty[a]);
      }
      if (p.dbg & 4) trace(5, live);
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 4) ptx::tmem_dealloc(tmem_base, p.acc_cols * p.acc_bufs);
}

// The TMA view maps of the non-SpMM modes: they depend only on the shape class,
// not on any pointer (the view's base is kViewBase), so one table per device
// serves every launch.  A (k, rows): dims (k, 256, 2^24, 2^20), box (Wk, rows,
// 1, 1); B (n, k): dims (Wn, k, n / Wn, 2^24, 2^20), box (Wn, Wk, n / Wn, 1, 1);
// Wk = min(k, 64), Wn = min(n, 64), swizzle 2 Wk / 2 Wn bytes.
// Built on the first launch that is not being captured into a CUDA graph (the
// allocation and copy are not capturable); until then the copies are used.
const CUtensorMap* vb_view_maps(cudaStream_t stream) {
  static std::mutex mu;
  static const CUtensorMap* table[64] = {};
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return nullptr;
  std::lock_guard<std::mutex> lock(mu);
  if (table[dev]) return table[dev];
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  if (cudaStreamIsCapturing(stream, &cs) != cudaSuccess || cs != cudaStreamCaptureStatusNone) return nullptr;
  PFN_encodeTiled enc = get_encode_tiled();
  if (!enc) return nullptr;
  constexpr int kMaps = 96 + 36;
  CUtensorMap h[kMaps];
  memset(h, 0, sizeof(h));
  void* const vbase = reinterpret_cast<void*>(kViewBase);
  const cuuint64_t vlo = 1ull << 24, vhi = 1ull << 20, vstride_hi = 1ull << 28;
  const int cls[6] = {16, 32, 64, 128, 192, 256};
  auto swz = [](int bytes) {
    return bytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B;
  };
  for (int ki = 0; ki < 6; ++ki)
    for (int r = 8; r <= 128; r += 8) {
      const int k = cls[ki], wk = k < 64 ? k : 64;
      cuuint64_t dims[4] = {(cuuint64_t)k, 256, vlo, vhi};
      cuuint64_t strides[3] = {(cuuint64_t)k * 2, 16, vstride_hi};
      cuuint32_t box[4] = {(cuuint32_t)wk, (cuuint32_t)r, 1, 1};
      cuuint32_t es[4] = {1, 1, 1, 1};
      if (enc(&h[ki * 16 + r / 8 - 1], CU_TENSOR_MAP_DATA_TYPE_UINT16, 4, vbase, dims, strides, box, es,
              CU_TENSOR_MAP_INTERLEAVE_NONE, swz(wk * 2), CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
        return nullptr;
    }
  for (int ni = 0; ni < 6; ++ni)
    for (int ki = 0; ki < 6; ++ki) {
      const int n = cls[ni], k = cls[ki], wn = n < 64 ? n : 64, wk = k < 64 ? k : 64;
      cuuint64_t dims[5] = {(cuuint64_t)wn, (cuuint64_t)k, (cuuint64_t)(n / wn), vlo, vhi};
      cuuint64_t strides[4] = {(cuuint64_t)n * 2, (cuuint64_t)wn * 2, 16, vstride_hi};
      cuuint32_t box[5] = {(cuuint32_t)wn, (cuuint32_t)wk, (cuuint32_t)(n / wn), 1, 1};
      cuuint32_t es[5] = {1, 1, 1, 1, 1};
      if (enc(&h[96 + ni * 6 + ki], CU_TENSOR_MAP_DATA_TYPE_UINT16, 5, vbase, dims, strides, box, es,
              CU_TENSOR_MAP_INTERLEAVE_NONE, swz(wn * 2), CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
        return nullptr;
    }
  void* d = nullptr;
  if (cudaMalloc(&d, sizeof(h)) != cudaSuccess) return nullptr;
  if (cudaMemcpy(d, h, sizeof(h), cudaMemcpyHostToDevice) != cudaSuccess) {
    cudaFree(d);
    return nullptr;
  }
  table[dev] = static_cast<const CUtensorMap*>(d);  // process lifetime
  return table[dev];
}

// ---------------------------------------------------------------------------
// Class-sorted variable-size batches (pre-pass).  Entries are
// bucketed by their exact (m, n, k) (32^3 classes), each bucket is packed
// G(m, n) entries to a tile, and the unit table lists every bucket's tiles.
// Three small kernels on the caller's stream; positions inside a bucket come
// from atomics, so which entries share a tile varies from run to run, but an
// entry's result does not (block-diagonal tiles: an entry's rows and columns
// meet only its own operands, in the same K order).
constexpr int kClasses = 32 * 32 * 32;

// The pre-pass workspace comes from the library's own stream-ordered pool,
// which keeps its memory between calls (release threshold: unlimited), so a
// call does not re-map pages the way the default pool does after every
// synchronisation; the allocation is graph-capturable.
cudaMemPool_t vb_pool() {
  static std::mutex mu;
  static cudaMemPool_t pools[64] = {};
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return nullptr;
  std::lock_guard<std::mutex> lock(mu);
  if (!pools[dev]) {
    cudaMemPoolProps props;
    memset(&props, 0, sizeof(props));
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    cudaMemPool_t pool = nullptr;
    if (cudaMemPoolCreate(&pool, &props) != cudaSuccess) return nullptr;
    uint64_t thr = ~0ull;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    pools[dev] = pool;
  }
  return pools[dev];
}
// sizes on the kami.h grid (multiples of 8 in [8, 256]); an entry off the grid
// is skipped (not computed) rather than indexing past the class tables
__device__ __forceinline__ bool vb_on_grid(int m, int n, int k) {
  return ((m | n | k) & 7) == 0 && m >= 8 && n >= 8 && k >= 8 && m <= 256 && n <= 256 && k <= 256;
}

__global__ void vb_class_hist(long long batch, const int* dm, const int* dn, const int* dk, int* hist) {
  for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < batch;
       e += (long long)gridDim.x * blockDim.x) {
    const int m = __ldg(dm + e), n = __ldg(dn + e), k = __ldg(dk + e);
    const bool ok = vb_on_grid(m, n, k);
    const int c = ok ? vb_class(m, n, k) : -1;
    // warp-aggregated: one atomic per distinct class in the warp (a uniform
    // batch would otherwise serialise every entry on one address)
    const unsigned act = __activemask();
    const unsigned peers = __match_any_sync(act, c);
    if (ok && (threadIdx.x & 31) == __ffs(peers) - 1) atomicAdd(hist + c, __popc(peers));
  }
}

// one block of 1024 threads, 32 classes each: exclusive scans of the bucket
// sizes (entry offsets) and of the bucket unit counts (unit offsets).  Each
// array is staged in shared memory (coalesced, 128 KB) and every thread scans
// its 32 consecutive classes there.
__device__ __forceinline__ int vb_class_units(int c, int cnt) {
  if (cnt == 0) return 0;  // most classes are empty: no divisions for them
  const int m = ((c >> 10) + 1) << 3, n = (((c >> 5) & 31) + 1) << 3;
  const int G = vb_pack(m, n);
  return (cnt + G - 1) / G * ((m + 127) >> 7);
}
__global__ void __launch_bounds__(1024) vb_class_scan(const int* hist, int* eoff, int* uoff, int* nunits) {
  extern __shared__ int sh[];  // [kClasses]
  __shared__ int ws_e[32], ws_u[32];
  const int t = threadIdx.x, c0 = t * 32;
  for (int c = t; c < kClasses; c += 1024) sh[c] = __ldg(hist + c);
  __syncthreads();
  int se = 0, su = 0;
  for (int i = 0; i < 32; ++i) {
    const int c = c0 + ((i + t) & 31);  // rotated: no bank conflicts
    const int cnt = sh[c];
    se += cnt;
    su += vb_class_units(c, cnt);
  }
  int ie = se, iu = su;
  for (int o = 1; o < 32; o <<= 1) {
    const int xe = __shfl_up_sync(0xffffffffu, ie, o), xu = __shfl_up_sync(0xffffffffu, iu, o);
    if ((t & 31) >= o) {
      ie += xe;
      iu += xu;
    }
  }
  if ((t & 31) == 31) {
    ws_e[t >> 5] = ie;
    ws_u[t >> 5] = iu;
  }
  __syncthreads();
  if (t < 32) {
    int ve = ws_e[t], vu = ws_u[t];
    for (int o = 1; o < 32; o <<= 1) {
      const int xe = __shfl_up_sync(0xffffffffu, ve, o), xu = __shfl_up_sync(0xffffffffu, vu, o);
      if (t >= o) {
        ve += xe;
        vu += xu;
      }
    }
    ws_e[t] = ve;
    ws_u[t] = vu;
  }
  __syncthreads();
  const int be0 = ie - se + ((t >> 5) ? ws_e[(t >> 5) - 1] : 0);
  const int bu0 = iu - su + ((t >> 5) ? ws_u[(t >> 5) - 1] : 0);
  if (t == 1023) *nunits = bu0 + su;
  for (int pass = 0; pass < 2; ++pass) {
    __syncthreads();
    for (int c = t; c < kClasses; c += 1024) {
      const int cnt = __ldg(hist + c);
      sh[c] = pass ? vb_class_units(c, cnt) : cnt;
    }
    __syncthreads();
    int b = pass ? bu0 : be0;
    for (int i = 0; i < 32; ++i) {  // in place: the exclusive offsets
      const int v = sh[c0 + i];
      sh[c0 + i] = b;
      b += v;
    }
    __syncthreads();
    int* out = pass ? uoff : eoff;
    for (int c = t; c < kClasses; c += 1024) out[c] = sh[c];
    __syncthreads();
  }
}

// scatter: entry -> its bucket position; each entry writes its pointers into
// the record slots of its unit(s) (one per m-tile)
__global__ void vb_class_scatter(long long batch, const int* dm, const int* dn, const int* dk, const int* hist,
                                 const int* uoff, int* cursor, const void* const* A, const void* const* B,
                                 void* const* C, int4* rec) {
  for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < batch;
       e += (long long)gridDim.x * blockDim.x) {
    const int m = __ldg(dm + e), n = __ldg(dn + e), k = __ldg(dk + e);
    const bool ok = vb_on_grid(m, n, k);
    const int c = ok ? vb_class(m, n, k) : -1;
    const unsigned act = __activemask();
    const unsigned peers = __match_any_sync(act, c);
    const int lane = threadIdx.x & 31, leader = __ffs(peers) - 1;
    int base = 0;
    if (ok && lane == leader) base = atomicAdd(cursor + c, __popc(peers));
    base = __shfl_sync(peers, base, leader);
    if (!ok) continue;
    const int pos = base + __popc(peers & ((1u << lane) - 1u));
    const int G = vb_pack(m, n), cnt = hist[c], tile = pos / G, g = pos - tile * G;
    const int ng = cnt - tile * G < G ? cnt - tile * G : G, mt_n = (m + 127) >> 7;
    const unsigned long long a = (unsigned long long)A[e], b = (unsigned long long)B[e], cc = (unsigned long long)C[e];
    for (int mt = 0; mt < mt_n; ++mt) {
      int4* r = rec + (long long)(uoff[c] + tile * mt_n + mt) * 16;
      r[g] = make_int4((int)(a & 0xffffffffu), (int)(a >> 32), (int)(b & 0xffffffffu), (int)(b >> 32));
      r[8 + g] = make_int4((int)(cc & 0xffffffffu), (int)(cc >> 32), vb_hdr(ng, mt, G, c), 0);
    }
  }
}

int pow2_ceil(int x) {
  int q = 32;
  while (q < x) q <<= 1;
  return q;
}

// n_max: widest B tile (columns) a unit can need; G entries per unit
kami_status_t vb_launch(VbParams& p, bool bf16, int n_max, int max_m, cudaStream_t stream) {
  // widest tile: G n columns (sorted mode: any class, G n <= min(8 n_max, 256))
  const int N = p.G * n_max < 256 ? p.G * n_max : 256;
  const uint32_t b_region = (uint32_t)((N + 63) / 64) * 8192;
  p.stage_bytes = kAReg + b_region;
  p.acc_cols = pow2_ceil(N);
  p.acc_bufs = 512 / p.acc_cols < kMaxAcc ? 512 / p.acc_cols : kMaxAcc;
  const int budget = kSmemLimit - 1024 /*align*/ - 2048 /*barriers, tables*/ - 2 * (int)kCBuf;
  int st = budget / (int)p.stage_bytes;
  if (st > kMaxStages) st = kMaxStages;
  if (st < 2) return KAMI_ERROR_NOT_SUPPORTED;
  p.stages = st;
  p.c_off = st * p.stage_bytes;
  p.bar_off = p.c_off + 2 * kCBuf;
  p.mtiles = (p.G > 1 && !p.sorted) ? 1 : (max_m + 127) / 128;
  // (sorted mode: an upper bound; the kernel reads the live count)
  p.units = p.sorted ? p.batch * p.mtiles : ((p.batch + p.G - 1) / p.G) * p.mtiles;
  {
    const char* d = getenv("KAMI_VB_DEBUG");
    p.dbg = d ? atoi(d) : 0;
    const char* e = getenv("KAMI_VB_EARLY");
    p.early = (e && atoi(e) == 0) ? 0 : 1;
  }
  // TMA views (KAMI_VB_VIEWS=0 disables them, A/B experiments)
  if (!p.bsr) {
    const char* v = getenv("KAMI_VB_VIEWS");
    if (!v || atoi(v) != 0) p.vmap = vb_view_maps(stream);
    p.vsmall = (v && atoi(v) == 2) ? 0 : 1;
    const char* pf = getenv("KAMI_VB_PREFETCH");
    p.vprefetch = (pf && atoi(pf) == 1) ? 1 : 0;
  }
  const uint32_t smem = p.bar_off + 2048 + 1024;
  auto fn = bf16 ? kami_tc16_vb_kernel<true> : kami_tc16_vb_kernel<false>;
  if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return KAMI_ERROR_CUDA;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  long long grid = p.units < sms ? p.units : sms;
  // Mixed sizes: units u = entry * mtiles + mt are strided by the grid, so a
  // grid that shares a factor with mtiles pins every CTA to one m-tile index
  // (148 CTAs, mtiles = 2: even CTAs take every entry's first tile, odd CTAs
  // only the second tiles of m > 128 entries -- a ~3 : 1 imbalance).  A grid
  // coprime to mtiles walks each CTA through all m-tile indices.
  // (uniform sizes with a short last m-tile, m % 128 != 0, likewise)
  if (!p.sorted && p.mtiles > 1 && (p.dm || max_m % 128 != 0))
    while (grid > 1 && std::gcd(grid, (long long)p.mtiles) != 1) --grid;
  grid = apply_grid_cap(grid);
  fn<<<(unsigned)grid, kVbThreads, smem, stream>>>(p);
  if (p.strided) {
    set_last_kernel(bf16 ? "kami_tc16_vb_kernel<bf16,strided>" : "kami_tc16_vb_kernel<f16,strided>");
    return (kami_status_t)launch_status((int)cudaGetLastError());
  }
  if (p.zorder) {
    set_last_kernel(bf16 ? "kami_tc16_vb_kernel<bf16,spmm_zmorton>" : "kami_tc16_vb_kernel<f16,spmm_zmorton>");
    return (kami_status_t)launch_status((int)cudaGetLastError());
  }
  if (p.sorted) {
    set_last_kernel(bf16 ? "kami_tc16_vb_kernel<bf16,sorted>" : "kami_tc16_vb_kernel<f16,sorted>");
    return (kami_status_t)launch_status((int)cudaGetLastError());
  }
  set_last_kernel(p.bsr ? (bf16 ? "kami_tc16_vb_kernel<bf16,spmm_bsr>" : "kami_tc16_vb_kernel<f16,spmm_bsr>")
                        : (bf16 ? "kami_tc16_vb_kernel<bf16>" : "kami_tc16_vb_kernel<f16>"));
  return (kami_status_t)launch_status((int)cudaGetLastError());
}

int packing(int m, int n) {  // entries per 128-lane tile (same rule as tc16.cu)
  if (m > 128) return 1;
  const int g1 = 128 / m, g2 = 256 / n;
  const int g = g1 < g2 ? g1 : g2;
  // at most 8: the per-unit entry pointer tables hold 8 (m = 8 would pack 16)
  return g < 1 ? 1 : (g > 8 ? 8 : g);
}

}  // namespace

extern "C" int kami_debug_vb_trace(long long* out) {
  return cudaMemcpyFromSymbol(out, g_vb_trace, sizeof(long long) * 8 * 1024) == cudaSuccess ? 0 : 1;
}

kami_status_t tc16_spmm_bsr_launch(int m, int n, int k, long long batch, bool bf16, const int* row_ptr,
                                   const int* col_blk, const void* vals, int max_nnzb, const void* B, void* C,
                                   cudaStream_t stream, bool zorder) {
  VbParams p;
  memset(&p, 0, sizeof(p));
  p.zorder = zorder ? 1 : 0;
  p.m = m;
  p.n = n;
  p.k = k;
  p.batch = batch;
  p.G = packing(m, n);
  p.bsr = 1;
  {
    // dense B by TMA: G entries x 64 k-rows x n per stage, N-major atoms of
    // Wn = 64, 32 or 16 columns (128-, 64-, 32-byte swizzle), zero-filled
    // past k and past the batch
    PFN_encodeTiled enc = get_encode_tiled();
    if (!enc) return KAMI_ERROR_CUDA;
    const CUtensorMapDataType dt = bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16;
    const int wn = n % 64 == 0 ? 64 : n % 32 == 0 ? 32 : 16;
    const CUtensorMapSwizzle sw =
        wn == 64 ? CU_TENSOR_MAP_SWIZZLE_128B : wn == 32 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B;
    cuuint64_t dims[4] = {(cuuint64_t)wn, (cuuint64_t)k, (cuuint64_t)(n / wn), (cuuint64_t)batch};
    cuuint64_t strides[3] = {(cuuint64_t)n * 2, (cuuint64_t)wn * 2, (cuuint64_t)k * n * 2};
    cuuint32_t box[4] = {(cuuint32_t)wn, 64, (cuuint32_t)(n / wn), (cuuint32_t)p.G};
    cuuint32_t es[4] = {1, 1, 1, 1};
    if (enc(&p.tmB, dt, 4, const_cast<void*>(B), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
    p.b_tma = 1;
    p.b_wb = 2 * wn;
    p.b_tx = (uint32_t)(128 * n * p.G);
    // A's blocks: (16 columns, 16 rows, batch max_nnzb blocks), one block per box
    const long long nb = batch * (long long)max_nnzb;
    cuuint64_t adims[3] = {16, 16, (cuuint64_t)(nb > 0 ? nb : 1)};
    cuuint64_t astr[2] = {32, 512};
    cuuint32_t abox[3] = {16, 16, 1};
    if (enc(&p.tmA, dt, 3, const_cast<void*>(nb > 0 ? vals : B), adims, astr, abox, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  p.max_nnzb = max_nnzb;
  p.rowptr = row_ptr;
  p.colblk = col_blk;
  p.vals = static_cast<const uint16_t*>(vals);
  p.Bs = static_cast<const uint16_t*>(B);
  p.Cs = static_cast<uint16_t*>(C);
  return vb_launch(p, bf16, n, m, stream);
}

kami_status_t tc16_vb_strided_launch(int m, int n, int k, long long batch, bool bf16, const void* A, const void* B,
                                     void* C, cudaStream_t stream) {
  VbParams p;
  memset(&p, 0, sizeof(p));
  p.strided = 1;
  p.As = static_cast<const uint16_t*>(A);
  p.Bs = static_cast<const uint16_t*>(B);
  p.Cs = static_cast<uint16_t*>(C);
  p.m = m;
  p.n = n;
  p.k = k;
  p.batch = batch;
  p.G = packing(m, n);
  return vb_launch(p, bf16, n, m, stream);
}

kami_status_t tc16_vb_launch(long long batch, bool bf16, int m, int n, int k, const int* dm, const int* dn,
                             const int* dk, int max_m, int max_n, const void* const* A, const void* const* B,
                             void* const* C, cudaStream_t stream) {
  VbParams p;
  memset(&p, 0, sizeof(p));
  p.A = A;
  p.B = B;
  p.C = C;
  p.dm = dm;
  p.dn = dn;
  p.dk = dk;
  p.m = m;
  p.n = n;
  p.k = k;
  p.batch = batch;
  p.G = dm ? 1 : packing(m, n);  // mixed sizes share a tile only class-sorted
  // Variable sizes: class-sorted (pre-pass + packed tiles) for batches of at
  // least 256 entries, where the pre-pass's few microseconds are repaid;
  // KAMI_VB_SORT=0 / 1 forces it off / on (A/B experiments, tests).
  const char* env = getenv("KAMI_VB_SORT");
  const bool sort = dm && batch < (1ll << 30) && (env ? atoi(env) != 0 : batch >= 256);
  if (!sort) return vb_launch(p, bf16, dm ? max_n : n, dm ? max_m : m, stream);
  const long long mt_max = (max_m + 127) / 128;
  // records: 256 bytes per unit, at most batch * mt_max units
  const size_t bytes = sizeof(int) * (4 * (size_t)kClasses + 4) + 256 * (size_t)(batch * mt_max);
  void* ws = nullptr;
  cudaMemPool_t pool = vb_pool();
  if (!pool || cudaMallocFromPoolAsync(&ws, bytes, pool, stream) != cudaSuccess) return KAMI_ERROR_CUDA;
  int* hist = static_cast<int*>(ws);
  int* cursor = hist + kClasses;
  int* eoff = cursor + kClasses;
  int* uoff = eoff + kClasses;
  int* nunits = uoff + kClasses;
  int4* rec = reinterpret_cast<int4*>(nunits + 4);  // 16-byte aligned (4 kClasses + 4 ints)
  kami_status_t st = KAMI_SUCCESS;
  if (cudaMemsetAsync(hist, 0, sizeof(int) * 2 * kClasses, stream) != cudaSuccess) st = KAMI_ERROR_CUDA;
  if (cudaFuncSetAttribute(vb_class_scan, cudaFuncAttributeMaxDynamicSharedMemorySize,
                           kClasses * (int)sizeof(int)) != cudaSuccess)
    st = KAMI_ERROR_CUDA;
  if (st == KAMI_SUCCESS) {
    const int blocks = (int)((batch + 255) / 256 < 1184 ? (batch + 255) / 256 : 1184);
    vb_class_hist<<<blocks, 256, 0, stream>>>(batch, dm, dn, dk, hist);
    vb_class_scan<<<1, 1024, kClasses * sizeof(int), stream>>>(hist, eoff, uoff, nunits);
    vb_class_scatter<<<blocks, 256, 0, stream>>>(batch, dm, dn, dk, hist, uoff, cursor, A, B, C, rec);
    if (cudaGetLastError() != cudaSuccess) st = KAMI_ERROR_CUDA;
  }
  if (st == KAMI_SUCCESS) {
    p.sorted = 1;
    p.G = 8;  // buffer sizing: the widest packed tile (G n <= min(8 max_n, 256))
    p.rec = rec;
    p.nunits = nunits;
    st = vb_launch(p, bf16, max_n, max_m, stream);
  }
  cudaFreeAsync(ws, stream);  // stream-ordered: after the kernels
  return st;
}

}  // namespace kami
