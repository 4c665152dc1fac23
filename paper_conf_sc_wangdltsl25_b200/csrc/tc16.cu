// tc16.cu -- batched small GEMM on 5th-generation tensor cores (tcgen05 +
// TMEM + TMA), sm_100a.  Hot path of BASELINE.json configs 0, 1, 3 and 4
// (FP16 / BF16 in, FP32 accumulate) and of the f4 extensions (TF32 in / FP32
// out, FP8 E4M3 / E5M2 in / FP16 out, C = alpha A B + beta C).
//
// KAMI mapping (Table 1):
//   compute unit  = one SM sub-partition tensor core (n_tc = 4 per SM).  A
//                   cta_group::1 M=128 tcgen05.mma drives all four; unit i
//                   owns TMEM lanes [32i, 32i+32), i.e. rows of C_i.
//   local storage = TMEM: the C_i accumulators never leave it until the
//                   epilogue (the paper's registers, Sec. 4.2).
//   communication = shared memory: the B tile is written once (TMA) and
//                   broadcast to all four units by every MMA -- KAMI-1D
//                   (Alg. 1) with p = 4, where stage z of Alg. 1 is
//                   the z-th 32-byte K slice (k-slicing, Sec. 4.7).
//   batching      = G = min(128/m, 256/n) entries packed block-diagonally
//                   into one 128 x (G n) MMA tile: entry g's A rows occupy
//                   TMEM lanes [g m, g m + m) and its B columns [g n, g n + n),
//                   so one MMA chain computes G independent products (the
//                   off-diagonal blocks are discarded).  This is how the
//                   batched path (Sec. 5.4) fills the 128-lane
//                   datapath for m < 128.
//
// Pipeline (persistent, one CTA per SM, warp specialised):
//   warp 0     TMA producer: per (unit, k-chunk) one 3-D box of A (K-major,
//              swizzled) and one 4-D box of B (N-major, swizzled) into an
//              S-stage shared-memory ring guarded by full/empty mbarriers.
//   warp 1     MMA issuer (one lane) + TMEM allocator: tcgen05.mma,
//              accumulators double/quad-buffered in TMEM, tcgen05.commit ->
//              empty[s] (frees the stage) and tfull[a].
//   warps 2-9  epilogue, two warpgroups on alternate units: tcgen05.ld
//              32x32b, (beta != 0: TMA-load the old C tile into the staging
//              buffer first), alpha/beta, cvt.rn, swizzled conflict-free
//              st.shared into the C staging tile, one TMA tensor store.
//              FP32 output (TF32 inputs): alpha/beta and 32-byte full-sector
//              st.global straight from registers (a 128 x 256 FP32 staging
//              tile per warpgroup would not fit next to the ring).
//   warps 10-13 (TF32 only) B transposer.  kind::tf32 reads both operands
//              K-major only (an MN-major B descriptor yields zeros on sm_100a,
//              DESIGN.md R25), and TMA cannot transpose 4-byte elements, so
//              B lands N-major in a raw slot of the stage and these warps
//              rewrite it K-major (SW-swizzled, same canonical layout as A)
//              before arriving on bready[s], which the MMA issuer waits on.
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <numeric>

#include "kernels.h"
#include "ptx.cuh"
#include "sched.cuh"

namespace kami {

namespace {

// Diagnostic builds only (-DKAMI_PHASE_TIMING, tools/latency.py): CTA 0 records
// clock64 at the pipeline's phase boundaries and prints them at exit.
#ifdef KAMI_PHASE_TIMING
#define KAMI_TS(i) (kami_ts[i] = clock64())
#else
#define KAMI_TS(i) ((void)0)
#endif

constexpr int kThreads = 320;  // 10 warps: TMA, MMA, 2 x 4 epilogue
constexpr int kXposeThreads = 128;  // TF32: 4 more warps transpose B
constexpr int kEpiThreads = 128;
constexpr int kMaxStages = 8;
constexpr int kMaxAcc = 4;

// input kinds (A, B) and output kinds (C)
enum { IN_F16 = 0, IN_BF16 = 1, IN_TF32 = 2, IN_E4M3 = 3, IN_E5M2 = 4 };
enum { OUT_F16 = 0, OUT_BF16 = 1, OUT_F32 = 2 };
template <int kIn>
struct InTraits {
  static constexpr int ES = kIn == IN_TF32 ? 4 : (kIn >= IN_E4M3 ? 1 : 2);
};
constexpr int threads_for(int in) { return kThreads + (in == IN_TF32 ? kXposeThreads : 0); }
template <int kOut>
struct OutTraits {
  static constexpr int ES = kOut == OUT_F32 ? 4 : 2;
};

struct alignas(64) Tc16Params {
  CUtensorMap tmA;  // 3-D (k, m, batch), box (Wk, rowsA, G)
  CUtensorMap tmB;  // 4-D (Wn, k, n/Wn, batch), box (Wn, Wk, n/Wn, G)
  CUtensorMap tmC;  // 4-D (Wc, m, n/Wc, batch), box (Wc, rows_tile, n/Wc, G)
  CUtensorMap tmCa; // split stores: same tensor, box (Wc, rows_tile, 1, 1) = one 64-column atom
  long long batch;
  long long units;
  int m, n, k;
  int G, m_tiles, rows_tile;
  int slot;                  // TMEM lanes / A-tile rows per packed entry (m, or 32 for thin m, see plan)
  int colrep;                // thin m, one entry per tile: A replicated into colrep 32-lane slots (plan)
  int k_chunks, Wk, Wn, Wc;  // atom widths in ELEMENTS of their operand
  int ksteps_full, ksteps_last;
  int N_mma;
  int U, GU;               // sub-tiles (MMA tiles) per unit; entries per unit = G * U
  uint32_t a_sub, b_sub;   // byte offsets between sub-tiles' A and B operands
  uint32_t idesc;
  uint32_t a_layout, b_layout, c_swz_bits;
  uint32_t a_sbo, b_lbo, b_sbo, b_kstep;  // bytes
  uint32_t a_region, stage_bytes, tx_bytes, c_tx_bytes;
  int stages;
  int acc_cols, acc_bufs, tmem_cols;
  uint32_t c_buf_bytes;
  int c_bufs;
  uint32_t c_off;    // byte offset of C staging
  uint32_t bar_off;  // byte offset of barriers
  float alpha, beta;
  uint32_t b_raw_off;       // TF32: byte offset in the stage of the N-major raw B slot
  uint32_t raw_swz_bits, k_swz_bits;
  int wn_b, wk_b;           // atom widths in bytes
  void* Cg;                 // FP32 output: direct stores
  int scale;  // 0: C = AB, 1: C = alpha AB, 2: C = alpha AB + beta C (C read)
  int split_store;  // G == U == 1, 64-column atoms, n >= 128: one TMA store per atom as it is written
  // pointer arrays (kPtr): entry e's matrices at Aa[e], Ba[e], Ca[e]; the tensor
  // maps are address-space views (view_coords) and every entry is its own box
  const void* const* Aa;
  const void* const* Ba;
  void* const* Ca;
  uint32_t a_entry, b_entry, c_entry;  // shared-memory bytes of one entry's A / B / C box
  uint32_t entry_tx, entry_tx_t;       // TMA bytes of one entry's A + B boxes per k-chunk (full / tail m-tile)
  int l2hint;                          // 1: C stores evict_first in L2, 2: also the A loads (experiment)
  // tail packing (kTP; 128 < m <= 192, n <= 128): units come in threes per
  // pair of entries -- head(e), head(e+1), then both entries' last m - 128
  // rows packed block-diagonally into one tile (64-lane slots, N = 2n)
  int tpack;
  int warp_store;                      // kWS: every epilogue warp stores its own 32-row slabs (tmCw)
  CUtensorMap tmCw;                    // box (Wc, 32, 1, 1)
  uint32_t tx_tail, idesc_tail;
  CUtensorMap tmAt2, tmBt2, tmCt2;     // boxes (Wk, 64, 2), (Wn, Wk, n/Wn, 2), (Wc, 64, n/Wc, 2)
  int m_tail;                          // m > 128, m % 128 != 0: the last m-tile uses tmAt / tmCat
  CUtensorMap tmAt, tmCat;             // pointer arrays: boxes of m % 128 rows for the last m-tile
};

// Pointer arrays on TMA: address-space views (view_coords, sched.cuh).

template <int kIn>
__device__ __forceinline__ void umma(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  if constexpr (kIn == IN_TF32) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
        "l"(a), "l"(b), "r"(idesc), "r"(acc)
        : "memory");
  } else if constexpr (kIn >= IN_E4M3) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f8f6f4 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
        "l"(a), "l"(b), "r"(idesc), "r"(acc)
        : "memory");
  } else {
    ptx::umma_f16_ss(d, a, b, idesc, acc);
  }
}

// 8 fp32 accumulators -> the output type, written as 16-byte chunks of the
// swizzled staging tile.  `off` is the unswizzled byte offset of the first
// element; old values (beta != 0) are read from the same locations.
template <int kOut, bool kUpd>
__device__ __forceinline__ void emit8(uint32_t cbase, uint32_t off, uint32_t swz_bits, const uint32_t* v,
                                      const Tc16Params& p) {
  float x[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) x[i] = __uint_as_float(v[i]);
  if (kUpd && p.scale) {
#pragma unroll
    for (int i = 0; i < 8; ++i) x[i] *= p.alpha;
  }
  if constexpr (kOut == OUT_F32) {
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const uint32_t a = cbase + ptx::swz(off + 16 * h, swz_bits);
      if (kUpd && p.scale == 2) {
        uint32_t o0, o1, o2, o3;
        ptx::ld_shared_v4(a, o0, o1, o2, o3);
        x[4 * h + 0] = fmaf(p.beta, __uint_as_float(o0), x[4 * h + 0]);
        x[4 * h + 1] = fmaf(p.beta, __uint_as_float(o1), x[4 * h + 1]);
        x[4 * h + 2] = fmaf(p.beta, __uint_as_float(o2), x[4 * h + 2]);
        x[4 * h + 3] = fmaf(p.beta, __uint_as_float(o3), x[4 * h + 3]);
      }
      ptx::st_shared_v4(a, __float_as_uint(x[4 * h + 0]), __float_as_uint(x[4 * h + 1]),
                        __float_as_uint(x[4 * h + 2]), __float_as_uint(x[4 * h + 3]));
    }
  } else {
    const uint32_t a = cbase + ptx::swz(off, swz_bits);
    if (kUpd && p.scale == 2) {
      uint32_t o[4];
      ptx::ld_shared_v4(a, o[0], o[1], o[2], o[3]);
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        float lo, hi;
        if (kOut == OUT_BF16) {
          lo = __uint_as_float(o[i] << 16);
          hi = __uint_as_float(o[i] & 0xffff0000u);
        } else {
          const __half2 h2 = *reinterpret_cast<const __half2*>(&o[i]);
          lo = __low2float(h2);
          hi = __high2float(h2);
        }
        x[2 * i] = fmaf(p.beta, lo, x[2 * i]);
        x[2 * i + 1] = fmaf(p.beta, hi, x[2 * i + 1]);
      }
    }
    uint32_t w[4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
      w[i] = kOut == OUT_BF16 ? ptx::pack_bf16x2(x[2 * i], x[2 * i + 1]) : ptx::pack_f16x2(x[2 * i], x[2 * i + 1]);
    ptx::st_shared_v4(a, w[0], w[1], w[2], w[3]);
  }
}

// FP32 output: 8 accumulators -> 32 contiguous bytes of C (one full sector).
template <bool kUpd>
__device__ __forceinline__ void emit8_f32_global(float* dst, const uint32_t* v, const Tc16Params& p) {
  float x[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) x[i] = __uint_as_float(v[i]);
  if (kUpd && p.scale) {
#pragma unroll
    for (int i = 0; i < 8; ++i) x[i] *= p.alpha;
  }
  if (kUpd && p.scale == 2) {
    const float4 o0 = *reinterpret_cast<const float4*>(dst);
    const float4 o1 = *reinterpret_cast<const float4*>(dst + 4);
    x[0] = fmaf(p.beta, o0.x, x[0]);
    x[1] = fmaf(p.beta, o0.y, x[1]);
    x[2] = fmaf(p.beta, o0.z, x[2]);
    x[3] = fmaf(p.beta, o0.w, x[3]);
    x[4] = fmaf(p.beta, o1.x, x[4]);
    x[5] = fmaf(p.beta, o1.y, x[5]);
    x[6] = fmaf(p.beta, o1.z, x[6]);
    x[7] = fmaf(p.beta, o1.w, x[7]);
  }
  ptx::st_global_v4(dst, make_uint4(__float_as_uint(x[0]), __float_as_uint(x[1]), __float_as_uint(x[2]),
                                    __float_as_uint(x[3])));
  ptx::st_global_v4(dst + 4, make_uint4(__float_as_uint(x[4]), __float_as_uint(x[5]), __float_as_uint(x[6]),
                                        __float_as_uint(x[7])));
}

// kUpd: the C-update epilogue (alpha != 1 or beta != 0); the plain C = AB
// instantiation carries none of its code.
template <int kIn, int kOut, bool kUpd, bool kSplit, bool kPtr = false, bool kTP = false, bool kWS = false>
__global__ void __launch_bounds__(threads_for(kIn), 1) kami_tc16_1d_kernel(const __grid_constant__ Tc16Params p) {
  constexpr bool kXpose = kIn == IN_TF32;
  constexpr bool kDirect = kOut == OUT_F32;
  constexpr int ESO = OutTraits<kOut>::ES;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1024-byte alignment for the 128B swizzle atoms
  // 1024-byte aligned base; pointer arithmetic on the __shared__ array keeps
  // the address space, so table reads compile to LDS rather than generic loads
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + p.bar_off);
  uint64_t* empty = full + kMaxStages;
  uint64_t* tfull = empty + kMaxStages;
  uint64_t* tempty = tfull + kMaxAcc;
  uint64_t* cfull = tempty + kMaxAcc;  // [2 warpgroups][2 staging buffers]: old C landed
  uint64_t* bready = cfull + 4;  // TF32: K-major B of stage s written
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bready + kMaxStages);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
#ifdef KAMI_PHASE_TIMING
  __shared__ long long kami_ts[12];
  if (threadIdx.x == 0) KAMI_TS(0);
#endif

  if (threadIdx.x == 0) {
    ptx::prefetch_tmap(&p.tmA);
    ptx::prefetch_tmap(&p.tmB);
    ptx::prefetch_tmap(&p.tmC);
    if (kSplit) ptx::prefetch_tmap(&p.tmCa);
    for (int s = 0; s < p.stages; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
      ptx::mbar_init(&bready[s], kXposeThreads);
    }
    for (int a = 0; a < p.acc_bufs; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], kEpiThreads / 32);
    }
    for (int c = 0; c < 4; ++c) ptx::mbar_init(&cfull[c], 1);
    ptx::fence_mbar_init();
    ptx::fence_proxy_async_smem();
  }
  if (warp == 1) ptx::tmem_alloc(tmem_slot, p.tmem_cols);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  if (threadIdx.x == 0 && blockIdx.x == 0) KAMI_TS(1);

  const uint32_t smem_base = ptx::smem_u32(smem);

  if (kPtr && warp == 0) {
    // ------------------------------------------- producer, pointer arrays
    // lane i < G U owns entry e0 + i of each unit: it holds that entry's A / B
    // view coordinates (fetched one unit ahead, so the pointer loads are off
    // the critical path) and issues its two TMA boxes; lane 0 does the ring
    // bookkeeping for the unit's valid entries.
    RingPos r;
    UnitIter ui(blockIdx.x, gridDim.x, p.m_tiles);
    const void* qa = nullptr;
    const void* qb = nullptr;
    {
      const long long e = (long long)(ui.grp * p.GU) + lane;
      if (lane < p.GU && e < p.batch) {
        qa = p.Aa[e];
        qb = p.Ba[e];
      }
    }
    for (long long u = blockIdx.x; u < p.units; u += gridDim.x) {
      const long long e0 = ui.grp * p.GU;
      const long long left = p.batch - e0;
      const int nvalid = left < p.GU ? (int)left : p.GU;
      int alo, ahi, blo, bhi;
      view_coords(qa, alo, ahi);
      view_coords(qb, blo, bhi);
      const int mt = ui.mt;
      ui.next();
      const void* na = nullptr;
      const void* nb = nullptr;
      if (u + gridDim.x < p.units) {  // next unit's pointers
        const long long e = (long long)(ui.grp * p.GU) + lane;
        if (lane < p.GU && e < p.batch) {
          na = p.Aa[e];
          nb = p.Ba[e];
        }
      }
      const bool tail = p.m_tail && mt == p.m_tiles - 1;
      const CUtensorMap* tma = tail ? &p.tmAt : &p.tmA;
      const uint32_t tx = (uint32_t)nvalid * (tail ? p.entry_tx_t : p.entry_tx);
      for (int kc = 0; kc < p.k_chunks; ++kc, r.next(p.stages)) {
        if (lane == 0) {
          ptx::mbar_wait(&empty[r.s], r.ph ^ 1);
          ptx::mbar_arrive_expect_tx(&full[r.s], tx);
        }
        __syncwarp();
        if (lane < nvalid) {
          uint8_t* sa = smem + r.s * p.stage_bytes;
          ptx::tma_load_4d(sa + lane * p.a_entry, tma, &full[r.s], kc * p.Wk, mt * 128, alo, ahi);
          ptx::tma_load_5d(sa + p.a_region + lane * p.b_entry, &p.tmB, &full[r.s], 0, kc * p.Wk, 0, blo, bhi);
        }
      }
      qa = na;
      qb = nb;
    }
  } else if (warp == 0) {
    // ------------------------------------------------------------ producer
    if (lane == 0) {
      const uint64_t pol = ptx::policy_evict_first();
      RingPos r;
      UnitIter ui(blockIdx.x, gridDim.x, p.m_tiles);
      for (long long u = blockIdx.x; u < p.units; u += gridDim.x, ui.next()) {
        const int e0 = (int)(ui.grp * p.GU);
        if constexpr (kTP) {  // head(2 grp), head(2 grp + 1), packed tail pair
          const int e2 = (int)(ui.grp * 2);
          const bool tl = ui.mt == 2;
          for (int kc = 0; kc < p.k_chunks; ++kc, r.next(p.stages)) {
            ptx::mbar_wait(&empty[r.s], r.ph ^ 1);
            ptx::mbar_arrive_expect_tx(&full[r.s], tl ? p.tx_tail : p.tx_bytes);
            uint8_t* sa = smem + r.s * p.stage_bytes;
            if (tl) {
              ptx::tma_load_3d(sa, &p.tmAt2, &full[r.s], kc * p.Wk, 128, e2);
              ptx::tma_load_4d(sa + p.a_region, &p.tmBt2, &full[r.s], 0, kc * p.Wk, 0, e2);
            } else {
              ptx::tma_load_3d(sa, &p.tmA, &full[r.s], kc * p.Wk, 0, e2 + ui.mt);
              ptx::tma_load_4d(sa + p.a_region, &p.tmB, &full[r.s], 0, kc * p.Wk, 0, e2 + ui.mt);
            }
          }
          continue;
        }
        for (int kc = 0; kc < p.k_chunks; ++kc, r.next(p.stages)) {
          ptx::mbar_wait(&empty[r.s], r.ph ^ 1);
          ptx::mbar_arrive_expect_tx(&full[r.s], p.tx_bytes);
          uint8_t* sa = smem + r.s * p.stage_bytes;
          uint8_t* sb = sa + p.a_region;
          if (p.l2hint >= 2) ptx::tma_load_3d_hint(sa, &p.tmA, &full[r.s], kc * p.Wk, ui.mt * 128, e0, pol);
          else ptx::tma_load_3d(sa, &p.tmA, &full[r.s], kc * p.Wk, ui.mt * 128, e0);
          for (int j = 1; j < p.colrep; ++j)  // the same A box into 32-lane slot j
            ptx::tma_load_3d(sa + j * 32 * p.wk_b, &p.tmA, &full[r.s], kc * p.Wk, ui.mt * 128, e0);
          ptx::tma_load_4d(kXpose ? sa + p.b_raw_off : sb, &p.tmB, &full[r.s], 0, kc * p.Wk, 0, e0);
          if (u == blockIdx.x && kc == 0) KAMI_TS(2);
        }
      }
    }
  } else if (warp == 1) {
    // ---------------------------------------------------------- MMA issuer
    RingPos r, ra;
    // descriptors of stage 0; a stage / K step only moves the 14-bit start
    // address field (addresses are < 256 KB, so the field never carries)
    const uint64_t adesc0 = ptx::make_smem_desc(smem_base, 16, p.a_sbo, p.a_layout);
    const uint64_t bdesc0 = ptx::make_smem_desc(smem_base + p.a_region, p.b_lbo, p.b_sbo, p.b_layout);
    const uint32_t stage16 = p.stage_bytes >> 4, bstep16 = p.b_kstep >> 4;
    UnitIter mui(blockIdx.x, gridDim.x, p.m_tiles);  // (kTP: the unit type)
    for (long long u = blockIdx.x; u < p.units; u += gridDim.x, ra.next(p.acc_bufs), mui.next()) {
      ptx::mbar_wait(&tempty[ra.s], ra.ph ^ 1);
      ptx::tc_fence_after();
      const uint32_t d_tmem = tmem_base + ra.s * p.acc_cols;
      const uint32_t idesc = (kTP && mui.mt == 2) ? p.idesc_tail : p.idesc;
      for (int kc = 0; kc < p.k_chunks; ++kc, r.next(p.stages)) {
        ptx::mbar_wait(kXpose ? &bready[r.s] : &full[r.s], r.ph);
        ptx::tc_fence_after();
        if (lane == 0 && u == blockIdx.x && kc == 0) KAMI_TS(3);
        if (lane == 0) {
          const uint64_t ad = adesc0 + r.s * stage16, bd = bdesc0 + r.s * stage16;
          const int nsteps = (kc == p.k_chunks - 1) ? p.ksteps_last : p.ksteps_full;
          for (int j = 0; j < p.U; ++j) {  // sub-tile j: entries [jG, jG + G) of the unit
            const uint64_t adj = ad + j * (p.a_sub >> 4), bdj = bd + j * (p.b_sub >> 4);
            for (int ks = 0; ks < nsteps; ++ks) {
              // A: K-major, one K step = 32 bytes further along the swizzled row;
              // B: N-major, one K step = 32/es K rows further (TF32: K-major, 32 bytes)
              umma<kIn>(d_tmem + j * p.N_mma, adj + 2 * ks, bdj + bstep16 * ks, idesc, (kc | ks) != 0);
            }
          }
          ptx::umma_commit(&empty[r.s]);  // stage s may be refilled once these MMAs retire
        }
        __syncwarp();
      }
      if (lane == 0) ptx::umma_commit(&tfull[ra.s]);  // accumulator complete
      if (lane == 0) KAMI_TS(4);
      __syncwarp();
    }
  } else if (kXpose && warp >= kThreads / 32) {
    // ------------------------------------------------- TF32 B transposer
    // raw (N-major) element (kk, c) of the stage: atom c / Wn, row kk:
    //   ((c / Wn) Wk + kk) wn_b + (c % Wn) 4    [swizzled with raw_swz_bits]
    // K-major element (c, kk): c wk_b + 4 kk  [swizzled with k_swz_bits]
    // Thread t takes columns c = t, t + 128, ... (conflict-free 4-byte reads
    // along a raw row) and 4 consecutive kk (one 16-byte K-major chunk).
    const int t = threadIdx.x - kThreads;
    const int wn_shift = 31 - __clz(p.Wn);
    const int kq = p.Wk >> 2;
    RingPos r;
    for (long long u = blockIdx.x; u < p.units; u += gridDim.x) {
      for (int kc = 0; kc < p.k_chunks; ++kc, r.next(p.stages)) {
        const uint32_t s = r.s;
        ptx::mbar_wait(&full[s], r.ph);
        const uint32_t raw = smem_base + s * p.stage_bytes + p.b_raw_off;
        const uint32_t dst = smem_base + s * p.stage_bytes + p.a_region;
        for (int c = t; c < p.U * p.N_mma; c += kXposeThreads) {
          const uint32_t cbase = (uint32_t)((c >> wn_shift) * p.Wk) * p.wn_b + (uint32_t)(c & (p.Wn - 1)) * 4;
          for (int q = 0; q < kq; ++q) {
            uint32_t w[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) w[j] = ptx::ld_shared_u32(raw + ptx::swz(cbase + (4 * q + j) * p.wn_b,
                                                                                  p.raw_swz_bits));
            ptx::st_shared_v4(dst + ptx::swz((uint32_t)c * p.wk_b + 16 * q, p.k_swz_bits), w[0], w[1], w[2], w[3]);
          }
        }
        ptx::fence_proxy_async_smem();  // generic writes -> the MMA's async-proxy reads
        ptx::mbar_arrive(&bready[s]);
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue
    // Two warpgroups (warps 2-5 and 6-9) take alternate units, so one can
    // drain TMEM / write SMEM while the other's TMA store is in flight.
    const int wg = (warp - 2) >> 2;
    const int sp = warp & 3;  // TMEM sub-partition this warp may access (lanes 32sp..)
    const int L = sp * 32 + lane;
    const bool leader = ((warp & 3) == 2) && lane == 0;  // warps 2 and 6
    const uint32_t bar_id = 1 + wg;
    // ---- per-thread geometry, independent of the unit (no divisions in the loop)
    int g, r, col_lo, col_hi;
    bool row_ok;
    if (p.G > 1) {
      g = L / p.slot;
      r = L - g * p.slot;
      row_ok = g < p.G && r < p.m;
      const int glo = (sp * 32) / p.slot;
      int ghi = (sp * 32 + 31) / p.slot;
      if (ghi > p.G - 1) ghi = p.G - 1;
      col_lo = glo * p.n;
      col_hi = glo < p.G ? (ghi + 1) * p.n : col_lo;
    } else if (p.colrep) {
      // thin m, replicated A: sub-partition sp holds every column of the entry
      // in its lanes; its warp drains only the 64-column block sp
      g = 0;
      r = lane;
      row_ok = lane < p.m;
      col_lo = 64 * sp;
      col_hi = sp < p.colrep ? min(64 * sp + 64, p.n) : col_lo;
    } else {
      g = 0;
      r = L;
      row_ok = L < p.rows_tile;
      col_lo = 0;
      col_hi = (sp * 32 < p.rows_tile) ? p.n : 0;
    }
    const int my_lo = g * p.n, my_hi = my_lo + p.n;
    const uint32_t row_bytes = (uint32_t)p.Wc * ESO;
    const uint32_t atom_stride = (uint32_t)p.rows_tile * row_bytes;
    const uint32_t rowbase = (uint32_t)(g * (p.n / p.Wc) * p.rows_tile + r) * row_bytes;
    // kTP tail tiles: two entries' last t = m - 128 rows in 64-lane slots, N = 2n
    const int t_rows = p.m - 128;
    const int tg = L >> 6, tr = L & 63;
    const bool t_row_ok = tr < t_rows;
    const int t_col_lo = tg * p.n, t_col_hi = ((sp * 32) & 63) < t_rows ? t_col_lo + p.n : t_col_lo;
    const uint32_t t_atom_stride = 64u * row_bytes;
    const uint32_t t_rowbase = (uint32_t)(tg * (p.n / p.Wc) * 64 + tr) * row_bytes;
    const int wc_shift = 31 - __clz(p.Wc);
    const uint32_t c_smem = smem_base + p.c_off + (uint32_t)wg * p.c_bufs * p.c_buf_bytes;
    // this warpgroup's units: u0 + 2j gridDim; accumulators wg, wg + 2, ... (mod acc_bufs);
    // staging buffers 0, 1, 0, ... (mod c_bufs) -- all advanced incrementally
    const long long u0 = blockIdx.x + (long long)wg * gridDim.x;
    UnitIter ui(u0, 2ll * gridDim.x, p.m_tiles);
    uint32_t a = wg, aph = 0;
    if (a >= (uint32_t)p.acc_bufs) {  // acc_bufs >= 2 always (N_mma <= 256); kept general
      a -= p.acc_bufs;
      aph = 1;
    }
    RingPos cpos;
    // pointer arrays: lane i < G U of the leader warp stores entry e0 + i of the
    // unit (its own bulk groups); its C view coordinates are fetched one unit ahead
    const bool storer = kPtr ? (((warp & 3) == 2) && lane < p.GU) : leader;
    const uint64_t cpol = ptx::policy_evict_first();
    const void* qc = nullptr;
    if (kPtr && storer && u0 < p.units && ui.grp * p.GU + lane < p.batch) qc = p.Ca[ui.grp * p.GU + lane];
    for (long long u = u0; u < p.units; u += 2ll * gridDim.x, ui.next()) {
      const int mt = ui.mt;
      const uint32_t cb = cpos.s;
      // per-unit geometry (kTP: head units are one entry's rows 0..127, tail
      // units the packed last rows of two entries)
      const bool tl = kTP && mt == 2;
      const long long e0 = kTP ? ui.grp * 2 + (tl ? 0 : mt) : ui.grp * p.GU;
      const int mrow = kTP ? (tl ? 128 : 0) : mt * 128;  // first C row of the unit's tile
      const int q_g = tl ? tg : g, q_lo = tl ? t_col_lo : col_lo, q_hi = tl ? t_col_hi : col_hi;
      const int q_my_lo = tl ? tg * p.n : my_lo, q_my_hi = q_my_lo + p.n;
      const uint32_t q_rowbase = tl ? t_rowbase : rowbase, q_astride = tl ? t_atom_stride : atom_stride;
      const bool valid0 = tl ? t_row_ok : (row_ok && (p.G > 1 || kTP || mt * 128 + r < p.m));  // r = L except replicated tiles
      int clo = 0, chi = 0;
      bool cstore = false;
      if constexpr (kPtr) {
        cstore = storer && e0 + lane < p.batch;
        view_coords(qc, clo, chi);
        UnitIter nx = ui;
        nx.next();
        qc = nullptr;
        if (storer && u + 2ll * gridDim.x < p.units && nx.grp * p.GU + lane < p.batch) qc = p.Ca[nx.grp * p.GU + lane];
      }
      if constexpr (kWS) {
        // Per-warp C stores (one entry per tile, 64-column atoms): each warp
        // stages its own 32 rows of every atom (colrep tiles: its own atom) and
        // stores them with its own TMA box as soon as they are written -- no
        // warpgroup barrier; a warp only waits for its own previous stores to
        // leave shared memory before reusing its slab.
        const uint32_t cbase = c_smem + cb * p.c_buf_bytes;
        uint8_t* cbuf = smem + p.c_off + (wg * p.c_bufs + cb) * p.c_buf_bytes;
        const bool active = col_hi > col_lo;
        const bool valid = valid0 && e0 < p.batch;
        if (lane == 0) ptx::bulk_wait_read<0>();
        __syncwarp();
        ptx::mbar_wait(&tfull[a], aph);
        ptx::tc_fence_after();
        const uint32_t t_row = tmem_base + (uint32_t(sp * 32) << 16) + a * p.acc_cols;
        for (int c0 = col_lo; c0 < col_hi; c0 += 64) {
          uint32_t v[64];
          const int left = col_hi - c0;
          if (left >= 64) {
            ptx::tmem_ld_32x32b_x32(t_row + c0, *reinterpret_cast<uint32_t(*)[32]>(&v[0]));
            ptx::tmem_ld_32x32b_x32(t_row + c0 + 32, *reinterpret_cast<uint32_t(*)[32]>(&v[32]));
          } else {
            ptx::tmem_ld_32x32b_x32(t_row + c0, *reinterpret_cast<uint32_t(*)[32]>(&v[0]));
          }
          ptx::tmem_wait_ld();
          const uint32_t atom = (uint32_t)(c0 >> 6);
          if (valid) {
#pragma unroll
            for (int q = 0; q < 8; ++q)
              if (8 * q < left)
                emit8<kOut, kUpd>(cbase, rowbase + atom * atom_stride + (uint32_t)(8 * q) * ESO, p.c_swz_bits,
                                  &v[8 * q], p);
          }
          ptx::fence_proxy_async_smem();
          __syncwarp();
          if (lane == 0 && active) {
            const int row0 = p.colrep ? 0 : 32 * sp;  // colrep: the warp's atom holds every row
            const uint32_t off = atom * atom_stride + (uint32_t)(p.colrep ? 0 : 32 * sp) * row_bytes;
            if (p.l2hint)
              ptx::tma_store_4d_hint(&p.tmCw, cbuf + off, 0, mt * 128 + row0, (int)atom, (int)e0, cpol);
            else
              ptx::tma_store_4d(&p.tmCw, cbuf + off, 0, mt * 128 + row0, (int)atom, (int)e0);
            ptx::bulk_commit();
          }
        }
        ptx::tc_fence_before();  // accumulator a may be overwritten by the next MMA chain
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(&tempty[a]);
        a += 2;
        if (a >= (uint32_t)p.acc_bufs) {
          a -= p.acc_bufs;
          aph ^= 1;
        }
        cpos.next(p.c_bufs);
        continue;
      }
      // the TMA store that last read staging buffer cb must be done reading
      if (!kDirect && storer) {
        // per-atom stores (kSplit) into a single staging buffer: only atom 0 of
        // the unit that last used it must be read out here (A groups per unit,
        // so A - 1 newer groups may still be in flight); each later atom waits
        // for its own slot inside the atom loop (bf16 192^3: 298 -> 317
        // TFLOP/s).  With two buffers (small tiles) waiting for everything is
        // faster (bf16 16x192x16: 26.5 vs 23.2 with per-atom waits: more stores
        // queued on the TMA unit delay the next units' loads).
        if (kSplit && p.c_bufs == 1) ptx::bulk_wait_read_n((p.n >> 6) - 1);
        else if (p.c_bufs == 2 && !kSplit) ptx::bulk_wait_read<1>();
        else ptx::bulk_wait_read<0>();
        if (kUpd && p.scale == 2) {  // C update: bring the old C tile into the staging buffer
          uint64_t* cf = &cfull[wg * 2 + cb];
          ptx::mbar_arrive_expect_tx(cf, p.c_tx_bytes);
          ptx::tma_load_4d(smem + p.c_off + (wg * p.c_bufs + cb) * p.c_buf_bytes, &p.tmC, cf, 0, mt * 128, 0,
                           (int)e0);
        }
      }
      ptx::named_bar_sync(bar_id, kEpiThreads);
      ptx::mbar_wait(&tfull[a], aph);
      ptx::tc_fence_after();
      if (leader && wg == 0 && u == u0) KAMI_TS(5);
      if (kUpd && !kDirect && p.scale == 2) ptx::mbar_wait(&cfull[wg * 2 + cb], cpos.ph);
      const uint32_t cbase = c_smem + cb * p.c_buf_bytes;
      if constexpr (kSplit && !kDirect) {
        // one 64-column atom per chunk; every warp walks every chunk (the
        // per-atom named barriers need all four), the accumulator is released
        // as soon as its last TMEM load has landed, and each atom's TMA store
        // is issued as soon as it is staged, so the store engine starts on
        // atom 0 while atoms 1.. are still being converted
        const bool active = col_hi > col_lo;
        const bool valid = valid0 && (e0 + g < p.batch);
        const uint32_t t_row = tmem_base + (uint32_t(sp * 32) << 16) + a * p.acc_cols;
        uint8_t* cbuf = smem + p.c_off + (wg * p.c_bufs + cb) * p.c_buf_bytes;
        for (int c0 = 0; c0 < p.n; c0 += 64) {
          uint32_t v[64];
          if (active) {
            ptx::tmem_ld_32x32b_x32(t_row + c0, *reinterpret_cast<uint32_t(*)[32]>(&v[0]));
            ptx::tmem_ld_32x32b_x32(t_row + c0 + 32, *reinterpret_cast<uint32_t(*)[32]>(&v[32]));
          }
          ptx::tmem_wait_ld();
          if (c0 + 64 >= p.n) {  // accumulator a may be overwritten by the next MMA chain
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) ptx::mbar_arrive(&tempty[a]);
          }
          const uint32_t atom = (uint32_t)(c0 >> 6);
          if (valid) {
#pragma unroll
            for (int q = 0; q < 8; ++q)
              emit8<kOut, kUpd>(cbase, rowbase + atom * atom_stride + (uint32_t)(8 * q) * ESO, p.c_swz_bits,
                                &v[8 * q], p);
          }
          ptx::fence_proxy_async_smem();
          // single buffer: the next atom's slot (its store of the previous unit)
          // must be read out before the barrier releases the warps onto it
          if (storer && p.c_bufs == 1 && c0 + 64 < p.n) ptx::bulk_wait_read_n((p.n >> 6) - 2);
          ptx::named_bar_sync(bar_id, kEpiThreads);
          if (kPtr ? cstore : leader) {
            if constexpr (kPtr)
              ptx::tma_store_5d(p.m_tail && mt == p.m_tiles - 1 ? &p.tmCat : &p.tmCa, cbuf + atom * atom_stride, 0,
                                mt * 128, (int)atom, clo, chi);
            else if (p.l2hint)
              ptx::tma_store_4d_hint(&p.tmCa, cbuf + atom * atom_stride, 0, mt * 128, (int)atom, (int)e0, cpol);
            else ptx::tma_store_4d(&p.tmCa, cbuf + atom * atom_stride, 0, mt * 128, (int)atom, (int)e0);
            ptx::bulk_commit();
          }
        }
        a += 2;
        if (a >= (uint32_t)p.acc_bufs) {
          a -= p.acc_bufs;
          aph ^= 1;
        }
        cpos.next(p.c_bufs);
        continue;
      }
      for (int j = 0; j < p.U; ++j) {
      const bool valid = valid0 && (e0 + j * p.G + q_g < p.batch);
      float* crow = nullptr;
      if constexpr (kDirect)
        crow = reinterpret_cast<float*>(p.Cg) + ((e0 + j * p.G + g) * p.m + mt * 128 + r) * (long long)p.n;
      const uint32_t t_row = tmem_base + (uint32_t(sp * 32) << 16) + a * p.acc_cols + j * p.N_mma;
      const uint32_t rowbase_j = q_rowbase + (uint32_t)(j * p.G * (p.n / p.Wc)) * q_astride;
      for (int c0 = q_lo; c0 < q_hi; c0 += 64) {
        uint32_t v[64];
        // issue both TMEM loads, then one wait (never read past col_hi)
        const int left = q_hi - c0;
        if (left >= 64) {
          ptx::tmem_ld_32x32b_x32(t_row + c0, *reinterpret_cast<uint32_t(*)[32]>(&v[0]));
          ptx::tmem_ld_32x32b_x32(t_row + c0 + 32, *reinterpret_cast<uint32_t(*)[32]>(&v[32]));
        } else if (left >= 48) {
          ptx::tmem_ld_32x32b_x32(t_row + c0, *reinterpret_cast<uint32_t(*)[32]>(&v[0]));
          ptx::tmem_ld_32x32b_x16(t_row + c0 + 32, *reinterpret_cast<uint32_t(*)[16]>(&v[32]));
        } else if (left >= 32) {
          ptx::tmem_ld_32x32b_x32(t_row + c0, *reinterpret_cast<uint32_t(*)[32]>(&v[0]));
        } else {
          ptx::tmem_ld_32x32b_x16(t_row + c0, *reinterpret_cast<uint32_t(*)[16]>(&v[0]));
        }
        ptx::tmem_wait_ld();
        // only the 8-column groups this block has (narrow tiles: 2 or 4, not 8)
        auto emit_q = [&](int q) {
          const int col = c0 + 8 * q;
          if (valid && col >= q_my_lo && col < q_my_hi && col < q_hi) {
            const uint32_t jc = (uint32_t)(col - q_my_lo);
            if constexpr (kDirect) {
              emit8_f32_global<kUpd>(crow + jc, &v[8 * q], p);
            } else {
              const uint32_t atom = jc >> wc_shift;
              const uint32_t ce = jc & (uint32_t)(p.Wc - 1);
              emit8<kOut, kUpd>(cbase, rowbase_j + atom * q_astride + ce * ESO, p.c_swz_bits, &v[8 * q], p);
            }
          }
        };
        if (left <= 16) {
          emit_q(0);
          emit_q(1);
        } else if (left <= 32) {
#pragma unroll
          for (int q = 0; q < 4; ++q) emit_q(q);
        } else {
#pragma unroll
          for (int q = 0; q < 8; ++q) emit_q(q);
        }
      }
      }  // sub-tiles
      // accumulator a may be overwritten by the next MMA chain
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&tempty[a]);
      a += 2;
      if (a >= (uint32_t)p.acc_bufs) {
        a -= p.acc_bufs;
        aph ^= 1;
      }
      cpos.next(p.c_bufs);
      if constexpr (kDirect) continue;
      // make the generic-proxy smem writes visible to the TMA engine
      ptx::fence_proxy_async_smem();
      ptx::named_bar_sync(bar_id, kEpiThreads);
      if constexpr (kPtr) {
        if (cstore) {
          uint8_t* cent = smem + p.c_off + (wg * p.c_bufs + cb) * p.c_buf_bytes + lane * p.c_entry;
          if (p.m_tail && mt == p.m_tiles - 1) {
            // last m-tile of m > 128, m % 128 != 0: the staging tile keeps the
            // full tile's atom stride (128 rows per atom) while a box of m % 128
            // rows reads its smem densely, so store one 64-column atom at a time
            for (int at = 0; at < p.n / p.Wc; ++at)
              ptx::tma_store_5d(&p.tmCat, cent + (uint32_t)at * atom_stride, 0, mt * 128, at, clo, chi);
          } else {
            ptx::tma_store_5d(&p.tmC, cent, 0, mt * 128, 0, clo, chi);
          }
          ptx::bulk_commit();
        }
      } else if (leader) {
        const CUtensorMap* tmc = tl ? &p.tmCt2 : &p.tmC;
        if (p.l2hint)
          ptx::tma_store_4d_hint(tmc, smem + p.c_off + (wg * p.c_bufs + cb) * p.c_buf_bytes, 0, mrow, 0, (int)e0,
                                 cpol);
        else
          ptx::tma_store_4d(tmc, smem + p.c_off + (wg * p.c_bufs + cb) * p.c_buf_bytes, 0, mrow, 0, (int)e0);
        ptx::bulk_commit();
        if (wg == 0) KAMI_TS(6);
      }
    }
    if (!kDirect && (kWS ? lane == 0 : storer)) ptx::bulk_wait<0>();
    if (leader && wg == 0) KAMI_TS(7);
  }

  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 1) ptx::tmem_dealloc(tmem_base, p.tmem_cols);
#ifdef KAMI_PHASE_TIMING
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    KAMI_TS(8);
    printf("KAMI_TS setup %lld firstTMA %lld dataLanded %lld lastCommit %lld accReady %lld storeIssued %lld "
           "storeDone %lld exit %lld\n",
           kami_ts[1] - kami_ts[0], kami_ts[2] - kami_ts[0], kami_ts[3] - kami_ts[0], kami_ts[4] - kami_ts[0],
           kami_ts[5] - kami_ts[0], kami_ts[6] - kami_ts[0], kami_ts[7] - kami_ts[0], kami_ts[8] - kami_ts[0]);
  }
#endif
}

// ------------------------------------------------------------------- host

int pick_atom_bytes(int bytes) {  // largest swizzle atom (bytes) dividing the row bytes
  if (bytes % 128 == 0) return 128;
  if (bytes % 64 == 0) return 64;
  if (bytes % 32 == 0) return 32;
  return 0;
}
int swz_bits_for(int atom_bytes) { return atom_bytes == 128 ? 3 : atom_bytes == 64 ? 2 : 1; }
CUtensorMapSwizzle swz_mode_for(int atom_bytes) {
  return atom_bytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
         : atom_bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                            : CU_TENSOR_MAP_SWIZZLE_32B;
}
uint32_t align_up(uint32_t x, uint32_t a) { return (x + a - 1) / a * a; }
int pow2_ceil(int x) {
  int p = 32;
  while (p < x) p <<= 1;
  return p;
}
int in_es(int in) { return in == IN_TF32 ? 4 : (in >= IN_E4M3 ? 1 : 2); }
int out_es(int out) { return out == OUT_F32 ? 4 : 2; }

constexpr int kSmemLimit = 232448;  // 227 KB opt-in per CTA

// Experiment knobs (tools/tc_tune.py), read once: KAMI_TC_TUNE="stages,cbufs,grid,promo,U,split,slot"
// (0 / -1 = planner default; promo = TMA L2 promotion 0 none, 1 64B, 2 128B, 3 256B;
// U = sub-tiles per unit; split = -1 disables per-atom C stores, 1 forces them where
// possible; slot = -1 disables thin-m slots; hint = -1 no L2 policy, 1 C evict_first,
// 2 C and A evict_first, 0 planner rule).  Unset in production.
struct TcTune {
  int stages = 0, cbufs = 0, grid = 0, promo = -1, U = 0, split = 0, slot = 0, hint = 0, tp = 0, ws = 0;
};
const TcTune& tc_tune() {
  static const TcTune t = [] {
    TcTune r;
    if (const char* e = getenv("KAMI_TC_TUNE")) sscanf(e, "%d,%d,%d,%d,%d,%d,%d,%d,%d,%d", &r.stages, &r.cbufs, &r.grid, &r.promo, &r.U, &r.split, &r.slot,
                 &r.hint, &r.tp, &r.ws);
    return r;
  }();
  return t;
}

template <int kIn, int kOut>
void launch_kernel(const Tc16Params& p, unsigned grid, size_t smem, cudaStream_t stream, const char* name) {
  if constexpr (kIn <= IN_BF16) {
    if (p.warp_store) {  // per-warp C stores (strided C = AB, one entry per tile)
      cudaFuncSetAttribute(kami_tc16_1d_kernel<kIn, kOut, false, false, false, false, true>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      kami_tc16_1d_kernel<kIn, kOut, false, false, false, false, true><<<grid, threads_for(kIn), smem, stream>>>(p);
      set_last_kernel(kIn == IN_BF16 ? "kami_tc16_1d_kernel<bf16,warpstore>" : "kami_tc16_1d_kernel<f16,warpstore>");
      return;
    }
    if (p.tpack) {  // tail packing (strided C = AB only)
      cudaFuncSetAttribute(kami_tc16_1d_kernel<kIn, kOut, false, false, false, true>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      kami_tc16_1d_kernel<kIn, kOut, false, false, false, true><<<grid, threads_for(kIn), smem, stream>>>(p);
      set_last_kernel(kIn == IN_BF16 ? "kami_tc16_1d_kernel<bf16,tailpack>" : "kami_tc16_1d_kernel<f16,tailpack>");
      return;
    }
    if (p.Aa) {  // pointer arrays (C = AB only)
      if (p.split_store) {
        cudaFuncSetAttribute(kami_tc16_1d_kernel<kIn, kOut, false, true, true>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        kami_tc16_1d_kernel<kIn, kOut, false, true, true><<<grid, threads_for(kIn), smem, stream>>>(p);
      } else {
        cudaFuncSetAttribute(kami_tc16_1d_kernel<kIn, kOut, false, false, true>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        kami_tc16_1d_kernel<kIn, kOut, false, false, true><<<grid, threads_for(kIn), smem, stream>>>(p);
      }
      set_last_kernel(kIn == IN_BF16 ? "kami_tc16_1d_kernel<bf16,ptr>" : "kami_tc16_1d_kernel<f16,ptr>");
      return;
    }
  }
  if (p.scale) {  // the update form always stores whole units
    cudaFuncSetAttribute(kami_tc16_1d_kernel<kIn, kOut, true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)smem);
    kami_tc16_1d_kernel<kIn, kOut, true, false><<<grid, threads_for(kIn), smem, stream>>>(p);
  } else if (kOut != OUT_F32 && p.split_store) {
    cudaFuncSetAttribute(kami_tc16_1d_kernel<kIn, kOut, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)smem);
    kami_tc16_1d_kernel<kIn, kOut, false, true><<<grid, threads_for(kIn), smem, stream>>>(p);
  } else {
    cudaFuncSetAttribute(kami_tc16_1d_kernel<kIn, kOut, false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         (int)smem);
    kami_tc16_1d_kernel<kIn, kOut, false, false><<<grid, threads_for(kIn), smem, stream>>>(p);
  }
  set_last_kernel(name);
}

}  // namespace

kami_status_t tc16_plan_shape_kind(int m, int n, int k, int in_kind, int out_kind, Tc16Shape* s, bool no_tp) {
  const int esi = in_es(in_kind), eso = out_es(out_kind);
  // m, n multiples of 16 (TMEM lane groups / swizzle atoms of whole 16-element
  // rows); 8 mod 16 goes to the LDG-fed kernel (tc16_vb.cu)
  if (m % 16 || n % 16) return KAMI_ERROR_NOT_SUPPORTED;
  s->G = 1;
  if (m <= 128) {
    int g1 = 128 / m, g2 = 256 / n;
    s->G = g1 < g2 ? g1 : g2;
    if (s->G < 1) s->G = 1;
  }
  s->m_tiles = (s->G > 1 || m <= 128) ? 1 : (m + 127) / 128;
  s->rows_tile = m < 128 ? m : 128;
  // Tail packing: for 128 < m <= 192 the last m-tile holds only m - 128 <= 64
  // rows, so two entries' tails share one tile (block-diagonal, N = 2n <= 256):
  // 1.5 units per entry instead of 2 (three units per pair: head, head, tail)
  s->tpack = (m > 128 && m <= 192 && n <= 128 && in_kind <= IN_BF16 && !no_tp && tc_tune().tp >= 0) ? 1 : 0;
  if (s->tpack) s->m_tiles = 3;
  // Thin m packed 2 or 4 to a tile would sit in one or two TMEM sub-partitions
  // (lanes 0..G m), leaving the other epilogue warps idle: give each entry a
  // 32-lane slot instead (the A box is 32 rows; TMA zero-fills rows m..31),
  // so every entry has its own sub-partition and warp.  Strided maps only
  // (pointer-array boxes must stay inside their entry).
  s->slot = (m == 16 && (s->G == 2 || s->G == 4) && tc_tune().slot >= 0) ? 32 : s->rows_tile;
  // One thin entry per tile (m <= 32, n > 192): all of C sits in sub-partition
  // 0 and one warp drained it.  The A box is loaded into ceil(n/64) 32-lane
  // slots instead (a few hundred bytes each), so every sub-partition holds the
  // whole product and epilogue warp j drains its 64-column block j.  The MMA
  // is unchanged (it always spans 128 lanes).  Measured (profiles/r1/
  // colrep_ab_r1.txt): bf16 16x256x16 0.56 -> 0.66 of roofline, 16x256x32
  // 0.83 -> 0.95, 32x256x16 0.84 -> 0.90; n = 192 (3 blocks) and k >= 64 are
  // as fast or faster with the per-atom split stores, so they keep those.
  // With per-warp stores (below) n = 192 at k = 16 and the n % 64 != 0 shapes
  // (no per-atom split stores there) gain too: 16x192x16 0.51 -> 0.52,
  // 32x192x16 0.77 -> 0.80, 16x144x16 0.22 -> 0.38; 32x192x32 keeps the split
  // stores (0.97 vs 0.90-0.96).
  const bool rep_n = (k <= 16 && n > 128) || (k <= 32 && (n > 192 || n % 64 != 0));
  s->colrep = (s->G == 1 && m <= 32 && n > 128 && rep_n && s->m_tiles == 1 && tc_tune().slot >= 0)
                  ? (n + 63) / 64
                  : 0;
  const int kgran = 32 / esi;  // elements per 32-byte MMA K step
  const int kpad = (k + kgran - 1) / kgran * kgran;
  const int wk_b = pick_atom_bytes(kpad * esi), wn_b = pick_atom_bytes(n * esi), wc_b = pick_atom_bytes(n * eso);
  if (!wk_b || !wn_b || !wc_b) return KAMI_ERROR_NOT_SUPPORTED;
  s->Wk = wk_b / esi;
  s->Wn = wn_b / esi;
  s->Wc = wc_b / eso;
  s->k_chunks = (kpad + s->Wk - 1) / s->Wk;
  s->N_mma = s->G > 1 ? s->G * n : (s->tpack ? 2 * n : n);
  // Sub-tiles per unit: small tiles are bound by the per-unit fixed cost of
  // the single-thread producer / MMA roles and the epilogue barriers, so
  // U MMA tiles (G U entries) share one unit until a unit moves >= 32 KB
  // (f16 32^3: 48.6 -> 61.4 TFLOP/s, bf16 48^3: 45 -> 68; fp8 64^3 at 32 KB
  // per tile is faster unsplit: U = 2 would halve its C double-buffering).
  s->U = 1;
  {  // (m > 128: the U sub-tiles are U entries at the same m-tile)
    const long long rt = s->rows_tile;
    const long long tile_bytes =
        (long long)s->G * (rt * k * esi + (long long)k * n * esi + rt * n * eso);
    const int n_mma = s->tpack ? n : s->N_mma;  // (sub-tiles are decided on the unpacked tile)
    while (s->U < 4 && tile_bytes * s->U < 32 * 1024 && 2 * s->U * n_mma <= 256 && s->G * 2 * s->U <= 256)
      s->U *= 2;
  }
  if (tc_tune().U > 0) s->U = tc_tune().U;
  // Tail packing needs one entry per head unit; narrow tiles small enough for
  // sub-tiles (n <= 32 and U > 1) stay with U entries per m-tile, which is
  // faster there (bf16 192x16x16 0.53 vs 0.35 packed, 192x32x16 0.64 vs 0.53),
  // while packing wins from n = 64 or once the tile is big (192x64x16 0.78 ->
  // 0.88, 192x128x16 0.75 -> 0.97, 192x16x128 0.66 -> 0.89, 192x128x128 0.95
  // -> 1.05; profiles/r1/tp_ab_r1.txt).
  if (s->tpack && s->U > 1 && n <= 32) {
    s->tpack = 0;
    s->m_tiles = (m + 127) / 128;
    s->N_mma = n;
  }
  if (s->tpack) s->U = 1;
  for (;; s->U /= 2) {  // fall back to fewer sub-tiles if the ring does not fit
    const int rowsA = s->slot;
    const uint32_t a_region = align_up((uint32_t)((s->U - 1) * s->G * rowsA + 128) * wk_b, 1024);
    const uint32_t b_region = align_up((uint32_t)(s->U * s->N_mma) * wk_b, 1024);
    // TF32: + the raw N-major B slot the transposer reads
    s->stage_bytes = a_region + b_region * (in_kind == IN_TF32 ? 2 : 1);
    // FP32 output is stored straight from registers (no staging)
    s->c_buf_bytes = out_kind == OUT_F32 ? 0 : align_up((uint32_t)(s->U * s->G) * n * s->rows_tile * eso, 1024);
    // two epilogue warpgroups, each with c_bufs staging tiles
    s->c_bufs = (4 * s->c_buf_bytes <= 64 * 1024) ? 2 : 1;
    if (tc_tune().cbufs) s->c_bufs = tc_tune().cbufs;
    const int budget = kSmemLimit - 1024 /*align slack*/ - 1024 /*barriers*/;
    int st = (budget - (int)(2 * s->c_bufs * s->c_buf_bytes)) / (int)s->stage_bytes;
    if (st > kMaxStages) st = kMaxStages;
    // Bytes in flight per SM: beyond ~96 KB of outstanding TMA loads per SM the
    // sustained HBM throughput DROPS (measured, profiles/r1/stage_sweep_r1.txt:
    // f16 64^3 119 -> 137 TFLOP/s, f16 128^3 245 -> 283 going from 5 / 4 stages
    // of 32 KB to 3); shapes with smaller stages are insensitive.
    // At least 3 stages where they fit: stages of > 32 KB (n > 128, k >= 64)
    // would otherwise get 2 (bf16 192^3: 318 -> 344-352 TFLOP/s with 3; 256^3
    // and 192x256x192 unchanged, profiles/r1/stage_ab_r1.txt).
    int cap = (96 * 1024) / (int)s->stage_bytes;
    if (cap < 3) cap = 3;
    // Units that write at least as many bytes as they read (FP8 in / FP16 out,
    // thin-k tiles) run best with <= 4 stages: e4m3 / e5m2 64^3 175 -> 200
    // TFLOP/s going from 6 to 4; thin-k shapes unchanged; input-dominated
    // small tiles (bf16 16x16x64) want the deeper ring (-5% at 4),
    // profiles/r1/stage4_ab_r1.txt.
    {
      const long long rt = s->rows_tile;
      const long long in_b = (long long)s->G * s->U * (rt * k + (long long)k * n) * esi;
      const long long out_b = (long long)s->G * s->U * rt * n * eso;
      s->write_heavy = out_b >= in_b ? 1 : 0;
      if (s->write_heavy && cap > 4) cap = 4;
    }
    if (tc_tune().stages > 0) {
      if (st > tc_tune().stages) st = tc_tune().stages;
    } else if (st > cap) {
      st = cap;
    }
    s->stages = st;
    s->smem_bytes = s->stages * s->stage_bytes + 2 * s->c_bufs * s->c_buf_bytes + 1024 + 1024;
    s->acc_cols = pow2_ceil(s->U * s->N_mma);
    if (s->acc_cols > 256) return KAMI_ERROR_NOT_SUPPORTED;
    s->acc_bufs = 512 / s->acc_cols;
    if (s->acc_bufs > kMaxAcc) s->acc_bufs = kMaxAcc;
    if (st >= 2 || s->U == 1) break;
  }
  if (s->U != 1) s->colrep = 0;  // replication is defined for one entry per unit
  s->units = 0;
  return s->stages >= 2 ? KAMI_SUCCESS : KAMI_ERROR_NOT_SUPPORTED;
}

kami_status_t tc16_plan_shape(int m, int n, int k, Tc16Shape* s) {
  return tc16_plan_shape_kind(m, n, k, IN_F16, OUT_F16, s);
}

kami_status_t tc16_launch_kind(int m, int n, int k, long long batch, int in_kind, int out_kind, const void* A,
                               const void* B, void* C, float alpha, float beta, cudaStream_t stream, int max_ctas,
                               const void* const* Aa, const void* const* Ba, void* const* Ca) {
  const bool ptr = Aa != nullptr;
  if (ptr && (in_kind > IN_BF16 || alpha != 1.0f || beta != 0.0f || !Ba || !Ca)) return KAMI_ERROR_NOT_SUPPORTED;
  Tc16Shape s;
  // (tail packing: strided C = AB only)
  kami_status_t st = tc16_plan_shape_kind(m, n, k, in_kind, out_kind, &s, ptr || alpha != 1.0f || beta != 0.0f);
  if (st != KAMI_SUCCESS) return st;
  PFN_encodeTiled enc = get_encode_tiled();
  if (!enc) return KAMI_ERROR_CUDA;
  const int esi = in_es(in_kind), eso = out_es(out_kind);

  Tc16Params p;
  memset(&p, 0, sizeof(p));
  p.batch = batch;
  p.m = m;
  p.n = n;
  p.k = k;
  p.G = s.G;
  p.m_tiles = s.m_tiles;
  p.rows_tile = s.rows_tile;
  p.k_chunks = s.k_chunks;
  p.Wk = s.Wk;
  p.Wn = s.Wn;
  p.Wc = s.Wc;
  const int wk_b = s.Wk * esi, wn_b = s.Wn * esi, wc_b = s.Wc * eso;
  const int kgran = 32 / esi;
  const int kpad = (k + kgran - 1) / kgran * kgran;
  p.ksteps_full = wk_b / 32;
  p.ksteps_last = (kpad - (s.k_chunks - 1) * s.Wk) / kgran;
  p.N_mma = s.N_mma;
  if (in_kind == IN_TF32) {
    p.idesc = ptx::make_idesc_fmt(2, 2, 128, s.N_mma, 0, 0);  // both K-major (R25)
  } else if (in_kind >= IN_E4M3) {
    const int f = in_kind == IN_E5M2 ? 1 : 0;
    p.idesc = ptx::make_idesc_fmt(f, f, 128, s.N_mma, 0, 1);
  } else {
    p.idesc = ptx::make_idesc_f16(in_kind == IN_BF16 ? 1 : 0, 128, s.N_mma, /*a MN-major*/ 0, /*b MN-major*/ 1);
  }
  p.a_layout = ptx::umma_layout_code(wk_b);
  p.b_layout = ptx::umma_layout_code(wn_b);
  p.c_swz_bits = swz_bits_for(wc_b);
  p.a_sbo = 8 * wk_b;                      // 8 rows of the K-major A tile
  p.b_sbo = 8 * wn_b;                      // 8 K-rows of one N-atom
  p.b_lbo = s.Wk * wn_b;                   // next N-atom
  p.b_kstep = (uint32_t)(kgran / 8) * p.b_sbo;  // one 32-byte K step of B rows
  if (ptr) s.slot = s.rows_tile;  // view boxes never reach past the entry
  p.tpack = s.tpack;
  const int U = s.U, G = s.G, rowsA = s.slot;
  p.slot = s.slot;
  p.colrep = ptr ? 0 : s.colrep;
  p.U = U;
  p.GU = G * U;
  p.a_region = align_up((uint32_t)((U - 1) * G * rowsA + 128) * wk_b, 1024);
  p.a_sub = (uint32_t)(G * rowsA * wk_b);      // sub-tile j's A rows start j G m rows further
  p.b_sub = (uint32_t)(G * (n / s.Wn)) * p.b_lbo;  // and its B columns j G n columns further
  p.wn_b = wn_b;
  p.wk_b = wk_b;
  p.raw_swz_bits = swz_bits_for(wn_b);
  p.k_swz_bits = swz_bits_for(wk_b);
  p.Cg = C;
  if (in_kind == IN_TF32) {  // B is transposed in shared memory to K-major (same geometry as A)
    p.b_raw_off = p.a_region + align_up((uint32_t)(U * s.N_mma) * wk_b, 1024);
    p.b_sub = (uint32_t)(G * n * wk_b);  // K-major: one row per column
    p.b_layout = p.a_layout;
    p.b_sbo = p.a_sbo;
    p.b_lbo = 16;
    p.b_kstep = 32;
  }
  p.stage_bytes = s.stage_bytes;
  p.tx_bytes = (uint32_t)(wk_b * rowsA * G * U) + (uint32_t)(wk_b * n * G * U);
  if (p.colrep > 1) p.tx_bytes += (uint32_t)((p.colrep - 1) * wk_b * rowsA);  // replicated A boxes (G = U = 1)
  p.c_tx_bytes = (uint32_t)(G * U * n * s.rows_tile * eso);
  p.stages = s.stages;
  p.acc_cols = s.acc_cols;
  p.acc_bufs = s.acc_bufs;
  p.tmem_cols = s.acc_cols * s.acc_bufs;
  p.c_buf_bytes = s.c_buf_bytes;
  p.c_bufs = s.c_bufs;
  p.c_off = s.stages * s.stage_bytes;
  p.bar_off = p.c_off + 2 * s.c_bufs * s.c_buf_bytes;
  p.alpha = alpha;
  p.beta = beta;
  p.scale = beta != 0.0f ? 2 : (alpha != 1.0f ? 1 : 0);
  // Units that write at least what they read store C with an L2 evict_first
  // policy (streamed, never re-read): f16 lr-16 82 -> 90 TFLOP/s (0.88 -> 0.97
  // of roofline), lr-32 +0.5 %; read-dominated tiles are left alone (f16 64^3
  // was 6 % slower with it), profiles/r1/hint_ab_r1.txt.
  p.l2hint = tc_tune().hint > 0 ? tc_tune().hint : (tc_tune().hint < 0 ? 0 : s.write_heavy);
  const long long groups = s.tpack ? (batch + 1) / 2 : (batch + G * U - 1) / (G * U);
  p.units = groups * s.m_tiles;
  if (s.tpack) {
    p.tx_bytes = (uint32_t)(wk_b * 128 + wk_b * n);            // head: one entry's 128 rows
    p.tx_tail = (uint32_t)(2 * (wk_b * 64 + wk_b * n));         // tail: two entries' 64-row slots
    p.idesc_tail = p.idesc;                                     // N = 2n
    p.idesc = ptx::make_idesc_f16(in_kind == IN_BF16 ? 1 : 0, 128, n, 0, 1);  // head: N = n
  }

  const CUtensorMapDataType dti = in_kind == IN_BF16   ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                                  : in_kind == IN_F16  ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16
                                  : in_kind == IN_TF32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32
                                                       : CU_TENSOR_MAP_DATA_TYPE_UINT8;
  const CUtensorMapDataType dto = out_kind == OUT_BF16  ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                                  : out_kind == OUT_F16 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16
                                                        : CU_TENSOR_MAP_DATA_TYPE_FLOAT32;
  const CUtensorMapL2promotion promo =
      tc_tune().promo < 0 ? CU_TENSOR_MAP_L2_PROMOTION_L2_256B : (CUtensorMapL2promotion)tc_tune().promo;
  p.Aa = Aa;
  p.Ba = Ba;
  p.Ca = Ca;
  p.a_entry = (uint32_t)(rowsA * wk_b);
  p.b_entry = (uint32_t)(n * wk_b);
  p.c_entry = (uint32_t)(n * s.rows_tile * eso);
  p.entry_tx = p.tx_bytes / (uint32_t)(G * U);
  // pointer arrays: address-space views (view_coords), one entry per box
  void* const vbase = reinterpret_cast<void*>(kViewBase);
  const cuuint64_t vlo = 1ull << 24, vhi = 1ull << 20, vstride_hi = 1ull << 28;
  // Pointer-array boxes never leave their entry: on sm_100a a TMA box that is
  // partly out of bounds of an address-space view faults (measured: every k
  // tail, 64x64x40, 64x64x8, 48x80x40), where the strided maps zero-fill.  So
  // a k tail (k = 8 mod 16, the MMA K step is 16) is left to the LDG-fed
  // kernel, which zero-fills in its producer, and the last m-tile of
  // m > 128, m % 128 != 0 gets maps whose boxes have exactly m % 128 rows.
  if (ptr && (k % s.Wk) != 0) return KAMI_ERROR_NOT_SUPPORTED;
  p.m_tail = (ptr && s.G == 1 && m > 128 && (m % 128) != 0) ? 1 : 0;
  const int rows_t = m % 128;
  p.entry_tx_t = (uint32_t)(wk_b * rows_t + wk_b * n);
  if (ptr) {
    for (int t = 0; t <= p.m_tail; ++t) {  // A: (k, m, 16 B offset, 2^28 B offset)
      cuuint64_t dims[4] = {(cuuint64_t)k, (cuuint64_t)m, vlo, vhi};
      cuuint64_t strides[3] = {(cuuint64_t)k * esi, 16, vstride_hi};
      cuuint32_t box[4] = {(cuuint32_t)s.Wk, (cuuint32_t)(t ? rows_t : rowsA), 1, 1};
      cuuint32_t es[4] = {1, 1, 1, 1};
      if (enc(t ? &p.tmAt : &p.tmA, dti, 4, vbase, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
              swz_mode_for(wk_b), promo, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
        return KAMI_ERROR_NOT_SUPPORTED;  // view rejected: caller falls back
    }
    {  // B: (Wn, k, n/Wn, 16 B offset, 2^28 B offset)
      cuuint64_t dims[5] = {(cuuint64_t)s.Wn, (cuuint64_t)k, (cuuint64_t)(n / s.Wn), vlo, vhi};
      cuuint64_t strides[4] = {(cuuint64_t)n * esi, (cuuint64_t)wn_b, 16, vstride_hi};
      cuuint32_t box[5] = {(cuuint32_t)s.Wn, (cuuint32_t)s.Wk, (cuuint32_t)(n / s.Wn), 1, 1};
      cuuint32_t es[5] = {1, 1, 1, 1, 1};
      if (enc(&p.tmB, dti, 5, vbase, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, swz_mode_for(wn_b), promo,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
        return KAMI_ERROR_NOT_SUPPORTED;  // view rejected: caller falls back
    }
  } else {
  {  // A: (k, m, batch)
    cuuint64_t dims[3] = {(cuuint64_t)k, (cuuint64_t)m, (cuuint64_t)batch};
    cuuint64_t strides[2] = {(cuuint64_t)k * esi, (cuuint64_t)m * k * esi};
    cuuint32_t box[3] = {(cuuint32_t)s.Wk, (cuuint32_t)rowsA, (cuuint32_t)(G * U)};
    cuuint32_t es[3] = {1, 1, 1};
    if (enc(&p.tmA, dti, 3, const_cast<void*>(A), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
            swz_mode_for(wk_b), promo, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  {  // B: (Wn, k, n/Wn, batch)
    cuuint64_t dims[4] = {(cuuint64_t)s.Wn, (cuuint64_t)k, (cuuint64_t)(n / s.Wn), (cuuint64_t)batch};
    cuuint64_t strides[3] = {(cuuint64_t)n * esi, (cuuint64_t)wn_b, (cuuint64_t)k * n * esi};
    cuuint32_t box[4] = {(cuuint32_t)s.Wn, (cuuint32_t)s.Wk, (cuuint32_t)(n / s.Wn), (cuuint32_t)(G * U)};
    cuuint32_t es[4] = {1, 1, 1, 1};
    if (enc(&p.tmB, dti, 4, const_cast<void*>(B), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
            swz_mode_for(wn_b), promo, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  if (s.tpack) {  // tail tiles: rows 128.. of two entries (64-row slots), both entries' B
    cuuint64_t da[3] = {(cuuint64_t)k, (cuuint64_t)m, (cuuint64_t)batch};
    cuuint64_t sa_[2] = {(cuuint64_t)k * esi, (cuuint64_t)m * k * esi};
    cuuint32_t ba[3] = {(cuuint32_t)s.Wk, 64, 2};
    cuuint32_t es3[3] = {1, 1, 1};
    if (enc(&p.tmAt2, dti, 3, const_cast<void*>(A), da, sa_, ba, es3, CU_TENSOR_MAP_INTERLEAVE_NONE,
            swz_mode_for(wk_b), promo, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
    cuuint64_t db[4] = {(cuuint64_t)s.Wn, (cuuint64_t)k, (cuuint64_t)(n / s.Wn), (cuuint64_t)batch};
    cuuint64_t sb_[3] = {(cuuint64_t)n * esi, (cuuint64_t)wn_b, (cuuint64_t)k * n * esi};
    cuuint32_t bb[4] = {(cuuint32_t)s.Wn, (cuuint32_t)s.Wk, (cuuint32_t)(n / s.Wn), 2};
    cuuint32_t es4[4] = {1, 1, 1, 1};
    if (enc(&p.tmBt2, dti, 4, const_cast<void*>(B), db, sb_, bb, es4, CU_TENSOR_MAP_INTERLEAVE_NONE,
            swz_mode_for(wn_b), promo, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  }  // strided
  // Per-atom C stores (kSplit instantiation) for one-entry tiles with >= 2
  // 64-column atoms: the store engine starts on atom 0 while the rest is
  // converted and the accumulator is released early (bf16 16x192x16 0.27 ->
  // 0.52 of roofline, 192^3 0.66 -> 0.70, 256^3 0.82 -> 0.87, 32x256x64 0.89 ->
  // 0.95).  Not for full 128-row tiles with k <= 16 (C-store dominated low-rank:
  // lr-8 0.90 -> 0.84, lr-16 0.92 -> 0.85 measured), profiles/r1/split_store_r1.txt.
  // (replicated thin-m tiles store from all four warps at once: no per-atom split)
  p.split_store = (out_kind != OUT_F32 && !p.colrep && !p.tpack && s.G == 1 && s.U == 1 && s.Wc == 64 && n % 64 == 0 &&
                   n >= 128 &&
                   (!(s.rows_tile == 128 && k <= 16) || tc_tune().split > 0) && beta == 0.0f && alpha == 1.0f &&
                   tc_tune().split >= 0)
                      ? 1
                      : 0;
  if (ptr) {  // C: (Wc, m, n/Wc, 16 B offset, 2^28 B offset)
    for (int t = 0; t <= p.m_tail; ++t) {
      const cuuint32_t rows = (cuuint32_t)(t ? rows_t : s.rows_tile);
      cuuint64_t dims[5] = {(cuuint64_t)s.Wc, (cuuint64_t)m, (cuuint64_t)(n / s.Wc), vlo, vhi};
      cuuint64_t strides[4] = {(cuuint64_t)n * eso, (cuuint64_t)wc_b, 16, vstride_hi};
      cuuint32_t box[5] = {(cuuint32_t)s.Wc, rows, (cuuint32_t)(n / s.Wc), 1, 1};
      cuuint32_t es[5] = {1, 1, 1, 1, 1};
      if (!t && enc(&p.tmC, dto, 5, vbase, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    swz_mode_for(wc_b), CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
        return KAMI_ERROR_NOT_SUPPORTED;
      cuuint32_t box1[5] = {(cuuint32_t)s.Wc, rows, 1, 1, 1};
      // per-atom maps: split stores, and every tail m-tile (its staging keeps
      // the full tile's atom stride, so it is stored atom by atom)
      if ((p.split_store || t) && enc(t ? &p.tmCat : &p.tmCa, dto, 5, vbase, dims, strides, box1, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, swz_mode_for(wc_b), CU_TENSOR_MAP_L2_PROMOTION_NONE,
                               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
        return KAMI_ERROR_NOT_SUPPORTED;
    }
  } else {  // C: (Wc, m, n/Wc, batch)
    cuuint64_t dims[4] = {(cuuint64_t)s.Wc, (cuuint64_t)m, (cuuint64_t)(n / s.Wc), (cuuint64_t)batch};
    cuuint64_t strides[3] = {(cuuint64_t)n * eso, (cuuint64_t)wc_b, (cuuint64_t)m * n * eso};
    cuuint32_t box[4] = {(cuuint32_t)s.Wc, (cuuint32_t)s.rows_tile, (cuuint32_t)(n / s.Wc), (cuuint32_t)(G * U)};
    cuuint32_t es[4] = {1, 1, 1, 1};
    if (enc(&p.tmC, dto, 4, C, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, swz_mode_for(wc_b),
            CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
    cuuint32_t box1[4] = {(cuuint32_t)s.Wc, (cuuint32_t)s.rows_tile, 1, 1};
    if (p.split_store && enc(&p.tmCa, dto, 4, C, dims, strides, box1, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                             swz_mode_for(wc_b), CU_TENSOR_MAP_L2_PROMOTION_NONE,
                             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
    // Per-warp stores for replicated thin-m tiles (each warp owns one atom):
    // bf16 16x256x16 33.4 -> 35.2 TFLOP/s.  On wide one-entry tiles they tie
    // with the per-atom split stores (192^3 -2 % .. +5 %, 256^3 / 128x256x32 /
    // lr-32 within 1 % across two boxes) and lose on the full-tile k <= 16
    // low-rank shapes (lr-16 80 vs 84-92), so those keep their stores,
    // profiles/r1/ws_ab_r1.txt.  Knob ws: 1 forces where possible, -1 disables.
    const bool ws_ok = !ptr && !s.tpack && s.G == 1 && s.U == 1 && s.Wc == 64 && n % 64 == 0 && in_kind <= IN_BF16 &&
                       alpha == 1.0f && beta == 0.0f && (s.colrep || s.rows_tile % 32 == 0);
    p.warp_store = (ws_ok && (tc_tune().ws > 0 || (tc_tune().ws == 0 && s.colrep))) ? 1 : 0;
    if (p.warp_store) {
      p.split_store = 0;
      cuuint32_t boxw[4] = {(cuuint32_t)s.Wc, 32, 1, 1};
      if (enc(&p.tmCw, dto, 4, C, dims, strides, boxw, es, CU_TENSOR_MAP_INTERLEAVE_NONE, swz_mode_for(wc_b),
              CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
        return KAMI_ERROR_CUDA;
    }
    cuuint32_t boxt[4] = {(cuuint32_t)s.Wc, 64, (cuuint32_t)(n / s.Wc), 2};  // tail tiles (rows >= m clipped)
    if (s.tpack && enc(&p.tmCt2, dto, 4, C, dims, strides, boxt, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                       swz_mode_for(wc_b), CU_TENSOR_MAP_L2_PROMOTION_NONE,
                       CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }

  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  long long grid = p.units < sms ? p.units : sms;
  // Units u = group * m_tiles + mt are strided by the grid, so a grid sharing a
  // factor with m_tiles pins every CTA to one m-tile index.  When the last
  // m-tile (m % 128 rows) costs clearly less than a full one, that leaves the
  // CTAs of the full tiles on the critical path: 148 -> 147 CTAs for bf16
  // 192x192x32 112.6 -> 128.7, 192x192x64 186.6 -> 210.6, 192x256x128 329 ->
  // 345 TFLOP/s; at a cost ratio >= 0.8 (224x128x64) or k = 16 (192x256x16)
  // the lost SM weighs more (-2 %).  profiles/r1/grid_ab_r1.txt (tc_tune.py).
  if (tc_tune().grid == 0 && !s.tpack && p.m_tiles > 1 && m % 128 != 0 && k >= 32) {
    const double full = 128.0 * (k + n) + (double)k * n, last = (double)(m % 128) * (k + n) + (double)k * n;
    if (last < 0.8 * full)
      while (grid > 1 && std::gcd(grid, (long long)p.m_tiles) != 1) --grid;
  }
  if (tc_tune().grid > 0 && tc_tune().grid < p.units) grid = tc_tune().grid;  // knob overrides (A/B)
  if (max_ctas > 0 && grid > max_ctas) grid = max_ctas;
  grid = apply_grid_cap(grid);
  const size_t smem = s.smem_bytes;
  const unsigned g = (unsigned)grid;
  switch (in_kind) {
    case IN_F16: launch_kernel<IN_F16, OUT_F16>(p, g, smem, stream, "kami_tc16_1d_kernel<f16>"); break;
    case IN_BF16: launch_kernel<IN_BF16, OUT_BF16>(p, g, smem, stream, "kami_tc16_1d_kernel<bf16>"); break;
    case IN_TF32: launch_kernel<IN_TF32, OUT_F32>(p, g, smem, stream, "kami_tc16_1d_kernel<tf32,f32>"); break;
    case IN_E4M3: launch_kernel<IN_E4M3, OUT_F16>(p, g, smem, stream, "kami_tc16_1d_kernel<e4m3,f16>"); break;
    default: launch_kernel<IN_E5M2, OUT_F16>(p, g, smem, stream, "kami_tc16_1d_kernel<e5m2,f16>"); break;
  }
  return cudaGetLastError() == cudaSuccess ? KAMI_SUCCESS : KAMI_ERROR_CUDA;
}

kami_status_t tc16_launch(int m, int n, int k, long long batch, bool bf16, const void* A, const void* B, void* C,
                          cudaStream_t stream, int max_ctas) {
  return tc16_launch_kind(m, n, k, batch, bf16 ? IN_BF16 : IN_F16, bf16 ? OUT_BF16 : OUT_F16, A, B, C, 1.0f, 0.0f,
                          stream, max_ctas);
}

}  // namespace kami
