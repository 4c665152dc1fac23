// tc16_ts.cu -- KAMI 1D / 3D on tcgen05 with the LOCAL operand resident in
// tensor memory (the "TS" form of tcgen05.mma: A from TMEM, B from SMEM),
// FP16 / BF16 in, FP32 accumulate, sm_100a.  DESIGN.md "tcgen05 TS form".
//
// Why (Table 1; Sec. 4.2; L519): in KAMI each
// compute unit keeps its own tile in LOCAL storage (registers) and only the
// broadcast tile travels through shared memory.  The SS form of tcgen05.mma
// (tc16.cu) reads both operands from SMEM, so A crosses SMEM twice (TMA write,
// tensor-core read) like any non-CA tiled kernel.  Here A never touches
// SMEM: loader warps bring each thread's A row from global memory into
// registers (GMem2Reg, Alg. 1) and write it straight into the TMEM lanes
// of their sub-partition (tcgen05.st, the Reg2Reg of Alg. 1 onto the tensor
// core's local memory).  Only B is communicated through SMEM (TMA write +
// tensor-core broadcast read to the four sub-partition tensor cores), and C is
// staged once for the TMA store.  SMEM bytes per entry: 2 kn s_e + 2 mn s_e,
// against 2 (mk + kn) s_e + 2 mn s_e for tc16 and (mk + kn) s_e + (W_n mk +
// W_m kn) s_e for the non-CA tiled kernel.
//
// Roles mapped onto the SM (one persistent CTA per SM, 14 or 18 warps):
//   compute units = the 4 sub-partition tensor cores; unit q owns TMEM lanes
//                   [32q, 32q + 32): rows of A_q and C_q (p = 4).
//   warp 0        TMA producer of B (k-chunk boxes of G entries, N-major,
//                 swizzled) into an S-stage SMEM ring (full/empty mbarriers).
//   warp 1        TMEM allocator + MMA issuer: tcgen05.mma.kind::f16 with
//                 [a_tmem], b_desc; commits free the B stage, the A slot and
//                 publish the accumulator.
//   warps 2-9     epilogue, two warpgroups on alternate units (tcgen05.ld ->
//                 cvt.rn -> swizzled st.shared -> one TMA store per unit).
//   warps 10..    A loaders, LW warpgroups (warp w may only touch TMEM lanes
//                 32 (w % 4) ..): thread L loads its row of the item's k range
//                 with 16-byte LDGs (two items in flight per thread, double-
//                 buffered registers) and stores it with tcgen05.st.32x32b.
//
// Items: the A of a unit arrives in items of (k-chunk kc, layer l).
//   1D (layers = 1): one item per k-chunk; loader warpgroups alternate items.
//   3D (layers = 2 = cbrt(p), p = 8): every k-chunk splits into two k-layers
//       (Alg. 3: warp i holds A_i = m/cbrt(p) x k/cbrt(p)^2 of its
//       layer); loader warpgroup l owns layer l, and both layers' MMAs
//       accumulate into the SAME TMEM accumulator, so the layer reduction of
//       Alg. 3 L378 costs no SMEM traffic at all (the
//       "TMEM route").  The MMA of layer 0 starts as soon as layer 0 landed.
// Batching: G = min(128 / m, 128 / n) entries block-diagonal in one
// 128 x (G n) tile (as tc16), N_mma <= 128 so two accumulators (256 columns)
// and up to 16 A slots (256 columns) share the 512 TMEM columns.
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "kernels.h"
#include "ptx.cuh"
#include "sched.cuh"

namespace kami {
namespace {

constexpr int kTsBaseThreads = 320;  // TMA, MMA, 2 x 4 epilogue warps
constexpr int kTsEpiThreads = 128;
constexpr int kTsMaxStages = 8;
constexpr int kTsMaxSlots = 16;
constexpr int kTsAccCols = 256;  // accumulators live in columns [0, 256), A slots in [256, 512)

struct alignas(64) TsParams {
  CUtensorMap tmB;  // 4-D (Wn, k, n/Wn, batch), box (Wn, Wk, n/Wn, G)
  CUtensorMap tmC;  // 4-D (Wc, m, n/Wc, batch), box (Wc, rows, n/Wc, G)
  const uint16_t* A;
  long long batch, units;
  int m, n, k, G, rows_tile;
  int k_chunks, Wk, Wn, Wc;
  int layers, item_cols, slot_cols, a_slots;
  int ksteps_full, ksteps_last;  // K = 16 steps per chunk
  int N_mma, acc_cols, acc_bufs;
  uint32_t idesc, b_layout, b_lbo, b_sbo, b_kstep;
  uint32_t stage_bytes, tx_bytes;
  int stages;
  uint32_t c_buf_bytes, c_off, bar_off, c_swz_bits;
  int c_bufs;
};

// 16-byte read-only load through L1 (the two 16-byte halves of a sector are
// read by consecutive instructions of the same thread)
__device__ __forceinline__ uint4 ldg16(const void* p) {
  uint4 v;
  asm volatile("ld.global.nc.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p));
  return v;
}

template <int N>
__device__ __forceinline__ void tmem_st_x(uint32_t taddr, const uint32_t* r);
template <>
__device__ __forceinline__ void tmem_st_x<4>(uint32_t t, const uint32_t* r) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1,%2,%3,%4};" ::"r"(t), "r"(r[0]), "r"(r[1]),
               "r"(r[2]), "r"(r[3])
               : "memory");
}
template <>
__device__ __forceinline__ void tmem_st_x<8>(uint32_t t, const uint32_t* r) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(t), "r"(r[0]),
               "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7])
               : "memory");
}
template <>
__device__ __forceinline__ void tmem_st_x<16>(uint32_t t, const uint32_t* r) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], "
      "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(t),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]),
      "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15])
      : "memory");
}
template <>
__device__ __forceinline__ void tmem_st_x<32>(uint32_t t, const uint32_t* r) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], "
      "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
      "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(t),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]),
      "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]),
      "r"(r[17]), "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]),
      "r"(r[25]), "r"(r[26]), "r"(r[27]), "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])
      : "memory");
}

// position of one A item in the CTA's item sequence: unit u (entry group
// grp), k-chunk kc, layer l
struct ItemPos {
  long long u, grp;
  int kc, l;
  __device__ __forceinline__ void next(const TsParams& p, long long ustep) {
    if (++l == p.layers) {
      l = 0;
      if (++kc == p.k_chunks) {
        kc = 0;
        u += ustep;
        grp += ustep;  // (m_tiles = 1: unit = entry group)
      }
    }
  }
};

template <int kOut>
__device__ __forceinline__ void emit8(uint32_t cbase, uint32_t off, uint32_t swz_bits, const uint32_t* v) {
  uint32_t w[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const float lo = __uint_as_float(v[2 * i]), hi = __uint_as_float(v[2 * i + 1]);
    w[i] = kOut ? ptx::pack_bf16x2(lo, hi) : ptx::pack_f16x2(lo, hi);
  }
  ptx::st_shared_v4(cbase + ptx::swz(off, swz_bits), w[0], w[1], w[2], w[3]);
}

template <int kBf16, int kLW>
__global__ void __launch_bounds__(kTsBaseThreads + 128 * kLW, 1)
    kami_tc16_ts_kernel(const __grid_constant__ TsParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + p.bar_off);
  uint64_t* empty = full + kTsMaxStages;
  uint64_t* tfull = empty + kTsMaxStages;
  uint64_t* tempty = tfull + 2;
  uint64_t* afull = tempty + 2;
  uint64_t* aempty = afull + kTsMaxSlots;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(aempty + kTsMaxSlots);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    ptx::prefetch_tmap(&p.tmB);
    ptx::prefetch_tmap(&p.tmC);
    for (int s = 0; s < p.stages; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], kTsEpiThreads / 32);
    }
    for (int j = 0; j < p.a_slots; ++j) {
      ptx::mbar_init(&afull[j], 4);  // the four warps of the loading warpgroup
      ptx::mbar_init(&aempty[j], 1);
    }
    ptx::fence_mbar_init();
    ptx::fence_proxy_async_smem();
  }
  if (warp == 1) ptx::tmem_alloc(tmem_slot, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  const uint32_t smem_base = ptx::smem_u32(smem);

  if (warp == 0) {
    // -------------------------------------------------------- B producer
    if (lane == 0) {
      RingPos r;
      for (long long u = blockIdx.x; u < p.units; u += gridDim.x) {
        const int e0 = (int)(u * p.G);
        for (int kc = 0; kc < p.k_chunks; ++kc, r.next(p.stages)) {
          ptx::mbar_wait(&empty[r.s], r.ph ^ 1);
          ptx::mbar_arrive_expect_tx(&full[r.s], p.tx_bytes);
          ptx::tma_load_4d(smem + r.s * p.stage_bytes, &p.tmB, &full[r.s], 0, kc * p.Wk, 0, e0);
        }
      }
    }
  } else if (warp == 1) {
    // -------------------------------------------------------- MMA issuer
    RingPos rb, ra, rs;
    const uint64_t bdesc0 = ptx::make_smem_desc(smem_base, p.b_lbo, p.b_sbo, p.b_layout);
    const uint32_t stage16 = p.stage_bytes >> 4, bstep16 = p.b_kstep >> 4;
    const uint32_t a_base = tmem_base + kTsAccCols;
    for (long long u = blockIdx.x; u < p.units; u += gridDim.x, ra.next(p.acc_bufs)) {
      ptx::mbar_wait(&tempty[ra.s], ra.ph ^ 1);
      ptx::tc_fence_after();
      const uint32_t d_tmem = tmem_base + ra.s * p.acc_cols;
      for (int kc = 0; kc < p.k_chunks; ++kc, rb.next(p.stages)) {
        ptx::mbar_wait(&full[rb.s], rb.ph);
        const int nst = ((kc == p.k_chunks - 1) ? p.ksteps_last : p.ksteps_full) / p.layers;
        const uint64_t bd = bdesc0 + rb.s * stage16;
        for (int l = 0; l < p.layers; ++l, rs.next(p.a_slots)) {
          ptx::mbar_wait(&afull[rs.s], rs.ph);  // this layer's A rows are in TMEM
          ptx::tc_fence_after();
          if (lane == 0) {
            const uint32_t at = a_base + rs.s * p.slot_cols;
            for (int ks = 0; ks < nst; ++ks)
              ptx::umma_f16_ts(d_tmem, at + 8 * ks, bd + bstep16 * (l * nst + ks), p.idesc, (kc | l | ks) != 0);
            ptx::umma_commit(&aempty[rs.s]);  // A slot free once these MMAs have read it
          }
          __syncwarp();
        }
        if (lane == 0) ptx::umma_commit(&empty[rb.s]);  // B stage free
        __syncwarp();
      }
      if (lane == 0) ptx::umma_commit(&tfull[ra.s]);  // accumulator complete (all layers summed in it)
      __syncwarp();
    }
  } else if (warp >= kTsBaseThreads / 32) {
    // --------------------------------------------------------- A loaders
    const int lw = (warp - kTsBaseThreads / 32) >> 2;  // loader warpgroup
    const int q = warp & 3;                             // TMEM lane quadrant of this warp
    const int L = q * 32 + lane;                        // TMEM lane = tile row
    const int g = L / p.m, r = L - g * p.m;
    const bool row_in_tile = g < p.G;
    const uint32_t t_lane = (uint32_t)(q * 32) << 16;
    const uint32_t a_base = tmem_base + kTsAccCols + t_lane;
    const int nld = p.item_cols >> 3;  // 16-byte loads per item (<= 8)
    // items of this warpgroup: i = lw, lw + kLW, ... of the CTA's sequence
    ItemPos it{blockIdx.x, blockIdx.x, 0, 0};
    RingPos rs;
    for (int j = 0; j < lw; ++j) {
      it.next(p, gridDim.x);
      rs.next(p.a_slots);
    }
    auto load = [&](const ItemPos& x, uint32_t(&v)[32]) {
      const long long e = x.grp * p.G + g;
      const bool ok = row_in_tile && e < p.batch;
      const int c0 = x.kc * p.Wk + x.l * p.item_cols;
      const uint16_t* rowp = p.A + (e * p.m + r) * (long long)p.k + c0;
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        if (j < nld) {
          uint4 w = make_uint4(0, 0, 0, 0);
          if (ok && c0 + 8 * j < p.k) w = ldg16(rowp + 8 * j);
          v[4 * j] = w.x;
          v[4 * j + 1] = w.y;
          v[4 * j + 2] = w.z;
          v[4 * j + 3] = w.w;
        }
      }
    };
    auto store = [&](RingPos& s, const uint32_t(&v)[32]) {
      ptx::mbar_wait(&aempty[s.s], s.ph ^ 1);
      ptx::tc_fence_after();
      const uint32_t ta = a_base + s.s * p.slot_cols;
      switch (nld) {
        case 1: tmem_st_x<4>(ta, v); break;
        case 2: tmem_st_x<8>(ta, v); break;
        case 4: tmem_st_x<16>(ta, v); break;
        default: tmem_st_x<32>(ta, v); break;
      }
      ptx::tmem_wait_st();
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&afull[s.s]);
      for (int j = 0; j < kLW; ++j) s.next(p.a_slots);
    };
    auto advance = [&](ItemPos& x) {
      for (int j = 0; j < kLW; ++j) x.next(p, gridDim.x);
    };
    if (kLW == 1 && nld <= 4 && it.u < p.units) {  // (576-thread CTAs have no registers for it)
      // items of <= 32 columns (16 registers): FOUR in flight per thread.
      // With two, an item's LDG latency (~1500 cycles under load) was exposed
      // once per item (TS 32^3: 1587 cycles per one-item unit against 1094 of
      // HBM time).
      auto load16 = [&](const ItemPos& x, uint32_t(&v)[16]) {
        const long long e = x.grp * p.G + g;
        const bool ok = row_in_tile && e < p.batch;
        const int c0 = x.kc * p.Wk + x.l * p.item_cols;
        const uint16_t* rowp = p.A + (e * p.m + r) * (long long)p.k + c0;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          if (j < nld) {
            uint4 w = make_uint4(0, 0, 0, 0);
            if (ok && c0 + 8 * j < p.k) w = ldg16(rowp + 8 * j);
            v[4 * j] = w.x;
            v[4 * j + 1] = w.y;
            v[4 * j + 2] = w.z;
            v[4 * j + 3] = w.w;
          }
        }
      };
      auto store16 = [&](RingPos& sp_, const uint32_t(&v)[16]) {
        ptx::mbar_wait(&aempty[sp_.s], sp_.ph ^ 1);
        ptx::tc_fence_after();
        const uint32_t ta = a_base + sp_.s * p.slot_cols;
        if (nld == 1) tmem_st_x<4>(ta, v);
        else if (nld == 2) tmem_st_x<8>(ta, v);
        else tmem_st_x<16>(ta, v);
        ptx::tmem_wait_st();
        ptx::tc_fence_before();
        __syncwarp();
        if (lane == 0) ptx::mbar_arrive(&afull[sp_.s]);
        for (int j = 0; j < kLW; ++j) sp_.next(p.a_slots);
      };
      uint32_t q0[16], q1[16], q2[16], q3[16];
      ItemPos p0 = it, p1 = p0, p2;
      advance(p1);
      p2 = p1;
      advance(p2);
      load16(p0, q0);
      if (p1.u < p.units) load16(p1, q1);
      if (p2.u < p.units) load16(p2, q2);
      for (;;) {  // q0..q2 hold p0..p2 at the top of each round
        ItemPos p3 = p2;
        advance(p3);
        if (p3.u < p.units) load16(p3, q3);
        store16(rs, q0);
        if (p1.u >= p.units) break;
        ItemPos p4 = p3;
        advance(p4);
        if (p4.u < p.units) load16(p4, q0);
        store16(rs, q1);
        if (p2.u >= p.units) break;
        ItemPos p5 = p4;
        advance(p5);
        if (p5.u < p.units) load16(p5, q1);
        store16(rs, q2);
        if (p3.u >= p.units) break;
        ItemPos p6 = p5;
        advance(p6);
        if (p6.u < p.units) load16(p6, q2);
        store16(rs, q3);
        if (p4.u >= p.units) break;
        p0 = p4;
        p1 = p5;
        p2 = p6;
      }
    } else if (it.u < p.units) {
      uint32_t va[32], vb[32];
      load(it, va);
      // two items in flight per thread: the next item's loads are issued
      // before the current item is written to TMEM (static buffer roles)
      for (;;) {
        ItemPos nx = it;
        advance(nx);
        if (nx.u < p.units) load(nx, vb);
        store(rs, va);
        if (nx.u >= p.units) break;
        ItemPos n2 = nx;
        advance(n2);
        if (n2.u < p.units) load(n2, va);
        store(rs, vb);
        if (n2.u >= p.units) break;
        it = n2;
      }
    }
  } else {
    // ---------------------------------------------------------- epilogue
    const int wg = (warp - 2) >> 2;
    const int sp = warp & 3;
    const int L = sp * 32 + lane;
    const bool leader = ((warp & 3) == 2) && lane == 0;
    const uint32_t bar_id = 1 + wg;
    int g, r, col_lo, col_hi;
    bool row_ok;
    if (p.G > 1) {
      g = L / p.m;
      r = L - g * p.m;
      row_ok = g < p.G;
      const int glo = (sp * 32) / p.m;
      int ghi = (sp * 32 + 31) / p.m;
      if (ghi > p.G - 1) ghi = p.G - 1;
      col_lo = glo * p.n;
      col_hi = glo < p.G ? (ghi + 1) * p.n : col_lo;
    } else {
      g = 0;
      r = L;
      row_ok = L < p.m;
      col_lo = 0;
      col_hi = (sp * 32 < p.m) ? p.n : 0;
    }
    const int my_lo = g * p.n, my_hi = my_lo + p.n;
    const uint32_t row_bytes = (uint32_t)p.Wc * 2;
    const uint32_t atom_stride = (uint32_t)p.rows_tile * row_bytes;
    const uint32_t rowbase = (uint32_t)(g * (p.n / p.Wc) * p.rows_tile + r) * row_bytes;
    const int wc_shift = 31 - __clz(p.Wc);
    const uint32_t c_smem = smem_base + p.c_off + (uint32_t)wg * p.c_bufs * p.c_buf_bytes;
    uint32_t a = wg, aph = 0;
    RingPos cpos;
    for (long long u = blockIdx.x + (long long)wg * gridDim.x; u < p.units; u += 2ll * gridDim.x) {
      const uint32_t cb = cpos.s;
      const long long e0 = u * p.G;
      if (leader) {
        if (p.c_bufs == 2) ptx::bulk_wait_read<1>();
        else ptx::bulk_wait_read<0>();
      }
      ptx::named_bar_sync(bar_id, kTsEpiThreads);
      ptx::mbar_wait(&tfull[a], aph);
      ptx::tc_fence_after();
      const uint32_t cbase = c_smem + cb * p.c_buf_bytes;
      const bool valid = row_ok && (e0 + g < p.batch);
      const uint32_t t_row = tmem_base + (uint32_t(sp * 32) << 16) + a * p.acc_cols;
      for (int c0 = col_lo; c0 < col_hi; c0 += 64) {
        uint32_t v[64];
        const int left = col_hi - c0;
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
#pragma unroll
        for (int qq = 0; qq < 8; ++qq) {
          const int col = c0 + 8 * qq;
          if (valid && col >= my_lo && col < my_hi && col < col_hi) {
            const uint32_t jc = (uint32_t)(col - my_lo);
            const uint32_t atom = jc >> wc_shift;
            const uint32_t ce = jc & (uint32_t)(p.Wc - 1);
            emit8<kBf16>(cbase, rowbase + atom * atom_stride + ce * 2, p.c_swz_bits, &v[8 * qq]);
          }
        }
      }
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&tempty[a]);
      a += 2;
      if (a >= (uint32_t)p.acc_bufs) {
        a -= p.acc_bufs;
        aph ^= 1;
      }
      cpos.next(p.c_bufs);
      ptx::fence_proxy_async_smem();
      ptx::named_bar_sync(bar_id, kTsEpiThreads);
      if (leader) {
        ptx::tma_store_4d(&p.tmC, smem + p.c_off + (wg * p.c_bufs + cb) * p.c_buf_bytes, 0, 0, 0, (int)e0);
        ptx::bulk_commit();
      }
    }
    if (leader) ptx::bulk_wait<0>();
  }

  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 1) ptx::tmem_dealloc(tmem_base, 512);
}

int ts_atom_bytes(int bytes) { return bytes % 128 == 0 ? 128 : bytes % 64 == 0 ? 64 : bytes % 32 == 0 ? 32 : 0; }
int ts_swz_bits(int atom_bytes) { return atom_bytes == 128 ? 3 : atom_bytes == 64 ? 2 : 1; }
CUtensorMapSwizzle ts_swz_mode(int atom_bytes) {
  return atom_bytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
         : atom_bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                            : CU_TENSOR_MAP_SWIZZLE_32B;
}
uint32_t ts_align(uint32_t x, uint32_t a) { return (x + a - 1) / a * a; }

// Experiment knob (unset in production): KAMI_TS_TUNE="stages,slots,loader_wgs"
struct TsTune {
  int stages = 0, slots = 0, lw = 0;
};
const TsTune& ts_tune() {
  static const TsTune t = [] {
    TsTune r;
    if (const char* e = getenv("KAMI_TS_TUNE")) sscanf(e, "%d,%d,%d", &r.stages, &r.slots, &r.lw);
    return r;
  }();
  return t;
}

constexpr int kTsSmemLimit = 232448;

}  // namespace

kami_status_t tc16_ts_plan(int m, int n, int k, int layers, TsShape* s) {
  // scope: one m-tile, N_mma <= 128 (two accumulators + A slots fit TMEM)
  if (m < 16 || m > 128 || n < 16 || n > 128 || k < 8 || k > 256) return KAMI_ERROR_NOT_SUPPORTED;
  if (m % 16 || n % 16 || k % 8) return KAMI_ERROR_NOT_SUPPORTED;
  if (layers != 1 && layers != 2) return KAMI_ERROR_INVALID_VALUE;
  const int g1 = 128 / m, g2 = 128 / n;
  s->G = g1 < g2 ? g1 : g2;
  s->N_mma = s->G * n;
  const int kpad = (k + 15) / 16 * 16;
  const int wk_b = ts_atom_bytes(kpad * 2), wn_b = ts_atom_bytes(n * 2);
  if (!wk_b || !wn_b) return KAMI_ERROR_NOT_SUPPORTED;
  s->Wk = wk_b / 2;
  s->Wn = wn_b / 2;
  s->Wc = s->Wn;
  s->k_chunks = (kpad + s->Wk - 1) / s->Wk;
  s->ksteps_full = s->Wk / 16;
  s->ksteps_last = (kpad - (s->k_chunks - 1) * s->Wk) / 16;
  // 3D: each k-chunk splits into `layers` k-layers of whole K = 16 steps
  if (s->ksteps_full % layers || s->ksteps_last % layers) return KAMI_ERROR_NOT_SUPPORTED;
  s->layers = layers;
  s->item_cols = s->Wk / layers;    // 16-bit A elements per item
  s->slot_cols = s->item_cols / 2;  // 32-bit TMEM columns per item
  int slots = 256 / s->slot_cols;
  if (slots > kTsMaxSlots) slots = kTsMaxSlots;
  if (ts_tune().slots > 0 && ts_tune().slots < slots) slots = ts_tune().slots;
  s->a_slots = slots;
  s->loader_wgs = layers == 2 ? 2 : (ts_tune().lw == 2 ? 2 : 1);
  s->acc_cols = s->N_mma <= 32 ? 32 : s->N_mma <= 64 ? 64 : 128;
  s->stage_bytes = ts_align((uint32_t)(s->G * n) * wk_b, 1024);
  s->c_buf_bytes = ts_align((uint32_t)(s->G * n * m * 2), 1024);
  s->c_bufs = (4 * s->c_buf_bytes <= 64 * 1024) ? 2 : 1;
  const int budget = kTsSmemLimit - 2048;
  int st = (budget - (int)(2 * s->c_bufs * s->c_buf_bytes)) / (int)s->stage_bytes;
  if (st > kTsMaxStages) st = kTsMaxStages;
  // B bytes in flight: ~64 KB of B (A adds its own in registers); >= 3 stages
  int cap = (64 * 1024) / (int)s->stage_bytes;
  if (cap < 3) cap = 3;
  if (st > cap) st = cap;
  if (ts_tune().stages > 0 && st > ts_tune().stages) st = ts_tune().stages;
  if (st < 2) return KAMI_ERROR_NOT_SUPPORTED;
  s->stages = st;
  s->smem_bytes = s->stages * s->stage_bytes + 2 * s->c_bufs * s->c_buf_bytes + 2048;
  return KAMI_SUCCESS;
}

kami_status_t tc16_ts_launch(int m, int n, int k, long long batch, bool bf16, int layers, const void* A,
                             const void* B, void* C, cudaStream_t stream) {
  TsShape s;
  kami_status_t st = tc16_ts_plan(m, n, k, layers, &s);
  if (st != KAMI_SUCCESS) return st;
  PFN_encodeTiled enc = get_encode_tiled();
  if (!enc) return KAMI_ERROR_CUDA;
  TsParams p;
  memset(&p, 0, sizeof(p));
  p.A = static_cast<const uint16_t*>(A);
  p.batch = batch;
  p.m = m;
  p.n = n;
  p.k = k;
  p.G = s.G;
  p.rows_tile = m;
  p.k_chunks = s.k_chunks;
  p.Wk = s.Wk;
  p.Wn = s.Wn;
  p.Wc = s.Wc;
  p.layers = s.layers;
  p.item_cols = s.item_cols;
  p.slot_cols = s.slot_cols;
  p.a_slots = s.a_slots;
  p.ksteps_full = s.ksteps_full;
  p.ksteps_last = s.ksteps_last;
  p.N_mma = s.N_mma;
  p.acc_cols = s.acc_cols;
  p.acc_bufs = 2;
  const int wn_b = s.Wn * 2, wc_b = s.Wc * 2;
  p.idesc = ptx::make_idesc_f16(bf16 ? 1 : 0, 128, s.N_mma, /*a K-major*/ 0, /*b MN-major*/ 1);
  p.b_layout = ptx::umma_layout_code(wn_b);
  p.b_sbo = 8 * wn_b;
  p.b_lbo = s.Wk * wn_b;
  p.b_kstep = 2 * p.b_sbo;  // one K = 16 step = 16 B rows = two 8-row groups
  p.stage_bytes = s.stage_bytes;
  p.tx_bytes = (uint32_t)(s.Wk * 2 * n * s.G);
  p.stages = s.stages;
  p.c_buf_bytes = s.c_buf_bytes;
  p.c_bufs = s.c_bufs;
  p.c_off = s.stages * s.stage_bytes;
  p.bar_off = p.c_off + 2 * s.c_bufs * s.c_buf_bytes;
  p.c_swz_bits = ts_swz_bits(wc_b);
  p.units = (batch + s.G - 1) / s.G;
  const CUtensorMapDataType dt = bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16;
  {  // B: (Wn, k, n/Wn, batch)
    cuuint64_t dims[4] = {(cuuint64_t)s.Wn, (cuuint64_t)k, (cuuint64_t)(n / s.Wn), (cuuint64_t)batch};
    cuuint64_t strides[3] = {(cuuint64_t)n * 2, (cuuint64_t)wn_b, (cuuint64_t)k * n * 2};
    cuuint32_t box[4] = {(cuuint32_t)s.Wn, (cuuint32_t)s.Wk, (cuuint32_t)(n / s.Wn), (cuuint32_t)s.G};
    cuuint32_t es[4] = {1, 1, 1, 1};
    if (enc(&p.tmB, dt, 4, const_cast<void*>(B), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
            ts_swz_mode(wn_b), CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  {  // C: (Wc, m, n/Wc, batch)
    cuuint64_t dims[4] = {(cuuint64_t)s.Wc, (cuuint64_t)m, (cuuint64_t)(n / s.Wc), (cuuint64_t)batch};
    cuuint64_t strides[3] = {(cuuint64_t)n * 2, (cuuint64_t)wc_b, (cuuint64_t)m * n * 2};
    cuuint32_t box[4] = {(cuuint32_t)s.Wc, (cuuint32_t)m, (cuuint32_t)(n / s.Wc), (cuuint32_t)s.G};
    cuuint32_t es[4] = {1, 1, 1, 1};
    if (enc(&p.tmC, dt, 4, C, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, ts_swz_mode(wc_b),
            CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  long long grid = p.units < sms ? p.units : sms;
  grid = apply_grid_cap(grid);
  const size_t smem = s.smem_bytes;
  const char* name;
  if (s.loader_wgs == 2) {
    auto fn = bf16 ? kami_tc16_ts_kernel<1, 2> : kami_tc16_ts_kernel<0, 2>;
    cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    fn<<<(unsigned)grid, kTsBaseThreads + 256, smem, stream>>>(p);
    name = layers == 2 ? (bf16 ? "kami_tc16_ts_3d<bf16>" : "kami_tc16_ts_3d<f16>")
                       : (bf16 ? "kami_tc16_ts_1d<bf16,lw2>" : "kami_tc16_ts_1d<f16,lw2>");
  } else {
    auto fn = bf16 ? kami_tc16_ts_kernel<1, 1> : kami_tc16_ts_kernel<0, 1>;
    cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    fn<<<(unsigned)grid, kTsBaseThreads + 128, smem, stream>>>(p);
    name = bf16 ? "kami_tc16_ts_1d<bf16>" : "kami_tc16_ts_1d<f16>";
  }
  set_last_kernel(name);
  return cudaGetLastError() == cudaSuccess ? KAMI_SUCCESS : KAMI_ERROR_CUDA;
}

}  // namespace kami
