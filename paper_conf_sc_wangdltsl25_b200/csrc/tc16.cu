// tc16.cu -- FP16/BF16 batched small GEMM on 5th-generation tensor cores
// (tcgen05 + TMEM + TMA), sm_100a.  Hot path of BASELINE.json configs 0, 1,
// 3 and 4.
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
//                   the z-th K=16 slice (k-slicing, Sec. 4.7).
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
//   warp 1     MMA issuer (one lane) + TMEM allocator: tcgen05.mma
//              kind::f16, accumulators double/quad-buffered in TMEM,
//              tcgen05.commit -> empty[s] (frees the stage) and tfull[a].
//   warps 2-9  epilogue, two warpgroups on alternate units: tcgen05.ld
//              32x32b, cvt.rn to fp16/bf16, swizzled conflict-free st.shared
//              into a C staging tile, one TMA tensor store per unit.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstring>

#include "kernels.h"
#include "ptx.cuh"

namespace kami {

namespace {

constexpr int kThreads = 320;  // 10 warps: TMA, MMA, 2 x 4 epilogue
constexpr int kEpiThreads = 128;
constexpr int kMaxStages = 8;
constexpr int kMaxAcc = 4;

struct alignas(64) Tc16Params {
  CUtensorMap tmA;  // 3-D (k, m, batch), box (Wk, rowsA, G)
  CUtensorMap tmB;  // 4-D (Wn, k, n/Wn, batch), box (Wn, Wk, n/Wn, G)
  CUtensorMap tmC;  // 4-D (Wc, m, n/Wc, batch), box (Wc, rows_tile, n/Wc, G)
  long long batch;
  long long units;
  int m, n, k;
  int G, m_tiles, rows_tile;
  int k_chunks, Wk, Wn, Wc;
  int ksteps_full, ksteps_last;
  int N_mma;
  uint32_t idesc;
  uint32_t a_layout, b_layout, c_swz_bits;
  uint32_t a_sbo, b_lbo, b_sbo;
  uint32_t a_region, stage_bytes, tx_bytes;
  int stages;
  int acc_cols, acc_bufs, tmem_cols;
  uint32_t c_buf_bytes;
  int c_bufs;
  uint32_t c_off;    // byte offset of C staging
  uint32_t bar_off;  // byte offset of barriers
};

template <bool kBF16>
__global__ void __launch_bounds__(kThreads, 1) kami_tc16_1d_kernel(const __grid_constant__ Tc16Params p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1024-byte alignment for the 128B swizzle atoms
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + p.bar_off);
  uint64_t* empty = full + kMaxStages;
  uint64_t* tfull = empty + kMaxStages;
  uint64_t* tempty = tfull + kMaxAcc;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + kMaxAcc);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    ptx::prefetch_tmap(&p.tmA);
    ptx::prefetch_tmap(&p.tmB);
    ptx::prefetch_tmap(&p.tmC);
    for (int s = 0; s < p.stages; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < p.acc_bufs; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], kEpiThreads / 32);
    }
    ptx::fence_mbar_init();
    ptx::fence_proxy_async_smem();
  }
  if (warp == 1) ptx::tmem_alloc(tmem_slot, p.tmem_cols);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  const uint32_t smem_base = ptx::smem_u32(smem);

  if (warp == 0) {
    // ------------------------------------------------------------ producer
    if (lane == 0) {
      uint32_t it = 0;
      for (long long u = blockIdx.x; u < p.units; u += gridDim.x) {
        const long long grp = u / p.m_tiles;
        const int mt = (int)(u - grp * p.m_tiles);
        const int e0 = (int)(grp * p.G);
        for (int kc = 0; kc < p.k_chunks; ++kc, ++it) {
          const uint32_t s = it % p.stages;
          const uint32_t ph = (it / p.stages) & 1;
          ptx::mbar_wait(&empty[s], ph ^ 1);
          ptx::mbar_arrive_expect_tx(&full[s], p.tx_bytes);
          uint8_t* sa = smem + s * p.stage_bytes;
          uint8_t* sb = sa + p.a_region;
          ptx::tma_load_3d(sa, &p.tmA, &full[s], kc * p.Wk, mt * 128, e0);
          ptx::tma_load_4d(sb, &p.tmB, &full[s], 0, kc * p.Wk, 0, e0);
        }
      }
    }
  } else if (warp == 1) {
    // ---------------------------------------------------------- MMA issuer
    uint32_t it = 0, acc_it = 0;
    for (long long u = blockIdx.x; u < p.units; u += gridDim.x, ++acc_it) {
      const uint32_t a = acc_it % p.acc_bufs;
      const uint32_t aph = (acc_it / p.acc_bufs) & 1;
      ptx::mbar_wait(&tempty[a], aph ^ 1);
      ptx::tc_fence_after();
      const uint32_t d_tmem = tmem_base + a * p.acc_cols;
      for (int kc = 0; kc < p.k_chunks; ++kc, ++it) {
        const uint32_t s = it % p.stages;
        const uint32_t ph = (it / p.stages) & 1;
        ptx::mbar_wait(&full[s], ph);
        ptx::tc_fence_after();
        if (lane == 0) {
          const uint32_t sa = smem_base + s * p.stage_bytes;
          const uint32_t sb = sa + p.a_region;
          const int nsteps = (kc == p.k_chunks - 1) ? p.ksteps_last : p.ksteps_full;
          for (int ks = 0; ks < nsteps; ++ks) {
            // A: K-major, 16 elements = 32 bytes further along the swizzled row
            const uint64_t adesc = ptx::make_smem_desc(sa + ks * 32, 16, p.a_sbo, p.a_layout);
            // B: N-major, 16 K-rows further = 2 core-row groups
            const uint64_t bdesc = ptx::make_smem_desc(sb + ks * 2 * p.b_sbo, p.b_lbo, p.b_sbo, p.b_layout);
            ptx::umma_f16_ss(d_tmem, adesc, bdesc, p.idesc, (kc | ks) != 0);
          }
          ptx::umma_commit(&empty[s]);  // stage s may be refilled once these MMAs retire
        }
        __syncwarp();
      }
      if (lane == 0) ptx::umma_commit(&tfull[a]);  // accumulator a complete
      __syncwarp();
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
      row_ok = L < p.rows_tile;
      col_lo = 0;
      col_hi = (sp * 32 < p.rows_tile) ? p.n : 0;
    }
    const int my_lo = g * p.n, my_hi = my_lo + p.n;
    const uint32_t row_bytes = (uint32_t)p.Wc * 2;
    const uint32_t atom_stride = (uint32_t)p.rows_tile * row_bytes;
    const uint32_t rowbase = (uint32_t)(g * (p.n / p.Wc) * p.rows_tile + r) * row_bytes;
    const int wc_shift = p.Wc == 64 ? 6 : p.Wc == 32 ? 5 : 4;
    const uint32_t c_smem = smem_base + p.c_off + (uint32_t)wg * p.c_bufs * p.c_buf_bytes;
    uint32_t i = wg, local = 0;
    for (long long u = blockIdx.x + (long long)wg * gridDim.x; u < p.units;
         u += 2ll * gridDim.x, i += 2, ++local) {
      const long long grp = u / p.m_tiles;
      const int mt = (int)(u - grp * p.m_tiles);
      const long long e0 = grp * p.G;
      const uint32_t a = i % p.acc_bufs;
      const uint32_t aph = (i / p.acc_bufs) & 1;
      const uint32_t cb = local % p.c_bufs;
      const bool valid = row_ok && (e0 + g < p.batch) && (p.G > 1 || mt * 128 + L < p.m);
      // the TMA store that last read staging buffer cb must be done reading
      if (leader) {
        if (p.c_bufs == 2) ptx::bulk_wait_read<1>();
        else ptx::bulk_wait_read<0>();
      }
      ptx::named_bar_sync(bar_id, kEpiThreads);
      ptx::mbar_wait(&tfull[a], aph);
      ptx::tc_fence_after();
      const uint32_t t_row = tmem_base + (uint32_t(sp * 32) << 16) + a * p.acc_cols;
      const uint32_t cbase = c_smem + cb * p.c_buf_bytes;
      for (int c0 = col_lo; c0 < col_hi; c0 += 64) {
        uint32_t v[64];
        // issue both TMEM loads, then one wait (never read past col_hi)
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
        for (int q = 0; q < 8; ++q) {
          const int col = c0 + 8 * q;
          if (valid && col >= my_lo && col < my_hi && col < col_hi) {
            const uint32_t jc = (uint32_t)(col - my_lo);
            const uint32_t atom = jc >> wc_shift;
            const uint32_t ce = jc & (uint32_t)(p.Wc - 1);
            const uint32_t off = ptx::swz(rowbase + atom * atom_stride + ce * 2, p.c_swz_bits);
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
            ptx::st_shared_v4(cbase + off, w0, w1, w2, w3);
          }
        }
      }
      // accumulator a may be overwritten by the next MMA chain
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&tempty[a]);
      // make the generic-proxy smem writes visible to the TMA engine
      ptx::fence_proxy_async_smem();
      ptx::named_bar_sync(bar_id, kEpiThreads);
      if (leader) {
        ptx::tma_store_4d(&p.tmC, smem + p.c_off + (wg * p.c_bufs + cb) * p.c_buf_bytes, 0, mt * 128, 0, (int)e0);
        ptx::bulk_commit();
      }
    }
    if (leader) ptx::bulk_wait<0>();
  }

  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 1) ptx::tmem_dealloc(tmem_base, p.tmem_cols);
}

// ------------------------------------------------------------------- host

int pick_atom(int elems) {  // largest swizzle atom width (elements) dividing elems
  if (elems % 64 == 0) return 64;
  if (elems % 32 == 0) return 32;
  return 16;
}
int swz_bits_for(int atom_elems) { return atom_elems == 64 ? 3 : atom_elems == 32 ? 2 : 1; }
CUtensorMapSwizzle swz_mode_for(int atom_elems) {
  return atom_elems == 64 ? CU_TENSOR_MAP_SWIZZLE_128B
         : atom_elems == 32 ? CU_TENSOR_MAP_SWIZZLE_64B
                            : CU_TENSOR_MAP_SWIZZLE_32B;
}
uint32_t align_up(uint32_t x, uint32_t a) { return (x + a - 1) / a * a; }
int pow2_ceil(int x) {
  int p = 32;
  while (p < x) p <<= 1;
  return p;
}

constexpr int kSmemLimit = 232448;  // 227 KB opt-in per CTA

}  // namespace

kami_status_t tc16_plan_shape(int m, int n, int k, Tc16Shape* s) {
  s->G = 1;
  if (m <= 128) {
    int g1 = 128 / m, g2 = 256 / n;
    s->G = g1 < g2 ? g1 : g2;
    if (s->G < 1) s->G = 1;
  }
  s->m_tiles = (s->G > 1 || m <= 128) ? 1 : (m + 127) / 128;
  s->rows_tile = m < 128 ? m : 128;
  const int kpad = (k + 15) / 16 * 16;
  s->Wk = pick_atom(kpad);
  s->Wn = pick_atom(n);
  s->Wc = s->Wn;
  s->k_chunks = (kpad + s->Wk - 1) / s->Wk;
  s->N_mma = s->G > 1 ? s->G * n : n;
  const uint32_t a_region = align_up(128u * s->Wk * 2, 1024);
  const uint32_t b_region = align_up((uint32_t)s->N_mma * s->Wk * 2, 1024);
  s->stage_bytes = a_region + b_region;
  s->c_buf_bytes = align_up((uint32_t)s->G * n * s->rows_tile * 2, 1024);
  // two epilogue warpgroups, each with c_bufs staging tiles
  s->c_bufs = (4 * s->c_buf_bytes <= 64 * 1024) ? 2 : 1;
  const int budget = kSmemLimit - 1024 /*align slack*/ - 1024 /*barriers*/;
  int st = (budget - (int)(2 * s->c_bufs * s->c_buf_bytes)) / (int)s->stage_bytes;
  if (st > kMaxStages) st = kMaxStages;
  s->stages = st;
  s->smem_bytes = s->stages * s->stage_bytes + 2 * s->c_bufs * s->c_buf_bytes + 1024 + 1024;
  s->acc_cols = pow2_ceil(s->N_mma);
  s->acc_bufs = 512 / s->acc_cols;
  if (s->acc_bufs > kMaxAcc) s->acc_bufs = kMaxAcc;
  s->units = 0;
  return st >= 2 ? KAMI_SUCCESS : KAMI_ERROR_NOT_SUPPORTED;
}

kami_status_t tc16_launch(int m, int n, int k, long long batch, bool bf16, const void* A, const void* B, void* C,
                          cudaStream_t stream, int max_ctas) {
  Tc16Shape s;
  kami_status_t st = tc16_plan_shape(m, n, k, &s);
  if (st != KAMI_SUCCESS) return st;
  PFN_encodeTiled enc = get_encode_tiled();
  if (!enc) return KAMI_ERROR_CUDA;

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
  const int kpad = (k + 15) / 16 * 16;
  p.ksteps_full = s.Wk / 16;
  p.ksteps_last = (kpad - (s.k_chunks - 1) * s.Wk) / 16;
  p.N_mma = s.N_mma;
  p.idesc = ptx::make_idesc_f16(bf16 ? 1 : 0, 128, s.N_mma, /*a MN-major*/ 0, /*b MN-major*/ 1);
  p.a_layout = ptx::umma_layout_code(s.Wk * 2);
  p.b_layout = ptx::umma_layout_code(s.Wn * 2);
  p.c_swz_bits = swz_bits_for(s.Wc);
  p.a_sbo = 8 * s.Wk * 2;          // 8 rows of the K-major A tile
  p.b_sbo = 8 * s.Wn * 2;          // 8 K-rows of one N-atom
  p.b_lbo = s.Wk * s.Wn * 2;       // next N-atom (next 64/32/16 columns)
  p.a_region = align_up(128u * s.Wk * 2, 1024);
  p.stage_bytes = s.stage_bytes;
  const int G = s.G;
  const int rowsA = s.rows_tile;
  p.tx_bytes = (uint32_t)(s.Wk * rowsA * G * 2) + (uint32_t)(s.Wn * s.Wk * (n / s.Wn) * G * 2);
  p.stages = s.stages;
  p.acc_cols = s.acc_cols;
  p.acc_bufs = s.acc_bufs;
  p.tmem_cols = s.acc_cols * s.acc_bufs;
  p.c_buf_bytes = s.c_buf_bytes;
  p.c_bufs = s.c_bufs;
  p.c_off = s.stages * s.stage_bytes;
  p.bar_off = p.c_off + 2 * s.c_bufs * s.c_buf_bytes;
  const long long groups = (batch + G - 1) / G;
  p.units = groups * s.m_tiles;

  const CUtensorMapDataType dt = bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16;
  {  // A: (k, m, batch)
    cuuint64_t dims[3] = {(cuuint64_t)k, (cuuint64_t)m, (cuuint64_t)batch};
    cuuint64_t strides[2] = {(cuuint64_t)k * 2, (cuuint64_t)m * k * 2};
    cuuint32_t box[3] = {(cuuint32_t)s.Wk, (cuuint32_t)rowsA, (cuuint32_t)G};
    cuuint32_t es[3] = {1, 1, 1};
    if (enc(&p.tmA, dt, 3, const_cast<void*>(A), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
            swz_mode_for(s.Wk), CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  {  // B: (Wn, k, n/Wn, batch)
    cuuint64_t dims[4] = {(cuuint64_t)s.Wn, (cuuint64_t)k, (cuuint64_t)(n / s.Wn), (cuuint64_t)batch};
    cuuint64_t strides[3] = {(cuuint64_t)n * 2, (cuuint64_t)s.Wn * 2, (cuuint64_t)k * n * 2};
    cuuint32_t box[4] = {(cuuint32_t)s.Wn, (cuuint32_t)s.Wk, (cuuint32_t)(n / s.Wn), (cuuint32_t)G};
    cuuint32_t es[4] = {1, 1, 1, 1};
    if (enc(&p.tmB, dt, 4, const_cast<void*>(B), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
            swz_mode_for(s.Wn), CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  {  // C: (Wc, m, n/Wc, batch)
    cuuint64_t dims[4] = {(cuuint64_t)s.Wc, (cuuint64_t)m, (cuuint64_t)(n / s.Wc), (cuuint64_t)batch};
    cuuint64_t strides[3] = {(cuuint64_t)n * 2, (cuuint64_t)s.Wc * 2, (cuuint64_t)m * n * 2};
    cuuint32_t box[4] = {(cuuint32_t)s.Wc, (cuuint32_t)s.rows_tile, (cuuint32_t)(n / s.Wc), (cuuint32_t)G};
    cuuint32_t es[4] = {1, 1, 1, 1};
    if (enc(&p.tmC, dt, 4, C, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, swz_mode_for(s.Wc),
            CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }

  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  long long grid = p.units < sms ? p.units : sms;
  if (max_ctas > 0 && grid > max_ctas) grid = max_ctas;
  const size_t smem = s.smem_bytes;
  if (bf16) {
    cudaFuncSetAttribute(kami_tc16_1d_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    kami_tc16_1d_kernel<true><<<(unsigned)grid, kThreads, smem, stream>>>(p);
    set_last_kernel("kami_tc16_1d_kernel<bf16>");
  } else {
    cudaFuncSetAttribute(kami_tc16_1d_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    kami_tc16_1d_kernel<false><<<(unsigned)grid, kThreads, smem, stream>>>(p);
    set_last_kernel("kami_tc16_1d_kernel<f16>");
  }
  return cudaGetLastError() == cudaSuccess ? KAMI_SUCCESS : KAMI_ERROR_CUDA;
}

}  // namespace kami
