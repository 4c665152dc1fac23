// tc16_xt.cu -- thin-m 16-bit batched GEMM on tcgen05 through the transposed
// product C^T = B^T A^T (SURVEY.md 8(a) rows a2-a6 for the thin tiles of
// BASELINE configs[4]; Sec. 4.2, the 1D schedule).
//
// For m <= 32 the block-diagonal packing of tc16.cu puts G = min(128/m,
// 256/n) entries on one 128-lane tile, and with n >= 64 that is 2-4 entries:
// most of the tile's lanes and TMEM columns idle, and a unit moves too few
// bytes to cover its fixed cost (bf16 16x128x16: 0.47-0.55 of the HBM
// roofline).  Transposed, the roles turn: M = n (128 TMEM lanes = 128 columns
// of C), N = m (16 or 32 TMEM columns per entry), so one accumulator holds E
// entries side by side -- E MMAs of 128 x m x 16 per K step, one per entry,
// each writing its own TMEM columns.  The MMA's A operand is B^T: B's k x 64
// row-major boxes are exactly the MN-major 128-byte-swizzled atoms (a_major =
// MN in the instruction descriptor); its B operand is A^T = A read K-major.
// The KAMI-1D reading is unchanged: the four sub-partition tensor cores each
// own a 32-lane slice of the accumulator (local), and the entry's A -- the
// operand every slice needs -- is the one broadcast through shared memory.
//
// Warps: 0 producer (two TMA boxes per unit: E entries' B tiles, E entries'
// A), 1 MMA issuer + TMEM allocator, 2-5 and 6-9 two epilogue warpgroups on
// alternate units (warpgroup w always drains accumulator w).  Epilogue thread
// = one column n of C: tcgen05.ld of 64 accumulator columns (4 or 2 entries)
// per wait, cvt.rn, 16-bit stores into a staging tile in C's row-major box
// layout, one TMA store per unit.
// A unit = (group of E entries, 128-column tile of n) -- a *head* tile, P = 1
// -- or, for the 64-column pieces (n = 64, and the last 64 columns of
// n = 192), a *pair* tile, P = 2: lanes 0-63 hold entry 2g's 64 columns and
// lanes 64-127 entry 2g+1's, the MMA's N is 2m (A^T of both entries stacked),
// and only the two diagonal m-column blocks are kept (the block-diagonal
// packing of tc16.cu, in the transposed space).  Head and pair tiles have the
// same shared-memory geometry: 2E atoms of k x 64 for B, and the staging tile
// [2E][m][64] for C; only the boxes, N and the TMEM column of a lane half
// differ.  n = 192 runs three units per 2E entries: two heads, one pair.
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstring>

#include "kernels.h"
#include "ptx.cuh"
#include "sched.cuh"

namespace kami {
namespace {

constexpr int kXtThreads = 320;  // producer, MMA, two epilogue warpgroups
constexpr int kXtMaxStages = 8;
constexpr int kXtSmemLimit = 232448;

struct alignas(64) XtParams {
  CUtensorMap tmA;  // A (k, m, batch), box (k, m, E), 2k-byte swizzle
  CUtensorMap tmB;  // B (64, k, n/64, batch), box (64, k, 2, E), 128-byte swizzle
  CUtensorMap tmC;  // C (64, m, n/64, batch), box (64, m, 2, E), no swizzle
  CUtensorMap tmA2, tmB2, tmC2;  // pair tiles: boxes (k, m, 2E), (64, k, 1, 2E), (64, m, 1, 2E)
  int mode;         // 0: n % 128 == 0 (heads), 1: n == 64 (pairs), 2: n == 192 (two heads + one pair per 2E)
  uint32_t idesc2, tx2;
  int m, n, k, E, NT;
  long long batch, units;
  int stages;
  uint32_t stage_bytes, a_off, ent_b, ent_a;
  uint32_t c_off, c_buf, bar_off;
  uint32_t idesc, tx;
  int acc_cols, acc_bufs;  // accumulators of acc_cols TMEM columns (2 or 4)
};

// unit (grp, mt) -> pair tile?, first entry, first 64-column atom of n
struct XtUnit {
  bool pair;
  int e0, atom;
};
__device__ __forceinline__ XtUnit xt_unit(const XtParams& p, long long grp, int mt) {
  if (p.mode == 0) return {false, (int)(grp * p.E), 2 * mt};
  if (p.mode == 1) return {true, (int)(grp * 2 * p.E), 0};
  if (mt < 2) return {false, (int)(grp * 2 * p.E) + mt * p.E, 0};
  return {true, (int)(grp * 2 * p.E), 2};
}

template <bool kBF16, int kM>
__global__ void __launch_bounds__(kXtThreads, 1) kami_tc16_xt_kernel(const __grid_constant__ XtParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + p.bar_off);
  uint64_t* empty = full + kXtMaxStages;
  uint64_t* tfull = empty + kXtMaxStages;
  uint64_t* tempty = tfull + 4;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 4);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    ptx::prefetch_tmap(&p.tmA);
    ptx::prefetch_tmap(&p.tmB);
    ptx::prefetch_tmap(&p.tmC);
    if (p.mode) {
      ptx::prefetch_tmap(&p.tmA2);
      ptx::prefetch_tmap(&p.tmB2);
      ptx::prefetch_tmap(&p.tmC2);
    }
    for (int s = 0; s < p.stages; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < p.acc_bufs; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], 4);  // the four warps of the epilogue warpgroup draining it
    }
    ptx::fence_mbar_init();
  }
  if (warp == 1) ptx::tmem_alloc(tmem_slot, p.acc_bufs * p.acc_cols);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  const uint32_t smem_base = ptx::smem_u32(smem);

  if (warp == 0) {
    // ------------------------------------------------------------ producer
    if (lane == 0) {
      RingPos r;
      UnitIter ui(blockIdx.x, gridDim.x, p.NT);
      for (long long u = blockIdx.x; u < p.units; u += gridDim.x, ui.next(), r.next(p.stages)) {
        ptx::mbar_wait(&empty[r.s], r.ph ^ 1);
        const XtUnit U = xt_unit(p, ui.grp, ui.mt);
        ptx::mbar_arrive_expect_tx(&full[r.s], U.pair ? p.tx2 : p.tx);
        uint8_t* st = smem + r.s * p.stage_bytes;
        // B^T (the MMA's A operand) and A^T (its B operand)
        ptx::tma_load_4d(st, U.pair ? &p.tmB2 : &p.tmB, &full[r.s], 0, 0, U.atom, U.e0);
        ptx::tma_load_3d(st + p.a_off, U.pair ? &p.tmA2 : &p.tmA, &full[r.s], 0, 0, U.e0);
      }
    }
  } else if (warp == 1) {
    // ---------------------------------------------------------- MMA issuer
    RingPos r, ra;
    const uint32_t a_sw = (uint32_t)p.k * 2u;  // A rows: 2k bytes, 2k-byte swizzle
    const int ksteps = p.k / 16;
    UnitIter ui(blockIdx.x, gridDim.x, p.NT);
    for (long long u = blockIdx.x; u < p.units; u += gridDim.x, r.next(p.stages), ra.next(p.acc_bufs), ui.next()) {
      const bool pair = xt_unit(p, ui.grp, ui.mt).pair;
      const int P = pair ? 2 : 1;  // entries per 128-lane tile
      ptx::mbar_wait(&tempty[ra.s], ra.ph ^ 1);
      ptx::tc_fence_after();
      ptx::mbar_wait(&full[r.s], r.ph);
      ptx::tc_fence_after();
      if (lane == 0) {
        const uint32_t sb = smem_base + r.s * p.stage_bytes, sa = sb + p.a_off;
        const uint32_t idesc = pair ? p.idesc2 : p.idesc;
        for (int e = 0; e < p.E; ++e) {
          const uint32_t d = tmem_base + ra.s * p.acc_cols + e * P * p.m;
          for (int ks = 0; ks < ksteps; ++ks) {
            // B^T (MN-major): two 64-column atoms k*128 bytes apart, a K step = 16 rows of 128 B
            const uint64_t ad = ptx::make_smem_desc(sb + e * p.ent_b + ks * 2048, (uint32_t)p.k * 128, 1024, 2);
            // A^T (K-major): m rows of 2k bytes, a K step = 32 bytes along the row
            // (pair tiles: the two entries' A^T rows stacked, N = 2m)
            const uint64_t bd = ptx::make_smem_desc(sa + e * P * p.ent_a + ks * 32, 16, 8 * a_sw,
                                                    ptx::umma_layout_code((int)a_sw));
            ptx::umma_f16_ss(d, ad, bd, idesc, ks != 0);
          }
        }
        ptx::umma_commit(&empty[r.s]);
        ptx::umma_commit(&tfull[ra.s]);
      }
      __syncwarp();
    }
  } else {
    // ------------------------------------------------------------ epilogue
    // warpgroup wg takes the CTA's units i = wg, wg + 2, ...; unit i lives in
    // accumulator i mod acc_bufs (the MMA's ring), phase (i / acc_bufs) & 1
    const int wg = (warp - 2) >> 2;
    const int sp = warp & 3;          // TMEM sub-partition of this warp
    const int col = sp * 32 + lane;   // this thread's column of the 128-column tile
    const int half = col >> 6;        // head tiles: the 64-column atom; pair tiles: the entry of the pair
    const uint32_t col_b = (uint32_t)(col & 63) * 2u;
    const bool leader = (warp & 3) == 2 && lane == 0;
    const uint32_t cbuf = smem_base + p.c_off + wg * p.c_buf;
    constexpr int per = 64 / kM;      // entries per TMEM load batch (64 columns)
    uint32_t li = wg;  // the CTA-local unit index i
    UnitIter ui(blockIdx.x + (long long)wg * gridDim.x, 2ll * gridDim.x, p.NT);
    for (long long u = blockIdx.x + (long long)wg * gridDim.x; u < p.units; u += 2ll * gridDim.x, ui.next(), li += 2) {
      const uint32_t acc = li % (uint32_t)p.acc_bufs, ph = (li / (uint32_t)p.acc_bufs) & 1u;
      const XtUnit U = xt_unit(p, ui.grp, ui.mt);
      const int P = U.pair ? 2 : 1;
      const long long e0 = U.e0;
      const int ng = (int)((p.batch - e0 + P - 1) / P);  // live groups of P entries
      const int ne = ng < p.E ? ng : p.E;
      // this lane's first accumulator column: head tiles (g m), pair tiles (2 g m + half m)
      const int cs = P * kM;
      const int c_half = U.pair ? half * kM : 0;
      // this warpgroup's previous store is done reading the staging tile
      if (leader) ptx::bulk_wait_read<0>();
      ptx::named_bar_sync(1 + wg, 128);
      ptx::mbar_wait(&tfull[acc], ph);
      ptx::tc_fence_after();
      const uint32_t t_row = tmem_base + (uint32_t(sp * 32) << 16) + acc * p.acc_cols;
      for (int e1 = 0; e1 < ne; e1 += per) {
        uint32_t v[64];
        // one wait per 64 columns: a wait per entry serialised the TMEM load latency
        // groups e1 .. e1 + per - 1: kM columns each (c_half is warp-uniform)
#pragma unroll
        for (int gq = 0; gq < per; ++gq) {
          const uint32_t ta = t_row + (e1 + gq) * cs + c_half;
          if (kM == 32) ptx::tmem_ld_32x32b_x32(ta, *reinterpret_cast<uint32_t(*)[32]>(&v[gq * 32]));
          else ptx::tmem_ld_32x32b_x16(ta, *reinterpret_cast<uint32_t(*)[16]>(&v[gq * 16]));
        }
        ptx::tmem_wait_ld();
        if (e1 + per >= ne) {
          // every column of the unit is in registers: release the accumulator
          // before the conversions and stores of the last batch
          ptx::tc_fence_before();
          __syncwarp();
          if (lane == 0) ptx::mbar_arrive(&tempty[acc]);
        }
        {  // (every tile is full: head tiles 128 columns of one entry, pair tiles 64 of two)
#pragma unroll
          for (int q = 0; q < 64; ++q) {
            const int e = e1 + q / kM, j = q % kM;
            if (e < ne) {
              const float x = __uint_as_float(v[q]);
              const unsigned short h = kBF16 ? __bfloat16_as_ushort(__float2bfloat16_rn(x))
                                             : __half_as_ushort(__float2half_rn(x));
              const uint32_t addr = cbuf + (uint32_t)((e * 2 + half) * kM + j) * 128u + col_b;
              asm volatile("st.shared.u16 [%0], %1;" ::"r"(addr), "h"(h) : "memory");
            }
          }
        }
      }
      ptx::fence_proxy_async_smem();
      ptx::named_bar_sync(1 + wg, 128);
      if (leader) {
        ptx::tma_store_4d(U.pair ? &p.tmC2 : &p.tmC, smem + p.c_off + wg * p.c_buf, 0, 0, U.atom, (int)e0);
        ptx::bulk_commit();
      }
    }
    if (leader) ptx::bulk_wait_read<0>();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 1) ptx::tmem_dealloc(tmem_base, p.acc_bufs * p.acc_cols);
}

}  // namespace

bool tc16_xt_supported(int m, int n, int k) {
  return (m == 16 || m == 32) && n >= 64 && n <= 256 && n % 64 == 0 && (k == 16 || k == 32 || k == 64);
}

// entries per unit: the largest of 8, 4, 2, 1 that leaves at least three stages
kami_status_t tc16_xt_plan(int m, int n, int k, int* E_out, int* stages_out) {
  if (!tc16_xt_supported(m, n, k)) return KAMI_ERROR_NOT_SUPPORTED;
  const int pa = (n % 128 != 0) ? 2 : 1;  // pair tiles hold the A rows of 2E entries
  for (int E = 8; E >= 1; E >>= 1) {
    if (E * pa * m > 256) continue;         // one accumulator of <= 256 columns
    const int stage = E * (2 * k * 128 + pa * m * k * 2);
    const int cbuf = E * 2 * m * 128;
    int st = (kXtSmemLimit - 1024 - 256 - 2 * cbuf) / stage;
    if (st > kXtMaxStages) st = kXtMaxStages;
    if (st >= 3 || (E == 1 && st >= 2)) {
      *E_out = E;
      *stages_out = st;
      return KAMI_SUCCESS;
    }
  }
  return KAMI_ERROR_NOT_SUPPORTED;
}

kami_status_t tc16_xt_launch(int m, int n, int k, long long batch, bool bf16, const void* A, const void* B, void* C,
                             cudaStream_t stream) {
  XtParams p;
  memset(&p, 0, sizeof(p));
  int E = 0, stages = 0;
  kami_status_t st = tc16_xt_plan(m, n, k, &E, &stages);
  if (st != KAMI_SUCCESS) return st;
  PFN_encodeTiled enc = get_encode_tiled();
  if (!enc) return KAMI_ERROR_CUDA;
  const CUtensorMapDataType dt = bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16;
  cuuint32_t es[4] = {1, 1, 1, 1};
  {
    cuuint64_t dims[3] = {(cuuint64_t)k, (cuuint64_t)m, (cuuint64_t)batch};
    cuuint64_t str[2] = {(cuuint64_t)k * 2, (cuuint64_t)m * k * 2};
    cuuint32_t box[3] = {(cuuint32_t)k, (cuuint32_t)m, (cuuint32_t)E};
    const CUtensorMapSwizzle sw =
        k == 64 ? CU_TENSOR_MAP_SWIZZLE_128B : k == 32 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B;
    if (enc(&p.tmA, dt, 3, const_cast<void*>(A), dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  {
    cuuint64_t dims[4] = {64, (cuuint64_t)k, (cuuint64_t)(n / 64), (cuuint64_t)batch};
    cuuint64_t str[3] = {(cuuint64_t)n * 2, 128, (cuuint64_t)k * n * 2};
    cuuint32_t box[4] = {64, (cuuint32_t)k, 2, (cuuint32_t)E};
    if (enc(&p.tmB, dt, 4, const_cast<void*>(B), dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  {
    cuuint64_t dims[4] = {64, (cuuint64_t)m, (cuuint64_t)(n / 64), (cuuint64_t)batch};
    cuuint64_t str[3] = {(cuuint64_t)n * 2, 128, (cuuint64_t)m * n * 2};
    cuuint32_t box[4] = {64, (cuuint32_t)m, 2, (cuuint32_t)E};
    if (enc(&p.tmC, dt, 4, C, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  p.mode = n % 128 == 0 ? 0 : n == 64 ? 1 : 2;
  if (p.mode) {  // pair tiles: one 64-column atom of each of 2E entries
    cuuint64_t adims[3] = {(cuuint64_t)k, (cuuint64_t)m, (cuuint64_t)batch};
    cuuint64_t astr[2] = {(cuuint64_t)k * 2, (cuuint64_t)m * k * 2};
    cuuint32_t abox[3] = {(cuuint32_t)k, (cuuint32_t)m, (cuuint32_t)(2 * E)};
    const CUtensorMapSwizzle sw =
        k == 64 ? CU_TENSOR_MAP_SWIZZLE_128B : k == 32 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B;
    cuuint64_t bdims[4] = {64, (cuuint64_t)k, (cuuint64_t)(n / 64), (cuuint64_t)batch};
    cuuint64_t bstr[3] = {(cuuint64_t)n * 2, 128, (cuuint64_t)k * n * 2};
    cuuint32_t bbox[4] = {64, (cuuint32_t)k, 1, (cuuint32_t)(2 * E)};
    cuuint64_t cdims[4] = {64, (cuuint64_t)m, (cuuint64_t)(n / 64), (cuuint64_t)batch};
    cuuint64_t cstr[3] = {(cuuint64_t)n * 2, 128, (cuuint64_t)m * n * 2};
    cuuint32_t cbox[4] = {64, (cuuint32_t)m, 1, (cuuint32_t)(2 * E)};
    if (enc(&p.tmA2, dt, 3, const_cast<void*>(A), adims, astr, abox, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS ||
        enc(&p.tmB2, dt, 4, const_cast<void*>(B), bdims, bstr, bbox, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS ||
        enc(&p.tmC2, dt, 4, C, cdims, cstr, cbox, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  p.m = m;
  p.n = n;
  p.k = k;
  p.E = E;
  // UnitIter m-tile count: heads per entry group (mode 0), one pair (1), two heads + one pair (2)
  p.NT = p.mode == 0 ? n / 128 : p.mode == 1 ? 1 : 3;
  p.batch = batch;
  p.units = p.mode == 0 ? (batch + E - 1) / E * p.NT : (batch + 2 * E - 1) / (2 * E) * p.NT;
  p.stages = stages;
  p.ent_b = 2u * k * 128;  // two 64-column atoms of k rows
  p.ent_a = (uint32_t)m * k * 2;
  p.a_off = (uint32_t)E * p.ent_b;
  p.stage_bytes = (p.a_off + (uint32_t)(p.mode ? 2 : 1) * E * p.ent_a + 1023) & ~1023u;
  // (full boxes always land: entries past the batch are zero-filled and counted)
  p.tx = (uint32_t)E * (p.ent_b + p.ent_a);
  p.tx2 = (uint32_t)E * p.ent_b + 2u * E * p.ent_a;
  p.c_buf = (uint32_t)E * 2 * m * 128;
  p.c_off = (uint32_t)stages * p.stage_bytes;
  p.bar_off = p.c_off + 2 * p.c_buf;
  // the epilogue reads 64 / m groups per TMEM load batch, P m columns apart
  const int pmax = p.mode ? 2 : 1, per = 64 / m;
  int cols = 64;
  while (cols < (E > per ? E : per) * pmax * m) cols <<= 1;
  p.acc_cols = cols;
  p.acc_bufs = 512 / cols >= 4 ? 4 : 2;
  p.idesc = ptx::make_idesc_f16(bf16 ? 1 : 0, 128, m, /*a MN-major*/ 1, /*b K-major*/ 0);
  p.idesc2 = ptx::make_idesc_f16(bf16 ? 1 : 0, 128, 2 * m, 1, 0);
  const uint32_t smem = p.bar_off + 256 + 1024;
  if (smem > (uint32_t)kXtSmemLimit) return KAMI_ERROR_NOT_SUPPORTED;
  auto fn = bf16 ? (m == 16 ? kami_tc16_xt_kernel<true, 16> : kami_tc16_xt_kernel<true, 32>)
                 : (m == 16 ? kami_tc16_xt_kernel<false, 16> : kami_tc16_xt_kernel<false, 32>);
  if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return KAMI_ERROR_CUDA;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  long long grid = p.units < sms ? p.units : sms;
  grid = apply_grid_cap(grid);
  fn<<<(unsigned)grid, kXtThreads, smem, stream>>>(p);
  set_last_kernel(bf16 ? "kami_tc16_xt_kernel<bf16>" : "kami_tc16_xt_kernel<f16>");
  return (kami_status_t)launch_status((int)cudaGetLastError());
}

}  // namespace kami
