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
// A unit = (group of E entries, 128-column tile of n).
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
  int m, n, k, E, NT;
  long long batch, units;
  int stages;
  uint32_t stage_bytes, a_off, ent_b, ent_a;
  uint32_t c_off, c_buf, bar_off;
  uint32_t idesc, tx;
  int acc_cols;
};

template <bool kBF16, int kM>
__global__ void __launch_bounds__(kXtThreads, 1) kami_tc16_xt_kernel(const __grid_constant__ XtParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + p.bar_off);
  uint64_t* empty = full + kXtMaxStages;
  uint64_t* tfull = empty + kXtMaxStages;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    ptx::prefetch_tmap(&p.tmA);
    ptx::prefetch_tmap(&p.tmB);
    ptx::prefetch_tmap(&p.tmC);
    for (int s = 0; s < p.stages; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], 4);  // the four warps of epilogue warpgroup a
    }
    ptx::fence_mbar_init();
  }
  if (warp == 1) ptx::tmem_alloc(tmem_slot, 2 * p.acc_cols);
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
        ptx::mbar_arrive_expect_tx(&full[r.s], p.tx);
        uint8_t* st = smem + r.s * p.stage_bytes;
        const int e0 = (int)(ui.grp * p.E);
        ptx::tma_load_4d(st, &p.tmB, &full[r.s], 0, 0, 2 * ui.mt, e0);  // B^T: the MMA's A operand
        ptx::tma_load_3d(st + p.a_off, &p.tmA, &full[r.s], 0, 0, e0);   // A^T: the MMA's B operand
      }
    }
  } else if (warp == 1) {
    // ---------------------------------------------------------- MMA issuer
    RingPos r, ra;
    const uint32_t a_sw = (uint32_t)p.k * 2u;  // A rows: 2k bytes, 2k-byte swizzle
    const int ksteps = p.k / 16;
    for (long long u = blockIdx.x; u < p.units; u += gridDim.x, r.next(p.stages), ra.next(2)) {
      ptx::mbar_wait(&tempty[ra.s], ra.ph ^ 1);
      ptx::tc_fence_after();
      ptx::mbar_wait(&full[r.s], r.ph);
      ptx::tc_fence_after();
      if (lane == 0) {
        const uint32_t sb = smem_base + r.s * p.stage_bytes, sa = sb + p.a_off;
        for (int e = 0; e < p.E; ++e) {
          const uint32_t d = tmem_base + ra.s * p.acc_cols + e * p.m;
          for (int ks = 0; ks < ksteps; ++ks) {
            // B^T (MN-major): two 64-column atoms k*128 bytes apart, a K step = 16 rows of 128 B
            const uint64_t ad = ptx::make_smem_desc(sb + e * p.ent_b + ks * 2048, (uint32_t)p.k * 128, 1024, 2);
            // A^T (K-major): m rows of 2k bytes, a K step = 32 bytes along the row
            const uint64_t bd = ptx::make_smem_desc(sa + e * p.ent_a + ks * 32, 16, 8 * a_sw,
                                                    ptx::umma_layout_code((int)a_sw));
            ptx::umma_f16_ss(d, ad, bd, p.idesc, ks != 0);
          }
        }
        ptx::umma_commit(&empty[r.s]);
        ptx::umma_commit(&tfull[ra.s]);
      }
      __syncwarp();
    }
  } else {
    // ------------------------------------------------------------ epilogue
    // warpgroup wg takes the CTA's units i = wg, wg + 2, ... and always
    // accumulator wg (the MMA alternates accumulators unit by unit)
    const int wg = (warp - 2) >> 2;
    const int sp = warp & 3;          // TMEM sub-partition of this warp
    const int col = sp * 32 + lane;   // this thread's column of the 128-column tile
    const int atom = col >> 6;
    const uint32_t col_b = (uint32_t)(col & 63) * 2u;
    const bool leader = (warp & 3) == 2 && lane == 0;
    const uint32_t cbuf = smem_base + p.c_off + wg * p.c_buf;
    constexpr int per = 64 / kM;      // entries per TMEM load batch (64 columns)
    uint32_t ph = 0;
    UnitIter ui(blockIdx.x + (long long)wg * gridDim.x, 2ll * gridDim.x, p.NT);
    for (long long u = blockIdx.x + (long long)wg * gridDim.x; u < p.units; u += 2ll * gridDim.x, ui.next(), ph ^= 1) {
      const long long e0 = ui.grp * p.E;
      const int ne = p.batch - e0 < p.E ? (int)(p.batch - e0) : p.E;
      const bool live = ui.mt * 128 + col < p.n;
      // this warpgroup's previous store is done reading the staging tile
      if (leader) ptx::bulk_wait_read<0>();
      ptx::named_bar_sync(1 + wg, 128);
      ptx::mbar_wait(&tfull[wg], ph);
      ptx::tc_fence_after();
      const uint32_t t_row = tmem_base + (uint32_t(sp * 32) << 16) + wg * p.acc_cols;
      for (int e1 = 0; e1 < ne; e1 += per) {
        uint32_t v[64];
        // one wait per 64 columns: a wait per entry serialised the TMEM load latency
        ptx::tmem_ld_32x32b_x32(t_row + e1 * kM, *reinterpret_cast<uint32_t(*)[32]>(&v[0]));
        ptx::tmem_ld_32x32b_x32(t_row + e1 * kM + 32, *reinterpret_cast<uint32_t(*)[32]>(&v[32]));
        ptx::tmem_wait_ld();
        if (live) {
#pragma unroll
          for (int q = 0; q < 64; ++q) {
            const int e = e1 + q / kM, j = q % kM;
            if (e < ne) {
              const float x = __uint_as_float(v[q]);
              const unsigned short h = kBF16 ? __bfloat16_as_ushort(__float2bfloat16_rn(x))
                                             : __half_as_ushort(__float2half_rn(x));
              const uint32_t addr = cbuf + (uint32_t)((e * 2 + atom) * kM + j) * 128u + col_b;
              asm volatile("st.shared.u16 [%0], %1;" ::"r"(addr), "h"(h) : "memory");
            }
          }
        }
      }
      ptx::tc_fence_before();  // accumulator wg may be overwritten by the MMA of this warpgroup's next unit
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&tempty[wg]);
      ptx::fence_proxy_async_smem();
      ptx::named_bar_sync(1 + wg, 128);
      if (leader) {
        ptx::tma_store_4d(&p.tmC, smem + p.c_off + wg * p.c_buf, 0, 0, 2 * ui.mt, (int)e0);
        ptx::bulk_commit();
      }
    }
    if (leader) ptx::bulk_wait_read<0>();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 1) ptx::tmem_dealloc(tmem_base, 2 * p.acc_cols);
}

}  // namespace

bool tc16_xt_supported(int m, int n, int k) {
  return (m == 16 || m == 32) && n >= 64 && n <= 256 && n % 64 == 0 && (k == 16 || k == 32 || k == 64);
}

// entries per unit: the largest of 8, 4, 2, 1 that leaves at least three stages
kami_status_t tc16_xt_plan(int m, int n, int k, int* E_out, int* stages_out) {
  if (!tc16_xt_supported(m, n, k)) return KAMI_ERROR_NOT_SUPPORTED;
  for (int E = 8; E >= 1; E >>= 1) {
    const int stage = E * (2 * k * 128 + m * k * 2);
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
  p.m = m;
  p.n = n;
  p.k = k;
  p.E = E;
  p.NT = (n + 127) / 128;
  p.batch = batch;
  p.units = (batch + E - 1) / E * p.NT;
  p.stages = stages;
  p.ent_b = 2u * k * 128;  // two 64-column atoms of k rows
  p.ent_a = (uint32_t)m * k * 2;
  p.a_off = (uint32_t)E * p.ent_b;
  p.stage_bytes = (p.a_off + (uint32_t)E * p.ent_a + 1023) & ~1023u;
  // (full boxes always land: OOB atoms of a 64-column last tile and entries
  // past the batch are zero-filled and counted)
  p.tx = (uint32_t)E * (p.ent_b + p.ent_a);
  p.c_buf = (uint32_t)E * 2 * m * 128;
  p.c_off = (uint32_t)stages * p.stage_bytes;
  p.bar_off = p.c_off + 2 * p.c_buf;
  int cols = 64;  // >= 64: the epilogue reads 64 columns per TMEM load batch
  while (cols < E * m) cols <<= 1;
  p.acc_cols = cols;
  p.idesc = ptx::make_idesc_f16(bf16 ? 1 : 0, 128, m, /*a MN-major*/ 1, /*b K-major*/ 0);
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
