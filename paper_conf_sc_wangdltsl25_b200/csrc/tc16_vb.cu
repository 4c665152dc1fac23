// tc16_vb.cu -- FP16/BF16 batched GEMM on tcgen05 for POINTER-ARRAY and
// VARIABLE-SIZE batches ("supports various matrix orders in
// a batch").
//
// Same KAMI-1D mapping as tc16.cu (4 sub-partition tensor cores, C_i in TMEM,
// B broadcast through shared memory), but the operands cannot be described by
// one TMA tensor map (every entry has its own pointer and possibly its own
// m, n, k), so a producer warpgroup performs the paper's GMem2Reg + Reg2SMem
// itself: coalesced 16-byte cp.async (LDGSTS) copies of A and B rows straight
// into the UMMA canonical layouts (128-byte swizzle, K-major A, N-major B),
// zero-filling k beyond the entry's order; once a stage's copy group has
// landed, a generic->async proxy fence and an mbarrier arrive hand it to the
// MMA warp.
//
// Warps: 0-3 producer, 4 MMA issuer + TMEM allocator, 5-12 epilogue (two
// warpgroups on alternate units; tcgen05.ld -> cvt.rn -> padded SMEM staging
// -> coalesced 16-byte st.global).
// A unit is one (entry, 128-row m-tile); N = the entry's n (<= 256).
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstring>

#include "kernels.h"
#include "ptx.cuh"

namespace kami {
namespace {

constexpr int kVbThreads = 416;  // 13 warps
constexpr int kVbStages = 3;
constexpr uint32_t kAReg = 128 * 128;       // 128 rows x 64 k (128 B)
constexpr uint32_t kBReg = 4 * 64 * 128;    // 4 N-atoms x 64 k-rows x 128 B
constexpr uint32_t kStage = kAReg + kBReg;  // 48 KB
constexpr uint32_t kCRow = 128 * 2 + 16;               // padded staging row (128 columns)
constexpr uint32_t kCBuf = 128 * kCRow;                 // one warpgroup's C staging (34 KB)
constexpr uint32_t kCStage = kVbStages * kStage;        // offset of the C staging buffers
constexpr uint32_t kBarOff = kCStage + 2 * kCBuf;       // barriers + tables
constexpr uint32_t kVbSmem = kBarOff + 1024 + 1024;

struct VbParams {
  const void* const* A;
  const void* const* B;
  void* const* C;
  const int* dm;  // per-entry sizes (device) or nullptr -> uniform m, n, k
  const int* dn;
  const int* dk;
  int m, n, k;
  int mtiles;  // m-tiles per entry slot (1 or 2)
  long long batch;
  // SpMM (Sec. 4.6): A block-sparse in BSR with 16 x 16 dense blocks
  // (block-row order, the 1D storage of Fig. 7(a)); B, C dense and strided.
  int bsr, max_nnzb;
  const int* rowptr;
  const int* colblk;
  const uint16_t* vals;
  const uint16_t* Bs;
  uint16_t* Cs;
};

__device__ __forceinline__ const uint16_t* entry_B(const VbParams& p, long long e, int k, int n) {
  return p.bsr ? p.Bs + e * (long long)k * n : reinterpret_cast<const uint16_t*>(p.B[e]);
}
__device__ __forceinline__ uint16_t* entry_C(const VbParams& p, long long e, int m, int n) {
  return p.bsr ? p.Cs + e * (long long)m * n : reinterpret_cast<uint16_t*>(p.C[e]);
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

template <bool kBF16>
__global__ void __launch_bounds__(kVbThreads, 1) kami_tc16_vb_kernel(const __grid_constant__ VbParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + kBarOff);
  uint64_t* empty = full + kVbStages;
  uint64_t* tfull = empty + kVbStages;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);
  int* blk_tab = reinterpret_cast<int*>(tmem_slot + 4);  // SpMM: [8 block rows][16 block cols] -> block index
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < kVbStages; ++s) {
      ptx::mbar_init(&full[s], 128);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], 4);
    }
    ptx::fence_mbar_init();
  }
  if (warp == 4) ptx::tmem_alloc(tmem_slot, 512);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  const uint32_t smem_base = ptx::smem_u32(smem);
  const long long units = p.batch * p.mtiles;

  if (warp < 4) {
    // ------------------------------------------------ producer warpgroup
    // cp.async (LDGSTS) straight into the swizzled stage buffers, zero-filled
    // outside the entry; a stage is handed to the MMA warp (fence.proxy.async
    // + mbarrier arrive) once its copy group has landed, kLag stages later, so
    // several stages stream concurrently without register staging.
    constexpr int kLag = kVbStages - 1;
    const int tid = threadIdx.x;  // 0..127
    uint32_t it = 0, handed = 0;
    auto hand_over = [&](int pending) {
      // copies of stage `handed` are complete when at most `pending` groups remain
      static_assert(kLag <= 3, "wait_group depth");
      if (pending >= 3) ptx::cp_async_wait<3>();
      else if (pending == 2) ptx::cp_async_wait<2>();
      else if (pending == 1) ptx::cp_async_wait<1>();
      else ptx::cp_async_wait<0>();
      ptx::fence_proxy_async_smem();
      ptx::mbar_arrive(&full[handed % kVbStages]);
      ++handed;
    };
    for (long long u = blockIdx.x; u < units; u += gridDim.x) {
      const long long e = u / p.mtiles;
      const int mt = (int)(u - e * p.mtiles);
      int m, n, k;
      entry_dims(p, e, m, n, k);
      if (mt * 128 >= m) continue;
      const uint16_t* A = p.bsr ? nullptr : reinterpret_cast<const uint16_t*>(p.A[e]);
      const uint16_t* B = entry_B(p, e, k, n);
      const int kchunks = (k + 63) / 64;
      if (p.bsr) {
        // this m-tile's block lookup table: -1 = absent block (zero-filled)
        ptx::named_bar_sync(3, 128);  // previous unit's copies issued: table reusable
        blk_tab[tid] = -1;
        ptx::named_bar_sync(3, 128);
        const int mb = m / 16;
        const int br0 = mt * 8, br1 = min(br0 + 8, mb);
        const int* rp = p.rowptr + e * (mb + 1);
        const int j0 = __ldg(rp + br0), j1 = __ldg(rp + br1);
        for (int j = j0 + tid; j < j1; j += 128) {
          int br = br0;
          while (__ldg(rp + br + 1) <= j) ++br;
          blk_tab[(br - br0) * 16 + __ldg(p.colblk + e * (long long)p.max_nnzb + j)] = j;
        }
        ptx::named_bar_sync(3, 128);
      }
      const int nc8 = n / 8;  // 16-byte chunks per B row
      for (int kc = 0; kc < kchunks; ++kc, ++it) {
        const uint32_t s = it % kVbStages;
        ptx::mbar_wait(&empty[s], ((it / kVbStages) & 1) ^ 1);
        const uint32_t sa = smem_base + s * kStage, sb = sa + kAReg;
        // A: 128 rows x 8 chunks; a warp covers 4 whole 128-byte row segments
#pragma unroll 4
        for (int i = tid; i < 128 * 8; i += 128) {
          const int r = i >> 3, j = i & 7;
          const int gr = mt * 128 + r, gc = kc * 64 + j * 8;
          bool ok = gr < m && gc < k;
          const uint16_t* src;
          if (p.bsr) {  // densify on load: block (r/16, gc/16) or zeros
            const int idx = ok ? blk_tab[(r >> 4) * 16 + (gc >> 4)] : -1;
            ok = idx >= 0;
            src = ok ? p.vals + ((e * (long long)p.max_nnzb + idx) * 256 + (r & 15) * 16 + (gc & 15)) : p.vals;
          } else {
            src = ok ? A + (long long)gr * k + gc : A;
          }
          ptx::cp_async_16(sa + r * 128 + ((j ^ (r & 7)) << 4), src, ok ? 16 : 0);
        }
        // B: 64 k-rows x n/8 chunks into N-atoms of 64 columns
        for (int i = tid; i < 64 * nc8; i += 128) {
          const int kr = i / nc8, j = i - kr * nc8;
          const int gk = kc * 64 + kr;
          const bool ok = gk < k;
          const uint16_t* src = ok ? B + (long long)gk * n + j * 8 : B;
          ptx::cp_async_16(sb + (j >> 3) * 8192 + kr * 128 + (((j & 7) ^ (kr & 7)) << 4), src, ok ? 16 : 0);
        }
        ptx::cp_async_commit();
        if (it + 1 - handed > (uint32_t)kLag) hand_over(kLag);
      }
    }
    while (handed < it) hand_over((int)(it - handed - 1));
  } else if (warp == 4) {
    // ------------------------------------------------------------- MMA
    uint32_t it = 0, acc_it = 0;
    for (long long u = blockIdx.x; u < units; u += gridDim.x) {
      const long long e = u / p.mtiles;
      const int mt = (int)(u - e * p.mtiles);
      int m, n, k;
      entry_dims(p, e, m, n, k);
      if (mt * 128 >= m) continue;
      const uint32_t a = acc_it & 1;
      ptx::mbar_wait(&tempty[a], ((acc_it >> 1) & 1) ^ 1);
      ptx::tc_fence_after();
      const uint32_t d_tmem = tmem_base + a * 256;
      const uint32_t idesc = ptx::make_idesc_f16(kBF16 ? 1 : 0, 128, n, 0, 1);
      const int kpad = (k + 15) / 16 * 16;
      const int kchunks = (k + 63) / 64;
      for (int kc = 0; kc < kchunks; ++kc, ++it) {
        const uint32_t s = it % kVbStages;
        ptx::mbar_wait(&full[s], (it / kVbStages) & 1);
        ptx::tc_fence_after();
        if (lane == 0) {
          const uint32_t sa = smem_base + s * kStage, sb = sa + kAReg;
          const int nsteps = (kpad - kc * 64) >= 64 ? 4 : (kpad - kc * 64) / 16;
          for (int ks = 0; ks < nsteps; ++ks) {
            const uint64_t adesc = ptx::make_smem_desc(sa + ks * 32, 16, 1024, 2);
            const uint64_t bdesc = ptx::make_smem_desc(sb + ks * 2048, 8192, 1024, 2);
            ptx::umma_f16_ss(d_tmem, adesc, bdesc, idesc, (kc | ks) != 0);
          }
          ptx::umma_commit(&empty[s]);
        }
        __syncwarp();
      }
      if (lane == 0) ptx::umma_commit(&tfull[a]);
      __syncwarp();
      ++acc_it;
    }
  } else {
    // -------------------------------------------------------- epilogue
    const int wg = (warp - 5) >> 2;
    const int sp = warp & 3;
    const int L = sp * 32 + lane;
    uint32_t acc_it = 0;
    for (long long u = blockIdx.x; u < units; u += gridDim.x) {
      const long long e = u / p.mtiles;
      const int mt = (int)(u - e * p.mtiles);
      int m, n, k;
      entry_dims(p, e, m, n, k);
      if (mt * 128 >= m) continue;
      const uint32_t a = acc_it & 1;
      const bool mine = (int)(acc_it & 1) == wg;  // accumulator a is drained by warpgroup a
      ++acc_it;
      if (!mine) continue;
      ptx::mbar_wait(&tfull[a], ((acc_it - 1) >> 1) & 1);
      ptx::tc_fence_after();
      // Stage the tile through padded shared memory (row stride 272 B: rows
      // land on different banks, conflict-free) in 128-column halves, then
      // copy out with coalesced 16-byte stores (a warp writes whole rows).
      const int rows = min(128, m - mt * 128);
      const bool warp_live = sp * 32 < rows;
      uint16_t* Cbase = entry_C(p, e, m, n) + (long long)mt * 128 * n;
      const uint32_t t_row = tmem_base + (uint32_t(sp * 32) << 16) + a * 256;
      const uint32_t cst = smem_base + kCStage + wg * kCBuf;
      for (int h0 = 0; h0 < n; h0 += 128) {
        const int hw = min(128, n - h0);
        if (warp_live) {
          for (int c0 = 0; c0 < hw; c0 += 32) {
            uint32_t v[32];
            if (hw - c0 >= 32) ptx::tmem_ld_32x32b_x32(t_row + h0 + c0, v);
            else ptx::tmem_ld_32x32b_x16(t_row + h0 + c0, *reinterpret_cast<uint32_t(*)[16]>(&v[0]));
            ptx::tmem_wait_ld();
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
        ptx::named_bar_sync(1 + wg, 128);
        // copy-out: chunk index i -> (row i / cpr, 16-byte chunk i % cpr)
        const int cpr = hw / 8;
        for (int i = L; i < rows * cpr; i += 128) {
          const int r = i / cpr, c = i - r * cpr;
          uint32_t x0, x1, x2, x3;
          ptx::ld_shared_v4(cst + r * kCRow + c * 16, x0, x1, x2, x3);
          ptx::st_global_v4(Cbase + (long long)r * n + h0 + c * 8, make_uint4(x0, x1, x2, x3));
        }
        ptx::named_bar_sync(1 + wg, 128);  // staging buffer reusable
      }
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&tempty[a]);
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (warp == 4) ptx::tmem_dealloc(tmem_base, 512);
}

}  // namespace

namespace {
kami_status_t vb_launch(const VbParams& p, bool bf16, cudaStream_t stream);
}

kami_status_t tc16_spmm_bsr_launch(int m, int n, int k, long long batch, bool bf16, const int* row_ptr,
                                   const int* col_blk, const void* vals, int max_nnzb, const void* B, void* C,
                                   cudaStream_t stream) {
  VbParams p;
  memset(&p, 0, sizeof(p));
  p.m = m;
  p.n = n;
  p.k = k;
  p.mtiles = (m + 127) / 128;
  p.batch = batch;
  p.bsr = 1;
  p.max_nnzb = max_nnzb;
  p.rowptr = row_ptr;
  p.colblk = col_blk;
  p.vals = static_cast<const uint16_t*>(vals);
  p.Bs = static_cast<const uint16_t*>(B);
  p.Cs = static_cast<uint16_t*>(C);
  return vb_launch(p, bf16, stream);
}

kami_status_t tc16_vb_launch(long long batch, bool bf16, int m, int n, int k, const int* dm, const int* dn,
                             const int* dk, int max_m, const void* const* A, const void* const* B, void* const* C,
                             cudaStream_t stream) {
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
  p.mtiles = (max_m + 127) / 128;
  p.batch = batch;
  return vb_launch(p, bf16, stream);
}

namespace {
kami_status_t vb_launch(const VbParams& p, bool bf16, cudaStream_t stream) {
  const long long batch = p.batch;
  auto fn = bf16 ? kami_tc16_vb_kernel<true> : kami_tc16_vb_kernel<false>;
  if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kVbSmem) != cudaSuccess)
    return KAMI_ERROR_CUDA;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const long long units = batch * p.mtiles;
  const long long grid = units < sms ? units : sms;
  fn<<<(unsigned)grid, kVbThreads, kVbSmem, stream>>>(p);
  set_last_kernel(p.bsr ? (bf16 ? "kami_tc16_vb_kernel<bf16,spmm_bsr>" : "kami_tc16_vb_kernel<f16,spmm_bsr>")
                        : (bf16 ? "kami_tc16_vb_kernel<bf16>" : "kami_tc16_vb_kernel<f16>"));
  return cudaGetLastError() == cudaSuccess ? KAMI_SUCCESS : KAMI_ERROR_CUDA;
}
}  // namespace

}  // namespace kami
