// dmma_tma.cu -- FP64 batched GEMM: KAMI-1D on the DMMA tensor path with the
// broadcast operand delivered by TMA (the B200 form of the FP64 schedule).
//
// KAMI-1D (Alg. 1) partitions one operand among p warps
// (local, registers) and broadcasts the other through shared memory.  Here we
// apply it to C^T = B^T A^T, i.e. the warps partition the COLUMNS:
//   warp w holds B_w = B[:, w n/p:(w+1) n/p] and C_w = C[:, w n/p:(w+1) n/p]
//   in registers as DMMA fragments (GMem2Reg straight from global);
//   A (m x k) is the broadcast operand: one TMA tensor copy per entry writes it
//   into shared memory in the 128-byte-swizzled layout, and every warp reads
//   its A fragments from there -- bank-conflict free (the 8-row XOR swizzle
//   spreads the 8 rows of a fragment over distinct 16-byte bank groups).
// Stage z of Alg. 1 is the z-th k-slice of 4 (one DMMA k-step); all p warps
// consume the same broadcast slice.  Each team (p warps) double-buffers A:
// the TMA for its next entry is issued while the current one computes, and
// the next entry's B is bulk-prefetched into L2, so HBM streaming overlaps the
// DMMA work.  SMEM traffic per entry: m k s_e written (TMA) + p m k s_e read.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>
#include <cstring>

#include "kernels.h"
#include "ptx.cuh"
#include "sched.cuh"

namespace kami {
namespace {

template <int M, int N, int K, int P, int TEAMS>
struct DmmaTmaCfg {
  static constexpr int NP = N / P;        // columns per warp
  static constexpr int FN = NP / 8;       // 8-wide DMMA n-fragments per warp
  static constexpr int FM = M / 8;        // 8-tall m-fragments
  static constexpr int FK = K / 4;        // k-steps
  static constexpr int A_BYTES = M * K * 8;
  static constexpr int KCH = K / 16;      // 128-byte (16-double) column chunks of A
  static constexpr int THREADS = P * 32 * TEAMS;
  static constexpr int SMEM = TEAMS * 2 * A_BYTES + 1024 /*align*/ + 256 /*barriers*/;
  static_assert(NP % 8 == 0 && K % 16 == 0 && M % 8 == 0, "shape");
};

struct DmmaTmaParams {
  CUtensorMap tmA;  // 4-D (16, m, k/16, batch), box (16, m, k/16, 1), SW128
                    // pointer arrays: 5-D (16, m, k/16, view lo, view hi), box (16, m, k/16, 1, 1)
  const double* B;
  double* C;
  long long batch;
  double alpha, beta;  // C = alpha A B + beta C (C read iff beta != 0)
  // pointer arrays (kPtr; kami_gemm_batched): entry e at Aa[e], Ba[e], Ca[e]
  const void* const* Aa;
  const double* const* Ba;
  double* const* Ca;
};

// Pointer-array A: address-space view (sched.cuh); the box is the whole entry
// (16, m, k/16), never partly out of bounds.
template <bool kPtr>
__device__ __forceinline__ void load_a_entry(void* dst, const DmmaTmaParams& prm, uint64_t* bar, long long e) {
  if constexpr (kPtr) {
    int lo, hi;
    view_coords(prm.Aa[e], lo, hi);
    ptx::tma_load_5d(dst, &prm.tmA, bar, 0, 0, 0, lo, hi);
  } else {
    ptx::tma_load_4d(dst, &prm.tmA, bar, 0, 0, 0, (int)e);
  }
}

// The k index lane t supplies in DMMA k-step kk.  The 128-byte swizzle puts
// 16-byte unit u of A row r at unit u ^ (r mod 8); an LDS.64 is served per
// half-warp (4 rows x 4 lanes), so with the natural order (lanes t = 0..3 ->
// columns 4 kk + t, i.e. units 2a, 2a + 1) rows r and r ^ 1 of a half-warp hit
// the same 8 banks: 4 wavefronts per LDS.64 instead of 2 (ncu: 69.4 M
// wavefronts for 33.5 M ideal at f64 64^3, profiles/r2).  Taking the k-step's
// four columns from units a and a ^ 4 of the 16-column chunk (lanes t = 0, 1:
// columns 2a, 2a + 1; t = 2, 3: 2a + 8, 2a + 9) gives the four rows of a
// half-warp eight distinct units.  Any permutation of k applied to A and B
// alike leaves the product unchanged.
// Used for k = 64 only (FK = 16 k-steps): at 32^3 the permuted B_w loads
// measured slower (14.8 vs 17.0-17.4 TF/s, profiles/r2/fp64_kperm_r2.txt)
// than the half-warp conflicts they remove.
template <bool kP>
__device__ __forceinline__ int kperm(int kk, int t) {
  return kP ? ((kk >> 2) << 4) + ((kk & 3) << 1) + (t & 1) + ((t >> 1) << 3) : kk * 4 + t;
}

// B_w fragments of k-steps [K0, K1) of one entry (k = kperm(kk, t), n = g of each 8x8 block).
// volatile asm keeps the loads where the schedule puts them relative to the MMAs.
template <int N, int FN, int K0, int K1, int FK>
__device__ __forceinline__ void load_b_steps(double (&b)[FK][FN], const double* Bg, int t, int g) {
#pragma unroll
  for (int kk = K0; kk < K1; ++kk)
#pragma unroll
    for (int j = 0; j < FN; ++j)
      asm volatile("ld.global.nc.f64 %0, [%1];" : "=d"(b[kk][j]) : "l"(Bg + kperm<(FK >= 16)>(kk, t) * N + j * 8 + g));
}

// One k-step range of the entry: A fragments from the swizzled broadcast tile
// (chunk = col/16, 16-B unit = (col%16)/2 ^ row%8), B_w and C_w in registers.
template <int M, int FM, int FN, int K0, int K1, int FK>
__device__ __forceinline__ void mma_steps(double (&c)[FM][FN][2], const double (&b)[FK][FN], uint32_t a_s, int t,
                                          int g) {
#pragma unroll
  for (int kk = K0; kk < K1; ++kk) {
    const int col = kperm<(FK >= 16)>(kk, t);
    const uint32_t chunk_off = (uint32_t)(col >> 4) * (M * 128) + ((col & 1) << 3);
    const uint32_t unit = (uint32_t)((col & 15) >> 1);
#pragma unroll
    for (int i = 0; i < FM; ++i) {
      const int row = i * 8 + g;
      const uint32_t addr = a_s + chunk_off + row * 128 + ((unit ^ (row & 7)) << 4);
      double a;
      asm volatile("ld.shared.f64 %0, [%1];" : "=d"(a) : "r"(addr));
#pragma unroll
      for (int j = 0; j < FN; ++j)
        asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                     : "+d"(c[i][j][0]), "+d"(c[i][j][1])
                     : "d"(a), "d"(b[kk][j]));
    }
  }
}

// kUpd: C = alpha A B + beta C epilogue; the plain instantiation has none of it.
template <int M, int N, int K, int P, int TEAMS, bool kUpd, bool kRot, bool kPtr = false>
__global__ void __launch_bounds__(P * 32 * TEAMS, 1) kami_dmma_tma_1d_kernel(const __grid_constant__ DmmaTmaParams prm) {
  using Cfg = DmmaTmaCfg<M, N, K, P, TEAMS>;
  static_assert(TEAMS < 16, "named barrier ids 1 + team must stay within bar.sync's 0..15");
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1024-byte aligned base; pointer arithmetic on the __shared__ array keeps
  // the address space, so table reads compile to LDS rather than generic loads
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + TEAMS * 2 * Cfg::A_BYTES);  // [TEAMS][2]
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int team = warp / P, w = warp % P;
  const int g = lane >> 2, t = lane & 3;
  if (threadIdx.x == 0) {
    ptx::prefetch_tmap(&prm.tmA);
    for (int i = 0; i < TEAMS * 2; ++i) ptx::mbar_init(&full[i], 1);
    ptx::fence_mbar_init();
    ptx::fence_proxy_async_smem();
  }
  __syncthreads();
  const long long nteams = (long long)gridDim.x * TEAMS;
  const long long first = (long long)blockIdx.x * TEAMS + team;
  const bool issuer = (w == 0 && lane == 0);
  const uint32_t bar = 1 + team;
  uint8_t* abuf = smem + team * 2 * Cfg::A_BYTES;
  uint64_t* tfull = full + team * 2;
  if (issuer && first < prm.batch) {  // prologue: A of the first entry
    ptx::mbar_arrive_expect_tx(&tfull[0], Cfg::A_BYTES);
    load_a_entry<kPtr>(abuf, prm, &tfull[0], first);
  }
  // entry e's B / C: packed strided, or the pointer arrays (B pointer carried
  // one entry ahead, so the entry's loads never wait on a pointer fetch)
  auto b_of = [&](long long e) -> const double* {
    if constexpr (kPtr) return prm.Ba[e];
    else return prm.B + e * (long long)K * N;
  };
  auto c_of = [&](long long e) -> double* {
    if constexpr (kPtr) return prm.Ca[e];
    else return prm.C + e * (long long)M * N;
  };
  const double* Bcur = first < prm.batch ? b_of(first) : nullptr;
  constexpr int H = Cfg::FK / 2;
  double b[Cfg::FK][Cfg::FN];
  // kRot: B_w rotates through the registers half an entry ahead -- the first
  // k-half of entry e+1 is loaded into the slots of entry e's first k-half as
  // soon as those MMAs have issued, so the next entry starts without an L2
  // round trip and no extra registers are needed.
  if (kRot && first < prm.batch) load_b_steps<N, Cfg::FN, 0, H>(b, Bcur + w * Cfg::NP, t, g);
  uint32_t it = 0;
  for (long long e = first; e < prm.batch; e += nteams, ++it) {
    const uint32_t s = it & 1;
    const long long en = e + nteams;
    const double* Bnext = en < prm.batch ? b_of(en) : nullptr;
    double* const Ce = c_of(e);
    // all warps of the team finished reading buffer s^1 (entry it-1) at the
    // barrier that ended the previous iteration: refill it with entry it+1
    if (issuer && en < prm.batch) {
      ptx::mbar_arrive_expect_tx(&tfull[s ^ 1], Cfg::A_BYTES);
      load_a_entry<kPtr>(abuf + (s ^ 1) * Cfg::A_BYTES, prm, &tfull[s ^ 1], en);
      ptx::prefetch_l2_bulk(Bnext, (uint32_t)(K * N * 8));
    }
    // GMem2Reg: this warp's B_w (k x n/p) as DMMA B fragments (k = t, n = g)
    const double* Bg = Bcur + w * Cfg::NP;
    if (kRot) {
      load_b_steps<N, Cfg::FN, H, Cfg::FK>(b, Bg, t, g);
    } else {
#pragma unroll
      for (int kk = 0; kk < Cfg::FK; ++kk)
#pragma unroll
        for (int j = 0; j < Cfg::FN; ++j) b[kk][j] = __ldg(Bg + kperm<(Cfg::FK >= 16)>(kk, t) * N + j * 8 + g);
    }
    double c[Cfg::FM][Cfg::FN][2];
#pragma unroll
    for (int i = 0; i < Cfg::FM; ++i)
#pragma unroll
      for (int j = 0; j < Cfg::FN; ++j) c[i][j][0] = c[i][j][1] = 0.0;
    ptx::mbar_wait(&tfull[s], (it >> 1) & 1);
    const uint32_t a_s = ptx::smem_u32(abuf + s * Cfg::A_BYTES);
    mma_steps<M, Cfg::FM, Cfg::FN, 0, H>(c, b, a_s, t, g);
    if (kRot && en < prm.batch) load_b_steps<N, Cfg::FN, 0, H>(b, Bnext + w * Cfg::NP, t, g);
    mma_steps<M, Cfg::FM, Cfg::FN, H, Cfg::FK>(c, b, a_s, t, g);
    // Reg2GMem: C_w, lane holds (row g, cols 2t, 2t+1) of each 8x8 block
    double* Cg = Ce + w * Cfg::NP;
#pragma unroll
    for (int i = 0; i < Cfg::FM; ++i)
#pragma unroll
      for (int j = 0; j < Cfg::FN; ++j)
      {
        double* dst = Cg + (i * 8 + g) * N + j * 8 + 2 * t;
        double r0 = c[i][j][0], r1 = c[i][j][1];
        if (kUpd && prm.beta != 0.0) {
          const double2 o = *reinterpret_cast<const double2*>(dst);
          r0 = fma(prm.beta, o.x, prm.alpha * r0);
          r1 = fma(prm.beta, o.y, prm.alpha * r1);
        } else if (kUpd && prm.alpha != 1.0) {
          r0 *= prm.alpha;
          r1 *= prm.alpha;
        }
        ptx::st_global_v2_f64(dst, r0, r1);
      }
    ptx::named_bar_sync(bar, P * 32);  // buffer s free for entry it+2
    Bcur = Bnext;
  }
}

template <int M, int N, int K, int P, int TEAMS, bool kRot = false>
kami_status_t launch(long long batch, const void* A, const void* B, void* C, cudaStream_t stream, const char* name,
                     double alpha, double beta, const void* const* Aa, const void* const* Ba, void* const* Ca) {
  using Cfg = DmmaTmaCfg<M, N, K, P, TEAMS>;
  PFN_encodeTiled enc = get_encode_tiled();
  if (!enc) return KAMI_ERROR_CUDA;
  const bool ptr = Aa != nullptr;
  if (ptr && (alpha != 1.0 || beta != 0.0 || !Ba || !Ca)) return KAMI_ERROR_NOT_SUPPORTED;
  DmmaTmaParams prm;
  memset(&prm, 0, sizeof(prm));
  if (ptr) {  // address-space view, one whole entry per box
    cuuint64_t dims[5] = {16, (cuuint64_t)M, (cuuint64_t)(K / 16), 1ull << 24, 1ull << 20};
    cuuint64_t strides[4] = {(cuuint64_t)K * 8, 128, 16, 1ull << 28};
    cuuint32_t box[5] = {16, (cuuint32_t)M, (cuuint32_t)(K / 16), 1, 1};
    cuuint32_t es[5] = {1, 1, 1, 1, 1};
    if (enc(&prm.tmA, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 5, reinterpret_cast<void*>(kViewBase), dims, strides, box,
            es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_NOT_SUPPORTED;
  } else {
    cuuint64_t dims[4] = {16, (cuuint64_t)M, (cuuint64_t)(K / 16), (cuuint64_t)batch};
    cuuint64_t strides[3] = {(cuuint64_t)K * 8, 128, (cuuint64_t)M * K * 8};
    cuuint32_t box[4] = {16, (cuuint32_t)M, (cuuint32_t)(K / 16), 1};
    cuuint32_t es[4] = {1, 1, 1, 1};
    if (enc(&prm.tmA, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, const_cast<void*>(A), dims, strides, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  prm.B = static_cast<const double*>(B);
  prm.C = static_cast<double*>(C);
  prm.Aa = Aa;
  prm.Ba = reinterpret_cast<const double* const*>(Ba);
  prm.Ca = reinterpret_cast<double* const*>(Ca);
  prm.batch = batch;
  prm.alpha = alpha;
  prm.beta = beta;
  auto fn = ptr ? kami_dmma_tma_1d_kernel<M, N, K, P, TEAMS, false, kRot, true>
            : (alpha != 1.0 || beta != 0.0) ? kami_dmma_tma_1d_kernel<M, N, K, P, TEAMS, true, kRot>
                                            : kami_dmma_tma_1d_kernel<M, N, K, P, TEAMS, false, kRot>;
  if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM) != cudaSuccess)
    return KAMI_ERROR_CUDA;
  int dev = 0, sms = 148, per_sm = 1;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, Cfg::THREADS, Cfg::SMEM) != cudaSuccess ||
      per_sm < 1)
    per_sm = 1;
  long long grid = (long long)sms * per_sm;
  const long long need = (batch + TEAMS - 1) / TEAMS;
  if (grid > need) grid = need;
  grid = apply_grid_cap(grid);
  fn<<<(unsigned)grid, Cfg::THREADS, Cfg::SMEM, stream>>>(prm);
  set_last_kernel(ptr ? (M == 64 ? "kami_dmma_tma_1d<64,ptr>" : M == 32 ? "kami_dmma_tma_1d<32,ptr>"
                                                                         : "kami_dmma_tma_1d<16,ptr>")
                      : name);
  return cudaGetLastError() == cudaSuccess ? KAMI_SUCCESS : KAMI_ERROR_CUDA;
}

}  // namespace

bool dmma_tma_supported(int m, int n, int k) { return m == n && n == k && (m == 16 || m == 32 || m == 64); }

// (p, teams) configuration; env KAMI_DMMA_TMA_CFG = 1/2/3/4 picks an alternative for sweeps
// (64^3 default rotates B half an entry ahead: 25.3 -> 26.1 TF/s, profiles/r1/dmma_tma_sweep_r1.txt;
// at 16^3 / 32^3 it made no difference and the plain form stays)
kami_status_t dmma_tma_launch(int m, int n, int k, long long batch, const void* A, const void* B, void* C,
                              cudaStream_t stream, double alpha, double beta, const void* const* Aa,
                              const void* const* Ba, void* const* Ca) {
  static const int cfg = [] {
    const char* e = getenv("KAMI_DMMA_TMA_CFG");
    return e ? atoi(e) : 0;
  }();
  if (m == 64 && n == 64 && k == 64) {
    if (cfg == 1) return launch<64, 64, 64, 8, 2>(batch, A, B, C, stream, "kami_dmma_tma_1d<64,p8>", alpha, beta, Aa, Ba, Ca);
    if (cfg == 4) return launch<64, 64, 64, 4, 3>(batch, A, B, C, stream, "kami_dmma_tma_1d<64,norot>", alpha, beta, Aa, Ba, Ca);
    return launch<64, 64, 64, 4, 3, true>(batch, A, B, C, stream, "kami_dmma_tma_1d<64>", alpha, beta, Aa, Ba, Ca);
  }
  if (m == 32 && n == 32 && k == 32) {
    if (cfg == 3) return launch<32, 32, 32, 4, 8, true>(batch, A, B, C, stream, "kami_dmma_tma_1d<32,rot>", alpha, beta, Aa, Ba, Ca);
    if (cfg == 1) return launch<32, 32, 32, 2, 8>(batch, A, B, C, stream, "kami_dmma_tma_1d<32,p2>", alpha, beta, Aa, Ba, Ca);
    if (cfg == 2) return launch<32, 32, 32, 4, 6>(batch, A, B, C, stream, "kami_dmma_tma_1d<32,t6>", alpha, beta, Aa, Ba, Ca);
    return launch<32, 32, 32, 4, 8>(batch, A, B, C, stream, "kami_dmma_tma_1d<32>", alpha, beta, Aa, Ba, Ca);
  }
  if (m == 16 && n == 16 && k == 16) {
    if (cfg == 3) return launch<16, 16, 16, 2, 8, true>(batch, A, B, C, stream, "kami_dmma_tma_1d<16,rot>", alpha, beta, Aa, Ba, Ca);
    if (cfg == 1) return launch<16, 16, 16, 1, 15>(batch, A, B, C, stream, "kami_dmma_tma_1d<16,p1>", alpha, beta, Aa, Ba, Ca);
    return launch<16, 16, 16, 2, 8>(batch, A, B, C, stream, "kami_dmma_tma_1d<16>", alpha, beta, Aa, Ba, Ca);
  }
  return KAMI_ERROR_NOT_SUPPORTED;
}

}  // namespace kami
