// dmma_gen.cu -- FP64 batched GEMM for the whole FP64 size grid (m, n, k
// multiples of 8 in [8, 256], non-square included): KAMI-1D on the DMMA path
// with k-slicing and a register / shared-memory RESIDENCY RATIO (PAPER.md
// Sec. 4.7 "when the matrix order grows ... a preset fraction of the
// local tile stays in registers and the rest is parked in shared memory";
// Sec. 5.2.5: the best ratio depends on the order -- parking 50 % at
// order 128 gives 1.34x, parking 75 % gives 0.71x).  SURVEY.md 8(a) row a7.
//
// Schedule (as dmma_tma.cu, on C^T = B^T A^T): a team of P = 4 warps owns one
// unit = (entry, 64-column block of C).  Warp w holds its column slice
// B_w = B[:, nb 64 + 16 w : +16] -- the LOCAL operand -- for the whole unit:
//   k-steps [0, rs)  resident in registers (DMMA B fragments),
//   k-steps [rs, ks) parked in the warp's private shared-memory slab (written
//                    once per unit in fragment order, so every read is one
//                    conflict-free LDS.64 per lane),
// with rs = ratio * ks (ks = k / 4 DMMA k-steps; at most kRK resident).  A is
// the broadcast operand: TM-row blocks of A (all of k) arrive by TMA in the
// 128-byte swizzled layout (double-buffered per team, the next block's copy
// overlaps the current block's MMAs) and all four warps read their A
// fragments from there.  C_w blocks (TM x 16) accumulate in registers and are
// stored straight from the fragments.  Every shape is one kernel; m, n and
// k tails are TMA zero-fill (A) and per-fragment guards (B, C).  A's k range
// is cut into swizzle chunks of 16 doubles (128-byte swizzle) when k % 16 == 0
// and of 8 doubles (64-byte swizzle) otherwise, so a box never reaches past
// its row.
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

constexpr int kGP = 4;    // warps per team
constexpr int kGFN = 2;   // 8-wide n-fragments per warp (16 columns)
constexpr int kGNB = kGP * kGFN * 8;  // 64 columns per unit
constexpr int kGTM = 32;  // A / C rows per block
constexpr int kGFM = kGTM / 8;
constexpr int kRK = 32;   // max resident k-steps (32 x 2 doubles = 128 registers)
constexpr int kRKSmall = 8;  // k <= 32: 16 registers of B, four teams per SM
constexpr int kGenSmem = 232448;

// k index lane t supplies in k-step kk: with 16-double swizzle chunks the
// bank-conflict-free order of dmma_tma.cu (units a and a ^ 4 per k-step);
// with 8-double chunks (64-byte swizzle) the natural order
__device__ __forceinline__ int kcol(int kk, int t, int ce_shift) {
  return ce_shift == 4 ? ((kk >> 2) << 4) + ((kk & 3) << 1) + (t & 1) + ((t >> 1) << 3) : kk * 4 + t;
}

struct DmmaGenParams {
  CUtensorMap tmA;  // 4-D (CE, m, k/CE, batch), box (CE, TM, k/CE, 1), CE = 16 (SW128) or 8 (SW64) doubles
  const double* B;
  double* C;
  long long batch, units;
  int m, n, k, ks, rs, nblocks, mblocks, kch;
  int ce_shift;       // log2 of the chunk width in doubles (4: 128-byte rows, 3: 64-byte rows)
  uint32_t swz_bits;  // 3 (SW128) or 2 (SW64)
  uint32_t a_block_bytes, park_bytes;  // per team buffer / per warp slab
  int teams;
  int nbuf;  // A blocks in flight per team (2 or 3)
  // pointer arrays (kPtr; kami_gemm_batched): entry e at Aa[e], Ba[e], Ca[e]
  // (device).  A blocks are copied by the team with 16-byte cp.async into the
  // same swizzled layout the TMA box writes (rows past m zero-filled): a TMA
  // view box could not stay inside an entry whose m is not a multiple of 32.
  const double* const* Aa;
  const double* const* Ba;
  double* const* Ca;
  // variable sizes (kami_gemm_vbatched; pointer arrays): per-entry m, n, k in
  // device arrays, units enumerated as (entry, 64-column block < max n); a
  // unit past its entry's n, or an entry off the FP64 grid, is skipped
  const int* dm;
  const int* dn;
  const int* dk;
  // unit records written by a pre-pass (gen_vb_units): {entry, 64-column
  // block, m | n << 16, k} of every live unit, *count of them -- no dead
  // units to walk and one load per unit
  const int4* recs;
  const int* count;
};

// an entry's sizes and the quantities the kernel derives from them
struct GenDims {
  int m, n, k, ks, rs, mblocks, ce_shift;
  uint32_t swz_bits;
};
__device__ __forceinline__ void gen_derive(const DmmaGenParams& p, GenDims& d) {
  d.ks = d.k / 4;
  d.rs = d.ks < p.rs ? d.ks : p.rs;  // the plan's resident count is for the largest k
  d.ce_shift = (d.k % 16 == 0) ? 4 : 3;
}
__device__ __forceinline__ GenDims gen_dims(const DmmaGenParams& p, long long e) {
  GenDims d;
  if (p.dm) {
    d.m = __ldg(p.dm + e);
    d.n = __ldg(p.dn + e);
    d.k = __ldg(p.dk + e);
    gen_derive(p, d);
  } else {
    d.m = p.m;
    d.n = p.n;
    d.k = p.k;
    d.ks = p.ks;
    d.rs = p.rs;
    d.ce_shift = p.ce_shift;
  }
  d.mblocks = (d.m + kGTM - 1) / kGTM;
  d.swz_bits = d.ce_shift == 4 ? 3u : 2u;
  return d;
}
// a unit with work: its 64-column block inside the entry's n, the entry on the grid
__device__ __forceinline__ bool gen_live(const DmmaGenParams& p, const GenDims& d, int nb);
// unit u -> entry, column block, sizes, live
struct GenUnit {
  long long e;
  int nb;
  GenDims d;
  bool live;
};
__device__ __forceinline__ GenUnit gen_unit_rec(const DmmaGenParams& p, const int4 q);
__device__ __forceinline__ GenUnit gen_unit(const DmmaGenParams& p, long long u) {
  GenUnit r;
  if (p.recs) return gen_unit_rec(p, __ldg(p.recs + u));
  {
    r.e = u / p.nblocks;
    r.nb = (int)(u - r.e * p.nblocks);
    r.d = gen_dims(p, r.e);
    r.live = gen_live(p, r.d, r.nb);
  }
  return r;
}
// a unit record already in registers (loaded a unit earlier by the consumer)
__device__ __forceinline__ GenUnit gen_unit_rec(const DmmaGenParams& p, const int4 q) {
  GenUnit r;
  {
    r.e = q.x;
    r.nb = q.y;
    r.d.m = q.z & 0xFFFF;
    r.d.n = q.z >> 16;
    r.d.k = q.w;
    gen_derive(p, r.d);
    r.d.mblocks = (r.d.m + kGTM - 1) / kGTM;
    r.d.swz_bits = r.d.ce_shift == 4 ? 3u : 2u;
    r.live = true;
  }
  return r;
}
__device__ __forceinline__ bool gen_live(const DmmaGenParams& p, const GenDims& d, int nb) {
  if (!p.dm) return true;
  const bool grid = d.m >= 8 && d.n >= 8 && d.k >= 8 && d.m <= 256 && d.n <= 256 && d.k <= 256 &&
                    d.m % 8 == 0 && d.n % 8 == 0 && d.k % 8 == 0 && d.k <= p.k && d.n <= p.n && d.m <= p.m;
  return grid && nb * kGNB < d.n;
}

template <int RK, bool kPtr>
__global__ void __launch_bounds__(RK == kRK ? kGP * 32 * 2 : kGP * 32 * 4, 1)
    kami_dmma_gen_kernel(const __grid_constant__ DmmaGenParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int team = warp / kGP, w = warp % kGP;
  const int g = lane >> 2, t = lane & 3;
  // per team: nbuf A blocks, then the four warps' parked slabs; barriers at the end
  const uint32_t team_bytes = p.nbuf * p.a_block_bytes + kGP * p.park_bytes;
  uint8_t* tbase = smem + team * team_bytes;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + p.teams * team_bytes) + team * 3;
  if (threadIdx.x == 0) {
    ptx::prefetch_tmap(&p.tmA);
    for (int i = 0; i < 3 * p.teams; ++i)  // TMA: one expect_tx arrival; cp.async: the team's 128 threads
      ptx::mbar_init(reinterpret_cast<uint64_t*>(smem + p.teams * team_bytes) + i, kPtr ? kGP * 32 : 1);
    ptx::fence_mbar_init();
    ptx::fence_proxy_async_smem();
  }
  __syncthreads();
  if (team >= p.teams) return;
  const long long units = p.recs ? (long long)*p.count : p.units;
  const long long nteams = (long long)gridDim.x * p.teams;
  const long long first = (long long)blockIdx.x * p.teams + team;
  const bool issuer = (w == 0 && lane == 0);
  const uint32_t bar = 1 + team;
  const uint32_t park = ptx::smem_u32(tbase + p.nbuf * p.a_block_bytes + w * p.park_bytes);
  // the team's block sequence: units u = first, first + nteams, ...; m-blocks 0.. of each
  const int tid = w * 32 + lane;  // 0..127 within the team
  auto issue = [&](long long e, int mb, int s, const GenDims& d) {
    if constexpr (kPtr) {  // every thread of the team: 16-byte chunks of the 32 x k block
      const double* Ae = p.Aa[e];
      const uint32_t dst0 = ptx::smem_u32(tbase + s * p.a_block_bytes);
      const int cpr = d.k >> 1;  // 16-byte chunks per row
      const uint32_t rowb = 8u << d.ce_shift;
      for (int i = tid; i < kGTM * cpr; i += kGP * 32) {
        const int r = i / cpr, c = i - r * cpr;  // row, chunk (two doubles)
        const int col = 2 * c;
        const int row = mb * kGTM + r;
        const uint32_t off = (uint32_t)(col >> d.ce_shift) * (kGTM * rowb) +
                             ptx::swz((uint32_t)r * rowb + (uint32_t)(col & ((1 << d.ce_shift) - 1)) * 8, d.swz_bits);
        const bool ok = row < d.m;
        ptx::cp_async_16(dst0 + off, ok ? Ae + (long long)row * d.k + col : Ae, ok ? 16u : 0u);
      }
      ptx::cp_async_mbar_arrive_noinc(&full[s]);
    } else {
      ptx::mbar_arrive_expect_tx(&full[s], p.a_block_bytes);
      ptx::tma_load_4d(tbase + s * p.a_block_bytes, &p.tmA, &full[s], 0, mb * kGTM, 0, (int)e);
    }
  };
  // the producer's cursor (pu, pmb) walks the live units' A blocks nbuf ahead
  // of the consumer; pd = the sizes of pu's entry
  long long pu = first;
  int pmb = 0;
  GenUnit pd{};
  auto skip_dead = [&]() {
    for (; pu < units; pu += nteams) {
      pd = gen_unit(p, pu);
      if (pd.live) break;
    }
  };
  auto advance = [&]() {
    if (++pmb == pd.d.mblocks) {
      pmb = 0;
      pu += nteams;
      skip_dead();
    }
  };
  // prologue: the first nbuf blocks
  skip_dead();
  if (issuer || kPtr) {
    for (int s = 0; s < p.nbuf && pu < units; ++s) {
      issue(pd.e, pmb, s, pd.d);
      advance();
    }
  }
  double b[RK][kGFN];
  RingPos ab;  // A buffer ring (slot, parity)
  // records: the next unit's record is loaded one unit ahead and decoded at
  // its turn (decoding right after the load put a global round trip on every
  // unit's critical path)
  int4 qn = make_int4(0, 0, 0, 0);
  if (p.recs && first < units) qn = __ldg(p.recs + first);
  for (long long u = first; u < units; u += nteams) {
    const GenUnit gu = p.recs ? gen_unit_rec(p, qn) : gen_unit(p, u);
    if (p.recs && u + nteams < units) qn = __ldg(p.recs + u + nteams);
    if (!gu.live) continue;  // (the producer cursor skips it too)
    const long long e = gu.e;
    const int nb = gu.nb;
    const GenDims d = gu.d;
    if (issuer && !p.dm && p.nblocks == 1 && u + nteams < units) {  // the next unit's B into L2 while this one computes
      const long long en = (u + nteams) / p.nblocks;
      ptx::prefetch_l2_bulk(kPtr ? p.Ba[en] : p.B + en * (long long)p.k * p.n, (uint32_t)(p.k * p.n * 8));
    }
    const int col0 = nb * kGNB + w * (kGFN * 8);
    const double* Bg = kPtr ? p.Ba[e] : p.B + e * (long long)p.k * p.n;
    const int n_e = d.n, ks_e = d.ks, rs_e = d.rs, ce_e = d.ce_shift;
    // GMem2Reg: the resident k-steps of B_w; the parked ones go to this warp's slab
#pragma unroll
    for (int kk = 0; kk < RK; ++kk)
#pragma unroll
      for (int j = 0; j < kGFN; ++j) {
        const int col = col0 + j * 8 + g;
        b[kk][j] = (kk < rs_e && col0 + j * 8 < n_e) ? __ldg(Bg + kcol(kk, t, ce_e) * (long long)n_e + col)
                                                      : 0.0;
      }
    for (int kk = rs_e; kk < ks_e; ++kk)
#pragma unroll
      for (int j = 0; j < kGFN; ++j) {
        const int col = col0 + j * 8 + g;
        const double v = col0 + j * 8 < n_e ? __ldg(Bg + kcol(kk, t, ce_e) * (long long)n_e + col) : 0.0;
        asm volatile("st.shared.f64 [%0], %1;" ::"r"(park + (uint32_t)(((kk - rs_e) * kGFN + j) * 32 + lane) * 8),
                     "d"(v)
                     : "memory");
      }
    __syncwarp();
    for (int mb = 0; mb < d.mblocks; ++mb, ab.next(p.nbuf)) {
      const uint32_t s = ab.s;
      double c[kGFM][kGFN][2];
#pragma unroll
      for (int i = 0; i < kGFM; ++i)
#pragma unroll
        for (int j = 0; j < kGFN; ++j) c[i][j][0] = c[i][j][1] = 0.0;
      ptx::mbar_wait(&full[s], ab.ph);
      const uint32_t a_s = ptx::smem_u32(tbase + s * p.a_block_bytes);
      const uint32_t rowb = 8u << ce_e;  // bytes of one swizzled row of a chunk
      auto step = [&](int kk, const double (&bb)[kGFN]) {
        const int col = kcol(kk, t, ce_e);
        const uint32_t chunk_off = (uint32_t)(col >> ce_e) * (kGTM * rowb);
        const uint32_t in_row = (uint32_t)(col & ((1 << ce_e) - 1)) * 8;
#pragma unroll
        for (int i = 0; i < kGFM; ++i) {
          const int row = i * 8 + g;
          double a;
          asm volatile("ld.shared.f64 %0, [%1];"
                       : "=d"(a)
                       : "r"(a_s + chunk_off + ptx::swz(row * rowb + in_row, d.swz_bits)));
#pragma unroll
          for (int j = 0; j < kGFN; ++j)
            asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                         : "+d"(c[i][j][0]), "+d"(c[i][j][1])
                         : "d"(a), "d"(bb[j]));
        }
      };
      // resident k-steps: B fragments from registers
#pragma unroll
      for (int kk = 0; kk < RK; ++kk)
        if (kk < rs_e) step(kk, b[kk]);
      // parked k-steps: B fragments from the warp's slab (one LDS.64 per fragment)
#pragma unroll 4
      for (int kk = rs_e; kk < ks_e; ++kk) {
        double bb[kGFN];
#pragma unroll
        for (int j = 0; j < kGFN; ++j)
          asm volatile("ld.shared.f64 %0, [%1];"
                       : "=d"(bb[j])
                       : "r"(park + (uint32_t)(((kk - rs_e) * kGFN + j) * 32 + lane) * 8));
        step(kk, bb);
      }
      // Reg2GMem: C_w block; lane holds (row g, cols 2t, 2t+1) of each 8x8 fragment
      double* Cg = kPtr ? p.Ca[e] : p.C + e * (long long)p.m * p.n;
#pragma unroll
      for (int i = 0; i < kGFM; ++i) {
        const int row = mb * kGTM + i * 8 + g;
#pragma unroll
        for (int j = 0; j < kGFN; ++j)
          if (row < d.m && col0 + j * 8 < n_e)
            ptx::st_global_v2_f64(Cg + (long long)row * n_e + col0 + j * 8 + 2 * t, c[i][j][0], c[i][j][1]);
      }
      ptx::named_bar_sync(bar, kGP * 32);  // every warp finished reading buffer s
      if ((issuer || kPtr) && pu < units) {  // refill it with the block nbuf ahead
        issue(pd.e, pmb, s, pd.d);
        advance();
      }
    }
  }
}

// Residency ratio: share of the ks k-steps of B_w kept in
// registers.  Default: as many as fit (kRK), i.e. 100 % up to k = 128, 50 %
// at k = 256.  KAMI_F64_RESIDENT_PCT overrides it (sweeps, tools/residency_sweep.py).
uint32_t align1k(uint32_t x) { return (x + 1023) / 1024 * 1024; }

// Plan of one launch: resident k-steps, register template, teams per CTA and
// shared-memory bytes.  The parked slabs must fit next to the A double buffer:
// a ratio that parks more than fits is raised to the smallest that fits.
struct GenPlan {
  int rk, rs, teams, ce_shift, nbuf;
  uint32_t a_block_bytes, park_bytes, smem;
};
GenPlan gen_plan(int m, int n, int k) {
  GenPlan g;
  const int ks = k / 4;
  g.ce_shift = (k % 16 == 0) ? 4 : 3;
  g.rk = ks <= kRKSmall ? kRKSmall : kRK;
  // read per call (not cached) so one process can sweep the ratio
  const char* env = getenv("KAMI_F64_RESIDENT_PCT");
  const int pct = env ? atoi(env) : -1;
  int rs = pct < 0 ? ks : (ks * pct + 50) / 100;
  if (rs > g.rk) rs = g.rk;
  if (rs > ks) rs = ks;
  if (rs < 0) rs = 0;
  g.a_block_bytes = align1k((uint32_t)(kGTM * k * 8));
  const int slab_step = kGFN * 32 * 8;  // bytes per parked k-step per warp
  const int room = (kGenSmem - 1024 - 64 - 2 * (int)g.a_block_bytes) / (kGP * slab_step);
  if (ks - rs > room) rs = ks - room;
  g.rs = rs;
  g.park_bytes = (uint32_t)((ks - rs) * slab_step);
  // three A blocks in flight when they fit next to the slabs (one more TMA
  // round trip of slack per team), else two
  g.nbuf = (3 * g.a_block_bytes + kGP * g.park_bytes + 1024 + 96 <= (uint32_t)kGenSmem) ? 3 : 2;
  const uint32_t team_bytes = g.nbuf * g.a_block_bytes + kGP * g.park_bytes;
  const int max_teams = g.rk == kRK ? 2 : 4;
  g.teams = 1;
  while (g.teams < max_teams && (g.teams + 1) * team_bytes + 1024 + 96 <= (uint32_t)kGenSmem) ++g.teams;
  g.smem = g.teams * team_bytes + 1024 /*align*/ + 96 /*barriers*/;
  return g;
}

}  // namespace

bool dmma_gen_supported(int m, int n, int k) {
  return m >= 8 && n >= 8 && k >= 8 && m <= 256 && n <= 256 && k <= 256 && m % 8 == 0 && n % 8 == 0 && k % 8 == 0;
}

int dmma_gen_resident_pct(int k) { return 100 * gen_plan(k, k, k).rs / (k / 4); }

kami_status_t dmma_gen_launch(int m, int n, int k, long long batch, const void* A, const void* B, void* C,
                              cudaStream_t stream, const void* const* Aa, const void* const* Ba, void* const* Ca) {
  if (!dmma_gen_supported(m, n, k)) return KAMI_ERROR_NOT_SUPPORTED;
  const bool ptr = Aa != nullptr;
  if (ptr && (!Ba || !Ca)) return KAMI_ERROR_INVALID_VALUE;
  PFN_encodeTiled enc = get_encode_tiled();
  if (!enc) return KAMI_ERROR_CUDA;
  DmmaGenParams p;
  memset(&p, 0, sizeof(p));
  p.Aa = reinterpret_cast<const double* const*>(Aa);
  p.Ba = reinterpret_cast<const double* const*>(Ba);
  p.Ca = reinterpret_cast<double* const*>(Ca);
  p.B = static_cast<const double*>(B);
  p.C = static_cast<double*>(C);
  p.batch = batch;
  p.m = m;
  p.n = n;
  p.k = k;
  p.ks = k / 4;
  const GenPlan gp = gen_plan(m, n, k);
  if (gp.smem > (uint32_t)kGenSmem) return KAMI_ERROR_NOT_SUPPORTED;
  p.rs = gp.rs;
  p.nblocks = (n + kGNB - 1) / kGNB;
  p.mblocks = (m + kGTM - 1) / kGTM;
  p.ce_shift = gp.ce_shift;
  p.swz_bits = gp.ce_shift == 4 ? 3 : 2;
  const int ce = 1 << p.ce_shift;
  p.kch = k / ce;
  p.units = batch * p.nblocks;
  p.a_block_bytes = gp.a_block_bytes;
  p.park_bytes = gp.park_bytes;
  p.teams = gp.teams;
  p.nbuf = gp.nbuf;
  const uint32_t smem = gp.smem;
  if (!ptr) {  // A: (CE doubles, m, k/CE chunks, batch), box (CE, TM, k/CE, 1); rows past m zero-filled
    cuuint64_t dims[4] = {(cuuint64_t)ce, (cuuint64_t)m, (cuuint64_t)p.kch, (cuuint64_t)batch};
    cuuint64_t strides[3] = {(cuuint64_t)k * 8, (cuuint64_t)ce * 8, (cuuint64_t)m * k * 8};
    cuuint32_t box[4] = {(cuuint32_t)ce, (cuuint32_t)kGTM, (cuuint32_t)p.kch, 1};
    cuuint32_t es[4] = {1, 1, 1, 1};
    if (enc(&p.tmA, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, const_cast<void*>(A), dims, strides, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, ce == 16 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  auto fn = ptr ? (gp.rk == kRK ? kami_dmma_gen_kernel<kRK, true> : kami_dmma_gen_kernel<kRKSmall, true>)
                : (gp.rk == kRK ? kami_dmma_gen_kernel<kRK, false> : kami_dmma_gen_kernel<kRKSmall, false>);
  if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return KAMI_ERROR_CUDA;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const long long need = (p.units + p.teams - 1) / p.teams;
  long long grid = sms < need ? sms : need;
  grid = apply_grid_cap(grid);
  fn<<<(unsigned)grid, kGP * 32 * (gp.rk == kRK ? 2 : 4), smem, stream>>>(p);
  set_last_kernel(ptr ? "kami_dmma_gen_1d<ptr>" : "kami_dmma_gen_1d");
  return cudaGetLastError() == cudaSuccess ? KAMI_SUCCESS : KAMI_ERROR_CUDA;
}

// the live units of a variable-size batch as records, in three k buckets
// (k <= 32, k <= 128, k > 128: each launched with its own plan), by a
// warp-aggregated append per bucket
constexpr int kVbBuckets = 3;
__host__ __device__ __forceinline__ int gen_bucket(int k) { return k <= 32 ? 0 : k <= 128 ? 1 : 2; }
__global__ void gen_vb_units(long long batch, const int* dm, const int* dn, const int* dk, int max_m, int max_n,
                             int max_k, int4* recs, long long stride, int* count) {
  for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < batch;
       e += (long long)gridDim.x * blockDim.x) {
    const int m = __ldg(dm + e), n = __ldg(dn + e), k = __ldg(dk + e);
    const bool ok = m >= 8 && n >= 8 && k >= 8 && m <= max_m && n <= max_n && k <= max_k && m % 8 == 0 &&
                    n % 8 == 0 && k % 8 == 0;
    const int nb = ok ? (n + kGNB - 1) / kGNB : 0;
    const int bk = gen_bucket(k);
    const unsigned act = __activemask();
    const int lane = threadIdx.x & 31, last = 31 - __clz(act);
#pragma unroll
    for (int b = 0; b < kVbBuckets; ++b) {
      const int mine = bk == b ? nb : 0;
      int incl = mine;  // inclusive warp scan of this bucket's unit counts
      for (int o = 1; o < 32; o <<= 1) {
        const int v = __shfl_up_sync(act, incl, o);
        if (lane >= o) incl += v;
      }
      int base = 0;
      if (lane == last && incl) base = atomicAdd(count + b, incl);
      base = __shfl_sync(act, base, last) + incl - mine;
      for (int j = 0; j < mine; ++j) recs[b * stride + base + j] = make_int4((int)e, j, m | (n << 16), k);
    }
  }
}

// Variable sizes (kami_gemm_vbatched, FP64; "supports various
// matrix orders in a batch"): the pointer-array kernel with per-entry m, n, k
// read on the device, one launch per k bucket planned for (max_m, max_n,
// the bucket's largest k): the A buffers and parked slabs of a k <= 32 bucket
// leave four teams per SM where a plan for k = 256 leaves one.
kami_status_t dmma_gen_vb_launch(long long batch, const int* dm, const int* dn, const int* dk, int max_m, int max_n,
                                 int max_k, const void* const* Aa, const void* const* Ba, void* const* Ca,
                                 cudaStream_t stream) {
  if (!dmma_gen_supported(max_m, max_n, max_k)) return KAMI_ERROR_NOT_SUPPORTED;
  if (!dm || !dn || !dk || !Aa || !Ba || !Ca) return KAMI_ERROR_INVALID_VALUE;
  const int nbmax = (max_n + kGNB - 1) / kGNB;
  const long long stride = batch * nbmax;
  void* ws = nullptr;
  if (cudaMallocAsync(&ws, 16 + sizeof(int4) * (size_t)stride * kVbBuckets, stream) != cudaSuccess)
    return KAMI_ERROR_CUDA;
  int* count = static_cast<int*>(ws);
  int4* recs = reinterpret_cast<int4*>(static_cast<char*>(ws) + 16);
  cudaMemsetAsync(count, 0, sizeof(int) * kVbBuckets, stream);
  {
    const int blocks = (int)((batch + 255) / 256 < 1184 ? (batch + 255) / 256 : 1184);
    gen_vb_units<<<blocks, 256, 0, stream>>>(batch, dm, dn, dk, max_m, max_n, max_k, recs, stride, count);
  }
  cudaError_t le = cudaGetLastError();
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int kb_hi[kVbBuckets] = {32, 128, 256};
  for (int b = 0; b < kVbBuckets && le == cudaSuccess; ++b) {
    const int klo = b == 0 ? 8 : kb_hi[b - 1] + 8;
    if (max_k < klo) break;  // no entry can fall in this bucket
    const int kb = max_k < kb_hi[b] ? max_k : kb_hi[b];
    DmmaGenParams p;
    memset(&p, 0, sizeof(p));
    p.Aa = reinterpret_cast<const double* const*>(Aa);
    p.Ba = reinterpret_cast<const double* const*>(Ba);
    p.Ca = reinterpret_cast<double* const*>(Ca);
    p.dm = dm;
    p.dn = dn;
    p.dk = dk;
    p.batch = batch;
    p.m = max_m;
    p.n = max_n;
    p.k = kb;
    p.ks = kb / 4;
    const GenPlan gp = gen_plan(max_m, max_n, kb);
    if (gp.smem > (uint32_t)kGenSmem) {
      le = cudaErrorInvalidValue;
      break;
    }
    p.rs = gp.rs;
    p.nblocks = nbmax;
    p.mblocks = (max_m + kGTM - 1) / kGTM;
    p.ce_shift = gp.ce_shift;
    p.swz_bits = gp.ce_shift == 4 ? 3 : 2;
    p.units = stride;  // upper bound; the kernel reads the bucket's count
    p.a_block_bytes = gp.a_block_bytes;
    p.park_bytes = gp.park_bytes;
    p.teams = gp.teams;
    p.nbuf = gp.nbuf;
    p.recs = recs + b * stride;
    p.count = count + b;
    auto fn = gp.rk == kRK ? kami_dmma_gen_kernel<kRK, true> : kami_dmma_gen_kernel<kRKSmall, true>;
    if ((le = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)gp.smem)) != cudaSuccess)
      break;
    const long long need = (p.units + p.teams - 1) / p.teams;
    long long grid = sms < need ? sms : need;
    grid = apply_grid_cap(grid);
    fn<<<(unsigned)grid, kGP * 32 * (gp.rk == kRK ? 2 : 4), gp.smem, stream>>>(p);
    le = cudaGetLastError();
  }
  cudaFreeAsync(ws, stream);  // stream-ordered: after the kernels
  set_last_kernel("kami_dmma_gen_1d<vbatched>");
  return (kami_status_t)launch_status((int)le);
}

}  // namespace kami
