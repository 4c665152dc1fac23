// tc16_pair.cu -- KAMI-2D across a CTA PAIR on tcgen05 (cta_group::2),
// FP16 / BF16 in, FP32 accumulate, sm_100a.  DESIGN.md 4.1d.
//
// For the largest orders (192 < m <= 256) one SM's 128 TMEM lanes hold only
// half of an entry's rows, and the single-CTA kernel (tc16.cu) runs the two
// m-tiles of an entry as independent units that each stream ALL of B.  Here
// two SMs of a TPC form a cluster and split the entry the way Alg. 2 (PAPER.md
// L262-301) splits it over a sqrt(p) x sqrt(p) grid of compute units:
//   compute units  = 2 CTAs x 4 sub-partition tensor cores; CTA r owns rows
//                    [128 r, 128 r + 128) of A and C (its TMEM lanes; the
//                    row direction of the grid),
//   local storage  = CTA r's shared memory holds ITS half of B's columns,
//                    B[:, r n/2 : (r+1) n/2] (the column direction), and its
//                    A rows; each CTA loads only its own halves by TMA,
//   communication  = one tcgen05.mma.cta_group::2 (M = 256, issued by the
//                    leader CTA) reads both CTAs' B halves through the pair's
//                    shared memory: every B column block is broadcast to the
//                    other CTA's row block -- Alg. 2's B_{z,c} broadcast along
//                    the grid column, done by the tensor core.  A is never
//                    exchanged (it stays with the rows it produces).
// So each entry's A and B cross HBM and shared memory exactly once (the
// single-CTA kernel reads B once per m-tile), and each CTA stores its rows.
//
// Pipeline (persistent pairs, one entry per unit, k in chunks of Wk):
//   warp 0 (both CTAs)  TMA of the CTA's A rows and B columns into a stage;
//                       completion is signalled on the LEADER's full[s]
//                       (.cta_group::2 TMA), whose expect_tx counts both CTAs
//   warp 1 (leader)     tcgen05.mma.cta_group::2; commits multicast to both
//                       CTAs' empty[s] and, per unit, tfull[a]
//   warp 1 (both)       TMEM allocation (cta_group::2, 512 columns)
//   warps 2-9 (both)    epilogue: two warpgroups on alternate units; each warp
//                       drains its 32 rows atom by atom (tcgen05.ld -> cvt.rn
//                       -> swizzled st.shared -> its own TMA store) and arrives
//                       on the leader's tempty[a] (remote arrive for the peer)
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "kernels.h"
#include "ptx.cuh"
#include "sched.cuh"

namespace kami {
namespace {

constexpr int kPThreads = 320;
constexpr int kPMaxStages = 6;

struct alignas(64) PairParams {
  CUtensorMap tmA;  // 3-D (k, m, batch), box (Wk, 128, 1)
  CUtensorMap tmB;  // 4-D (Wn, k, n/Wn, batch), box (Wn, Wk, (n/2)/Wn, 1)
  CUtensorMap tmC;  // 4-D (Wc, m, n/Wc, batch), box (Wc, 32, 1, 1): one warp's rows of one atom
  long long batch;
  int m, n, k, k_chunks, Wk, Wn, Wc, ksteps_full, ksteps_last;
  uint32_t idesc, a_layout, b_layout, a_sbo, b_lbo, b_sbo, b_kstep;
  uint32_t a_bytes, stage_bytes, tx_pair;
  int stages, acc_cols;
  uint32_t c_off, c_warp_bytes, bar_off, c_swz_bits;
  // kSparse: A in Z-Morton block storage (Sec. 4.6: the 2D
  // algorithm's storage).  CTA r's rows [128 r, 128 r + 128) are block rows
  // [8 r, 8 r + 8): with at most 16 block columns those blocks are exactly the
  // Morton codes [128 r, 128 r + 128) -- one contiguous range of the sorted
  // code array, found by binary search (the "efficient submatrix indexing")
  const int* nnzb;
  const int* zcode;
  const uint16_t* vals;
  int max_nnzb;
};

__device__ __forceinline__ uint32_t cta_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// address of the same shared variable in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t mapa(uint32_t saddr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
  return r;
}
__device__ __forceinline__ void mbar_arrive_cluster(uint32_t caddr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(caddr) : "memory");
}
// TMA whose completion is signalled on the pair leader's mbarrier
__device__ __forceinline__ void tma_load_3d_pair(uint32_t dst, const CUtensorMap* m, uint32_t bar, int c0, int c1,
                                                 int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cta.global.tile.mbarrier::complete_tx::bytes.cta_group::2"
      " [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(m)), "r"(bar), "r"(c0), "r"(c1), "r"(c2)
      : "memory");
}
__device__ __forceinline__ void tma_load_4d_pair(uint32_t dst, const CUtensorMap* m, uint32_t bar, int c0, int c1,
                                                 int c2, int c3) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cta.global.tile.mbarrier::complete_tx::bytes.cta_group::2"
      " [%0], [%1, {%3, %4, %5, %6}], [%2];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(m)), "r"(bar), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
      : "memory");
}
__device__ __forceinline__ void umma_pair(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
      "l"(a), "l"(b), "r"(idesc), "r"(acc)
      : "memory");
}
__device__ __forceinline__ void commit_pair(uint64_t* bar) {  // arrive on bar in both CTAs
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          ptx::smem_u32(bar)),
      "h"((uint16_t)3)
      : "memory");
}

// first index in the ascending codes zc[0, nz) whose value is >= v
__device__ __forceinline__ int lower_bound_dev(const int* zc, int nz, int v) {
  int lo = 0, hi = nz;
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if (__ldg(zc + mid) < v) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

template <int kBf16, bool kSparse>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kPThreads + (kSparse ? 128 : 0), 1)
    kami_tc16_pair_kernel(const __grid_constant__ PairParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (ptx::smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + p.bar_off);  // leader's are used
  uint64_t* empty = full + kPMaxStages;
  uint64_t* tfull = empty + kPMaxStages;
  uint64_t* tempty = tfull + 2;  // leader's are used
  uint64_t* afull = tempty + 2;  // kSparse: this CTA's A copies of stage s landed (32 cp.async lanes)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(afull + kPMaxStages);
  int* tab = reinterpret_cast<int*>(tmem_slot + 2);  // kSparse: [8 block rows][16 block cols] -> slot
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cta_rank();
  const long long pair = blockIdx.x >> 1, npairs = gridDim.x >> 1;

  if (threadIdx.x == 0) {
    if (!kSparse) ptx::prefetch_tmap(&p.tmA);
    ptx::prefetch_tmap(&p.tmB);
    ptx::prefetch_tmap(&p.tmC);
    for (int s = 0; s < p.stages; ++s) {
      // sparse: the leader's expect_tx (B) + the peer's relay of its A copies
      ptx::mbar_init(&full[s], kSparse ? 2 : 1);
      ptx::mbar_init(&empty[s], 1);
      ptx::mbar_init(&afull[s], 128);  // kSparse: the copier warpgroup
    }
    for (int a = 0; a < 2; ++a) {
      ptx::mbar_init(&tfull[a], 1);
      ptx::mbar_init(&tempty[a], 8);  // 4 epilogue warps x 2 CTAs
    }
    ptx::fence_mbar_init();
    ptx::fence_proxy_async_smem();
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(ptx::smem_u32(tmem_slot)),
                 "r"(512)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  ptx::tc_fence_before();
  cluster_sync();  // both CTAs' barriers initialised, TMEM allocated
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  const uint32_t smem_base = ptx::smem_u32(smem);

  if (kSparse && warp == 0) {
    // ------------------------------------- B TMA (both CTAs), sparse mode
    if (lane == 0) {
      RingPos r;
      const uint32_t full_leader = mapa(ptx::smem_u32(full), 0);
      for (long long e = pair; e < p.batch; e += npairs)
        for (int kc = 0; kc < p.k_chunks; ++kc, r.next(p.stages)) {
          ptx::mbar_wait(&empty[r.s], r.ph ^ 1);
          if (rank == 0) ptx::mbar_arrive_expect_tx(&full[r.s], p.tx_pair);
          tma_load_4d_pair(smem_base + r.s * p.stage_bytes + p.a_bytes, &p.tmB, full_leader + r.s * 8, 0,
                           kc * p.Wk, (int)rank * ((p.n >> 1) / p.Wn), (int)e);
        }
    }
  } else if (kSparse && warp >= kPThreads / 32) {
    // ------------- sparse A copier warpgroup (both CTAs): GMem2Reg + Reg2SMem
    const int tid = threadIdx.x - kPThreads;  // 0..127
    RingPos r;
    const int bcols = p.Wk >> 4;  // 16-column blocks per k-chunk
    const uint32_t a_bits = p.a_layout == 2 ? 3 : p.a_layout == 4 ? 2 : 1;
    const uint32_t wk_b = (uint32_t)p.Wk * 2;
    for (long long e = pair; e < p.batch; e += npairs) {
      // this CTA's blocks: Morton codes [128 rank, 128 rank + 128), one range
      const int* zc = p.zcode + e * (long long)p.max_nnzb;
      const int nz = __ldg(p.nnzb + e);
      const int lo = lower_bound_dev(zc, nz, 128 * (int)rank), hi = lower_bound_dev(zc, nz, 128 * (int)rank + 128);
      ptx::named_bar_sync(3, 128);  // the previous unit's copies are all issued: the table is free
      tab[tid] = -1;
      ptx::named_bar_sync(3, 128);
      for (int j = lo + tid; j < hi; j += 128) {
        const uint32_t z = (uint32_t)__ldg(zc + j);
        uint32_t br = 0, bc = 0;
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          bc |= ((z >> (2 * t)) & 1u) << t;
          br |= ((z >> (2 * t + 1)) & 1u) << t;
        }
        tab[(br & 7) * 16 + bc] = j;
      }
      ptx::named_bar_sync(3, 128);
      const uint16_t* ve = p.vals + e * (long long)p.max_nnzb * 256;
      for (int kc = 0; kc < p.k_chunks; ++kc, r.next(p.stages)) {
        ptx::mbar_wait(&empty[r.s], r.ph ^ 1);
        const uint32_t sa = smem_base + r.s * p.stage_bytes;
        // the present blocks densified into the K-major swizzled A tile
        // (absent blocks zero-filled); consecutive threads take consecutive
        // 16-byte chunks of a block (contiguous 512-byte block rows)
        for (int i = tid; i < 8 * bcols * 32; i += 128) {
          const int blk = i >> 5, ch = i & 31;
          const int lbr = blk / bcols, lbc = blk - lbr * bcols;
          const int slot = tab[lbr * 16 + kc * bcols + lbc];
          const int row = lbr * 16 + (ch >> 1), hh = ch & 1;
          const uint32_t dst = sa + ptx::swz((uint32_t)row * wk_b + (uint32_t)(lbc * 2 + hh) * 16, a_bits);
          const bool ok = slot >= 0;
          ptx::cp_async_16(dst, ok ? ve + (long long)slot * 256 + (ch >> 1) * 16 + hh * 8 : ve, ok ? 16u : 0u);
        }
        ptx::cp_async_mbar_arrive_noinc(&afull[r.s]);
      }
    }
    ptx::cp_async_wait<0>();
  } else if (kSparse && warp == 1 && rank == 1) {
    // ------------------ relay: the peer's A copies of stage s -> leader's full[s]
    if (lane == 0) {
      RingPos r;
      const uint32_t full_leader = mapa(ptx::smem_u32(full), 0);
      for (long long e = pair; e < p.batch; e += npairs)
        for (int kc = 0; kc < p.k_chunks; ++kc, r.next(p.stages)) {
          ptx::mbar_wait(&afull[r.s], r.ph);
          ptx::fence_proxy_async_smem();  // generic (cp.async) writes -> the tensor core's async-proxy reads
          mbar_arrive_cluster(full_leader + r.s * 8);
        }
    }
  } else if (warp == 0) {
    // ---------------------------------------------- TMA (both CTAs)
    if (lane == 0) {
      RingPos r;
      const uint32_t full_leader = mapa(ptx::smem_u32(full), 0);  // full[0] of the leader
      for (long long e = pair; e < p.batch; e += npairs) {
        for (int kc = 0; kc < p.k_chunks; ++kc, r.next(p.stages)) {
          ptx::mbar_wait(&empty[r.s], r.ph ^ 1);
          if (rank == 0) ptx::mbar_arrive_expect_tx(&full[r.s], p.tx_pair);
          const uint32_t bar = full_leader + r.s * 8;
          const uint32_t sa = smem_base + r.s * p.stage_bytes;
          tma_load_3d_pair(sa, &p.tmA, bar, kc * p.Wk, (int)rank * 128, (int)e);
          tma_load_4d_pair(sa + p.a_bytes, &p.tmB, bar, 0, kc * p.Wk, (int)rank * ((p.n >> 1) / p.Wn), (int)e);
        }
      }
    }
  } else if (warp == 1) {
    // ---------------------------------------------- MMA (leader only)
    if (rank == 0) {
      RingPos rb, ra;
      const uint64_t adesc0 = ptx::make_smem_desc(smem_base, 16, p.a_sbo, p.a_layout);
      const uint64_t bdesc0 = ptx::make_smem_desc(smem_base + p.a_bytes, p.b_lbo, p.b_sbo, p.b_layout);
      const uint32_t stage16 = p.stage_bytes >> 4, bstep16 = p.b_kstep >> 4;
      for (long long e = pair; e < p.batch; e += npairs, ra.next(2)) {
        ptx::mbar_wait(&tempty[ra.s], ra.ph ^ 1);
        ptx::tc_fence_after();
        const uint32_t d = tmem_base + ra.s * p.acc_cols;
        for (int kc = 0; kc < p.k_chunks; ++kc, rb.next(p.stages)) {
          ptx::mbar_wait(&full[rb.s], rb.ph);
          if constexpr (kSparse) {  // the leader's own A copies
            ptx::mbar_wait(&afull[rb.s], rb.ph);
            ptx::fence_proxy_async_smem();
          }
          ptx::tc_fence_after();
          if (lane == 0) {
            const int nst = kc == p.k_chunks - 1 ? p.ksteps_last : p.ksteps_full;
            const uint64_t ad = adesc0 + rb.s * stage16, bd = bdesc0 + rb.s * stage16;
            for (int ks = 0; ks < nst; ++ks) umma_pair(d, ad + 2 * ks, bd + bstep16 * ks, p.idesc, (kc | ks) != 0);
            commit_pair(&empty[rb.s]);  // both CTAs' stage s is free once these MMAs retire
          }
          __syncwarp();
        }
        if (lane == 0) commit_pair(&tfull[ra.s]);  // accumulator ready in both CTAs
        __syncwarp();
      }
    }
  } else {
    // ---------------------------------------------- epilogue (both CTAs)
    const int wg = (warp - 2) >> 2;
    const int sp = warp & 3;  // TMEM sub-partition = rows 32 sp .. of this CTA's 128
    const uint32_t row_bytes = (uint32_t)p.Wc * 2;
    const uint32_t cbuf0 = smem_base + p.c_off + (uint32_t)(warp - 2) * 2 * p.c_warp_bytes;
    uint8_t* cbuf0_ptr = smem + p.c_off + (warp - 2) * 2 * p.c_warp_bytes;
    const uint32_t tempty_leader = mapa(ptx::smem_u32(tempty), 0);
    const int atoms = p.n / p.Wc;
    uint32_t a = wg, aph = 0, cb = 0;
    const int row0 = (int)rank * 128 + sp * 32;
    for (long long e = pair + (long long)wg * npairs; e < p.batch; e += 2 * npairs) {
      ptx::mbar_wait(&tfull[a], aph);
      ptx::tc_fence_after();
      const uint32_t t_row = tmem_base + (uint32_t(sp * 32) << 16) + a * p.acc_cols;
      const bool live = row0 < p.m;
      for (int at = 0; at < atoms; ++at) {
        uint32_t v[64];
        const int cols = p.Wc;  // 16, 32 or 64
        if (cols == 64) {
          ptx::tmem_ld_32x32b_x32(t_row + at * 64, *reinterpret_cast<uint32_t(*)[32]>(&v[0]));
          ptx::tmem_ld_32x32b_x32(t_row + at * 64 + 32, *reinterpret_cast<uint32_t(*)[32]>(&v[32]));
        } else if (cols == 32) {
          ptx::tmem_ld_32x32b_x32(t_row + at * 32, *reinterpret_cast<uint32_t(*)[32]>(&v[0]));
        } else {
          ptx::tmem_ld_32x32b_x16(t_row + at * 16, *reinterpret_cast<uint32_t(*)[16]>(&v[0]));
        }
        ptx::tmem_wait_ld();
        if (at == atoms - 1) {  // accumulator drained: the leader may reuse it
          ptx::tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive_cluster(tempty_leader + a * 8);
        }
        if (!live) continue;
        // this warp's staging buffer cb must have been read out by its previous store
        if (lane == 0) ptx::bulk_wait_read<1>();
        __syncwarp();
        const uint32_t cbase = cbuf0 + cb * p.c_warp_bytes;
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          if (8 * q < cols) {
            uint32_t w[4];
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              const float lo = __uint_as_float(v[8 * q + 2 * i]), hi = __uint_as_float(v[8 * q + 2 * i + 1]);
              w[i] = kBf16 ? ptx::pack_bf16x2(lo, hi) : ptx::pack_f16x2(lo, hi);
            }
            ptx::st_shared_v4(cbase + ptx::swz((uint32_t)lane * row_bytes + 16 * q, p.c_swz_bits), w[0], w[1], w[2],
                              w[3]);
          }
        }
        ptx::fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) {
          ptx::tma_store_4d(&p.tmC, cbuf0_ptr + cb * p.c_warp_bytes, 0, row0, at, (int)e);
          ptx::bulk_commit();
        }
        cb ^= 1;
      }
      a += 2;
      if (a >= 2) {
        a -= 2;
        aph ^= 1;
      }
    }
    if (lane == 0) ptx::bulk_wait<0>();
  }

  ptx::tc_fence_before();
  cluster_sync();
  ptx::tc_fence_after();
  if (warp == 1) asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(512)
                              : "memory");
}

int pr_atom(int bytes) { return bytes % 128 == 0 ? 128 : bytes % 64 == 0 ? 64 : bytes % 32 == 0 ? 32 : 0; }
CUtensorMapSwizzle pr_swz(int atom) {
  return atom == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : atom == 64 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_32B;
}
uint32_t pr_align(uint32_t x) { return (x + 1023) / 1024 * 1024; }

}  // namespace

bool tc16_pair_supported(int m, int n, int k) {
  if (m <= 128 || m > 256 || n < 32 || n > 256 || k < 8 || k > 256) return false;
  if (m % 16 || n % 32 || k % 8) return false;
  const int kpad = (k + 15) / 16 * 16;
  return pr_atom(kpad * 2) && pr_atom(n) /* (n/2) * 2 bytes */ && pr_atom(n * 2);
}

kami_status_t tc16_pair_launch(int m, int n, int k, long long batch, bool bf16, const void* A, const void* B, void* C,
                               cudaStream_t stream, const int* nnzb, const int* zcode, const void* vals,
                               int max_nnzb) {
  if (!tc16_pair_supported(m, n, k)) return KAMI_ERROR_NOT_SUPPORTED;
  const bool sparse = zcode != nullptr;
  if (sparse && (k % 16 || !nnzb || !vals)) return KAMI_ERROR_NOT_SUPPORTED;
  PFN_encodeTiled enc = get_encode_tiled();
  if (!enc) return KAMI_ERROR_CUDA;
  PairParams p;
  memset(&p, 0, sizeof(p));
  const int kpad = (k + 15) / 16 * 16;
  const int wk_b = pr_atom(kpad * 2), wn_b = pr_atom(n), wc_b = pr_atom(n * 2);  // B half: n/2 columns
  p.batch = batch;
  p.m = m;
  p.n = n;
  p.k = k;
  p.Wk = wk_b / 2;
  p.Wn = wn_b / 2;
  p.Wc = wc_b / 2;
  p.k_chunks = (kpad + p.Wk - 1) / p.Wk;
  p.ksteps_full = wk_b / 32;
  p.ksteps_last = (kpad - (p.k_chunks - 1) * p.Wk) / 16;
  // M = 256 across the pair, N = n (each CTA's smem holds n/2 of B's columns)
  p.idesc = ptx::make_idesc_f16(bf16 ? 1 : 0, 256, n, 0, 1);
  p.a_layout = ptx::umma_layout_code(wk_b);
  p.b_layout = ptx::umma_layout_code(wn_b);
  p.a_sbo = 8 * wk_b;
  p.b_sbo = 8 * wn_b;
  p.b_lbo = p.Wk * wn_b;
  p.b_kstep = 2 * p.b_sbo;
  p.a_bytes = pr_align(128 * wk_b);
  p.stage_bytes = p.a_bytes + pr_align((uint32_t)(n / 2) * wk_b);
  // (sparse: only B arrives by TMA; A by the producer warps' cp.async)
  p.tx_pair = sparse ? 2 * (uint32_t)((n / 2) * wk_b) : 2 * (uint32_t)(128 * wk_b + (n / 2) * wk_b);
  p.nnzb = nnzb;
  p.zcode = zcode;
  p.vals = static_cast<const uint16_t*>(vals);
  p.max_nnzb = max_nnzb;
  p.c_swz_bits = wc_b == 128 ? 3 : wc_b == 64 ? 2 : 1;
  p.c_warp_bytes = pr_align(32 * wc_b);  // one atom x 32 rows, double-buffered per warp
  const uint32_t c_total = 8 * 2 * p.c_warp_bytes;
  int st = (int)((232448 - 2048 - c_total) / p.stage_bytes);
  if (st > kPMaxStages) st = kPMaxStages;
  if (st > 4) st = 4;  // ~128 KB of loads in flight per SM pair half
  if (st < 2) return KAMI_ERROR_NOT_SUPPORTED;
  p.stages = st;
  p.acc_cols = 256;
  p.c_off = st * p.stage_bytes;
  p.bar_off = p.c_off + c_total;
  const uint32_t smem = p.bar_off + 1024 + 1024;
  const CUtensorMapDataType dt = bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16;
  if (!sparse) {
    cuuint64_t dims[3] = {(cuuint64_t)k, (cuuint64_t)m, (cuuint64_t)batch};
    cuuint64_t strides[2] = {(cuuint64_t)k * 2, (cuuint64_t)m * k * 2};
    cuuint32_t box[3] = {(cuuint32_t)p.Wk, 128, 1};
    cuuint32_t es[3] = {1, 1, 1};
    if (enc(&p.tmA, dt, 3, const_cast<void*>(A), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, pr_swz(wk_b),
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  {
    cuuint64_t dims[4] = {(cuuint64_t)p.Wn, (cuuint64_t)k, (cuuint64_t)(n / p.Wn), (cuuint64_t)batch};
    cuuint64_t strides[3] = {(cuuint64_t)n * 2, (cuuint64_t)wn_b, (cuuint64_t)k * n * 2};
    cuuint32_t box[4] = {(cuuint32_t)p.Wn, (cuuint32_t)p.Wk, (cuuint32_t)((n / 2) / p.Wn), 1};
    cuuint32_t es[4] = {1, 1, 1, 1};
    if (enc(&p.tmB, dt, 4, const_cast<void*>(B), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, pr_swz(wn_b),
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  {
    cuuint64_t dims[4] = {(cuuint64_t)p.Wc, (cuuint64_t)m, (cuuint64_t)(n / p.Wc), (cuuint64_t)batch};
    cuuint64_t strides[3] = {(cuuint64_t)n * 2, (cuuint64_t)wc_b, (cuuint64_t)m * n * 2};
    cuuint32_t box[4] = {(cuuint32_t)p.Wc, 32, 1, 1};
    cuuint32_t es[4] = {1, 1, 1, 1};
    if (enc(&p.tmC, dt, 4, C, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, pr_swz(wc_b),
            CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return KAMI_ERROR_CUDA;
  }
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  long long pairs = sms / 2;
  if (pairs > batch) pairs = batch;
  const long long cap = apply_grid_cap(2 * pairs);
  pairs = cap / 2 > 0 ? cap / 2 : 1;
  auto fn = sparse ? (bf16 ? kami_tc16_pair_kernel<1, true> : kami_tc16_pair_kernel<0, true>)
                   : (bf16 ? kami_tc16_pair_kernel<1, false> : kami_tc16_pair_kernel<0, false>);
  cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  fn<<<(unsigned)(2 * pairs), kPThreads + (sparse ? 128 : 0), smem, stream>>>(p);
  set_last_kernel(sparse ? (bf16 ? "kami_tc16_pair_2d<bf16,spmm_zmorton>" : "kami_tc16_pair_2d<f16,spmm_zmorton>")
                         : (bf16 ? "kami_tc16_pair_2d<bf16>" : "kami_tc16_pair_2d<f16>"));
  return cudaGetLastError() == cudaSuccess ? KAMI_SUCCESS : KAMI_ERROR_CUDA;
}

}  // namespace kami
