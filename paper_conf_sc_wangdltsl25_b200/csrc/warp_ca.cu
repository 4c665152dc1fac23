// warp_ca.cu -- register-resident, warp-level communication-avoiding batched
// GEMM: the literal KAMI schedules (Alg. 1-3, Sec. 4.3-4.5) on the
// legacy warp-synchronous tensor-core path of sm_100a:
//   FP64      mma.sync.m8n8k4.f64   (DMMA -- the only FP64 tensor path; there
//             is no tcgen05 kind for f64)
//   FP16/BF16 mma.sync.m16n8k16 with FP32 accumulation (HMMA; the tcgen05
//             family in tc16.cu is the 16-bit production path, this one is the
//             CA-evidence and comparison family)
//
// Roles (Table 1): compute unit = warp; local storage = the warp's
// registers holding A_i, B_i, C_i as MMA fragments (Sec. 4.2); communication
// = shared memory.  A team of P warps owns one batch entry at a time; a CTA
// runs several teams; teams loop persistently over the batch.
//
// Shared-memory exchange is stored in *fragment order*:
//   word[(fragment * REGS + reg) * 32 + lane]
// so every LD/ST of a broadcast tile is a contiguous, bank-conflict-free
// warp access (theta_r = theta_w = 1 in the paper's Eq. 2/6/10) and the
// receivers obtain exactly the sender's fragments.
//
// One named barrier per stage (per team): the exchange buffers are double
// buffered on a running stage counter, so the paper's second
// __syncthreads() per stage (Alg. 1 line 11) is unnecessary.
//
// SMEM traffic per entry (kernel totals):
//   1D  p kn s_e              2D  sqrt(p) (mk + kn) s_e
//   3D  cbrt(p) (mk+kn) s_e + 2 (cbrt(p)-1) mn s_acc (layer reduction)
//   non-CA (W_m x W_n warps)  (mk + kn) s_e + (W_n mk + W_m kn) s_e
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>

#include "kernels.h"
#include "ptx.cuh"

namespace kami {
namespace {

// ------------------------------------------------------------ MMA atoms
struct F64Atom {
  using E = double;
  using R = double;
  using Acc = double;
  static constexpr int AM = 8, AN = 8, AK = 4;
  static constexpr int NA = 1, NB = 1, NC = 2;
  static constexpr bool kBF16 = false;
  __device__ static void a_pos(int lane, int, int& row, int& col) {
    row = lane >> 2;
    col = lane & 3;
  }
  __device__ static void b_pos(int lane, int, int& k, int& n) {
    k = lane & 3;
    n = lane >> 2;
  }
  __device__ static R load_a(const E* p, int ld, int row, int col) { return __ldg(p + row * ld + col); }
  __device__ static R load_b(const E* p, int ld, int k, int n) { return __ldg(p + k * ld + n); }
  __device__ static void mma(Acc (&c)[NC], const R (&a)[NA], const R (&b)[NB]) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                 : "+d"(c[0]), "+d"(c[1])
                 : "d"(a[0]), "d"(b[0]));
  }
  // C fragment: lane (g,t) holds (g, 2t) and (g, 2t+1)
  __device__ static void store_c(E* C, int ld, int row0, int col0, int lane, const Acc (&c)[NC]) {
    const int row = row0 + (lane >> 2), col = col0 + 2 * (lane & 3);
    ptx::st_global_v2_f64(C + row * ld + col, c[0], c[1]);
  }
};

// mma.sync.m16n8k8.f64 (sm_90+ DMMA shape): A 16x8 (4 regs), B 8x8 (2), C 16x8 (4)
struct F64Atom16 {
  using E = double;
  using R = double;
  using Acc = double;
  static constexpr int AM = 16, AN = 8, AK = 8;
  static constexpr int NA = 4, NB = 2, NC = 4;
  static constexpr bool kBF16 = false;
  __device__ static void a_pos(int lane, int r, int& row, int& col) {
    row = (lane >> 2) + 8 * (r & 1);
    col = (lane & 3) + 4 * (r >> 1);
  }
  __device__ static void b_pos(int lane, int r, int& k, int& n) {
    k = (lane & 3) + 4 * r;
    n = lane >> 2;
  }
  __device__ static R load_a(const E* p, int ld, int row, int col) { return __ldg(p + row * ld + col); }
  __device__ static R load_b(const E* p, int ld, int k, int n) { return __ldg(p + k * ld + n); }
  __device__ static void mma(Acc (&c)[NC], const R (&a)[NA], const R (&b)[NB]) {
    asm volatile(
        "mma.sync.aligned.m16n8k8.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+d"(c[0]), "+d"(c[1]), "+d"(c[2]), "+d"(c[3])
        : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(b[0]), "d"(b[1]));
  }
  __device__ static void store_c(E* C, int ld, int row0, int col0, int lane, const Acc (&c)[NC]) {
    const int row = row0 + (lane >> 2), col = col0 + 2 * (lane & 3);
    ptx::st_global_v2_f64(C + row * ld + col, c[0], c[1]);
    ptx::st_global_v2_f64(C + (row + 8) * ld + col, c[2], c[3]);
  }
};

template <bool BF>
struct F16Atom {
  using E = uint16_t;
  using R = uint32_t;
  using Acc = float;
  static constexpr int AM = 16, AN = 8, AK = 16;
  static constexpr int NA = 4, NB = 2, NC = 4;
  static constexpr bool kBF16 = BF;
  __device__ static void a_pos(int lane, int r, int& row, int& col) {
    row = (lane >> 2) + 8 * (r & 1);
    col = 2 * (lane & 3) + 8 * (r >> 1);
  }
  __device__ static void b_pos(int lane, int r, int& k, int& n) {
    k = 2 * (lane & 3) + 8 * r;
    n = lane >> 2;
  }
  __device__ static R load_a(const E* p, int ld, int row, int col) {
    return __ldg(reinterpret_cast<const unsigned int*>(p + row * ld + col));
  }
  __device__ static R load_b(const E* p, int ld, int k, int n) {
    const uint32_t lo = __ldg(reinterpret_cast<const unsigned short*>(p + k * ld + n));
    const uint32_t hi = __ldg(reinterpret_cast<const unsigned short*>(p + (k + 1) * ld + n));
    return lo | (hi << 16);
  }
  __device__ static void mma(Acc (&c)[NC], const R (&a)[NA], const R (&b)[NB]) {
    if (BF) {
      asm volatile(
          "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
          "{%0,%1,%2,%3};"
          : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
          : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
    } else {
      asm volatile(
          "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
          "{%0,%1,%2,%3};"
          : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
          : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
    }
  }
  // C fragment: c0,c1 -> (g, 2t..2t+1); c2,c3 -> (g+8, 2t..2t+1); RNE to 16 bit
  __device__ static void store_c(E* C, int ld, int row0, int col0, int lane, const Acc (&c)[NC]) {
    const int row = row0 + (lane >> 2), col = col0 + 2 * (lane & 3);
    const uint32_t lo = BF ? ptx::pack_bf16x2(c[0], c[1]) : ptx::pack_f16x2(c[0], c[1]);
    const uint32_t hi = BF ? ptx::pack_bf16x2(c[2], c[3]) : ptx::pack_f16x2(c[2], c[3]);
    ptx::st_global_b32(C + row * ld + col, lo);
    ptx::st_global_b32(C + (row + 8) * ld + col, hi);
  }
};

// ------------------------------------------------------- fragment tiles
template <class At, int TM, int TK>
struct TileA {
  static constexpr int FM = TM / At::AM, FK = TK / At::AK, WORDS = FM * FK * At::NA * 32;
  typename At::R v[FM][FK][At::NA];
};
template <class At, int TK, int TN>
struct TileB {
  static constexpr int FK = TK / At::AK, FN = TN / At::AN, WORDS = FK * FN * At::NB * 32;
  typename At::R v[FK][FN][At::NB];
};
template <class At, int TM, int TN>
struct TileC {
  static constexpr int FM = TM / At::AM, FN = TN / At::AN, WORDS = FM * FN * At::NC * 32;
  typename At::Acc v[FM][FN][At::NC];
};

// GMem2Reg: load a warp tile straight into fragment registers
template <class At, int TM, int TK>
__device__ __forceinline__ void load_a(TileA<At, TM, TK>& t, const typename At::E* A, int ld, int row0, int col0,
                                       int lane) {
#pragma unroll
  for (int i = 0; i < t.FM; ++i)
#pragma unroll
    for (int j = 0; j < t.FK; ++j)
#pragma unroll
      for (int r = 0; r < At::NA; ++r) {
        int row, col;
        At::a_pos(lane, r, row, col);
        t.v[i][j][r] = At::load_a(A, ld, row0 + i * At::AM + row, col0 + j * At::AK + col);
      }
}
template <class At, int TK, int TN>
__device__ __forceinline__ void load_b(TileB<At, TK, TN>& t, const typename At::E* B, int ld, int row0, int col0,
                                       int lane) {
#pragma unroll
  for (int i = 0; i < t.FK; ++i)
#pragma unroll
    for (int j = 0; j < t.FN; ++j)
#pragma unroll
      for (int r = 0; r < At::NB; ++r) {
        int k, n;
        At::b_pos(lane, r, k, n);
        t.v[i][j][r] = At::load_b(B, ld, row0 + i * At::AK + k, col0 + j * At::AN + n);
      }
}

// Reg2SMem / SMem2Reg in fragment order (contiguous per warp access)
template <class Tile, class W>
__device__ __forceinline__ void put(const Tile& t, W* s, int lane) {
  const W* f = &t.v[0][0][0];
  constexpr int n = sizeof(t.v) / sizeof(W);
#pragma unroll
  for (int i = 0; i < n; ++i) s[i * 32 + lane] = f[i];
}
template <class Tile, class W>
__device__ __forceinline__ void get(Tile& t, const W* s, int lane) {
  W* f = &t.v[0][0][0];
  constexpr int n = sizeof(t.v) / sizeof(W);
#pragma unroll
  for (int i = 0; i < n; ++i) f[i] = s[i * 32 + lane];
}

template <class At, int TM, int TN>
__device__ __forceinline__ void zero(TileC<At, TM, TN>& c) {
  typename At::Acc* f = &c.v[0][0][0];
#pragma unroll
  for (int i = 0; i < (int)(sizeof(c.v) / sizeof(typename At::Acc)); ++i) f[i] = 0;
}

// TensorCoreGEMM: C += A[:, KOFF fragments .. + B.FK] * B
template <class At, int TM, int TKA, int TKB, int TN>
__device__ __forceinline__ void mma_tile(TileC<At, TM, TN>& c, const TileA<At, TM, TKA>& a,
                                         const TileB<At, TKB, TN>& b, int koff) {
#pragma unroll
  for (int kk = 0; kk < TileB<At, TKB, TN>::FK; ++kk)
#pragma unroll
    for (int i = 0; i < TileC<At, TM, TN>::FM; ++i)
#pragma unroll
      for (int j = 0; j < TileC<At, TM, TN>::FN; ++j) At::mma(c.v[i][j], a.v[i][koff + kk], b.v[kk][j]);
}

template <class At, int TM, int TN>
__device__ __forceinline__ void store_c(const TileC<At, TM, TN>& c, typename At::E* C, int ld, int row0, int col0,
                                        int lane) {
#pragma unroll
  for (int i = 0; i < TileC<At, TM, TN>::FM; ++i)
#pragma unroll
    for (int j = 0; j < TileC<At, TM, TN>::FN; ++j)
      At::store_c(C, ld, row0 + i * At::AM, col0 + j * At::AN, lane, c.v[i][j]);
}

template <class T>
__device__ __forceinline__ void copy_tile(T& dst, const T& src) {
  dst = src;
}

// Per-phase cycle counters for the block-level mode (Sec. 5.6.2,
// Fig. 15: clock() around communication and computation phases).  Like the
// paper's, the compute phase counts issue time of the mma.sync sequence.
template <bool kTime>
struct PhaseClock {
  long long t0 = 0, comm = 0, comp = 0;
  __device__ __forceinline__ void begin() {
    if (kTime) t0 = clock64();
  }
  __device__ __forceinline__ void comm_done() {
    if (kTime) {
      const long long t = clock64();
      comm += t - t0;
      t0 = t;
    }
  }
  __device__ __forceinline__ void comp_done() {
    if (kTime) {
      const long long t = clock64();
      comp += t - t0;
      t0 = t;
    }
  }
  __device__ __forceinline__ void flush(long long* cyc, int lane) {
    if (kTime && cyc && lane == 0) {
      atomicAdd(reinterpret_cast<unsigned long long*>(cyc), (unsigned long long)comm);
      atomicAdd(reinterpret_cast<unsigned long long*>(cyc + 1), (unsigned long long)comp);
    }
  }
};

// ------------------------------------------------------------ schedules
// Each schedule runs one batch entry on a team of P warps.  wi = warp index
// in the team, bar = named barrier id of the team, stage = running stage
// counter of the team (selects the exchange buffer).

// KAMI-1D, Alg. 1: warp i holds A_i (m/p x k), B_i
// (k/p x n), C_i (m/p x n).  Stage z: warp z writes B_z to SMEM and keeps a
// register copy (Reg2Reg); the others read it; all do C_i += A_i[:, z] B_z.
template <class At, int M, int N, int K, int P>
struct Sched1D {
  static constexpr int MP = M / P, KP = K / P;
  using TA = TileA<At, MP, K>;
  using TB = TileB<At, KP, N>;
  using TC = TileC<At, MP, N>;
  static constexpr int XWORDS = TB::WORDS;          // one exchange tile
  static constexpr int SMEM_WORDS = 2 * XWORDS;     // double buffered
  static constexpr int SMEM_BYTES = SMEM_WORDS * sizeof(typename At::R);
  static_assert(MP % At::AM == 0 && KP % At::AK == 0 && N % At::AN == 0, "1D tile shape");
  template <bool kTime>
  __device__ static void run(const typename At::E* A, const typename At::E* B, typename At::E* C, uint8_t* smem,
                             int wi, int lane, int bar, uint32_t& stage, int reps, long long* cyc) {
    using W = typename At::R;
    W* xb = reinterpret_cast<W*>(smem);
    TA a;
    TB bi, br;
    TC c;
    load_a(a, A, K, wi * MP, 0, lane);  // GMem2Reg(A_i)
    load_b(bi, B, N, wi * KP, 0, lane);  // GMem2Reg(B_i)
    zero(c);
    PhaseClock<kTime> clk;
#pragma unroll 1
    for (int rep = 0; rep < reps; ++rep) {  // block-level mode repeats on-chip
#pragma unroll
      for (int z = 0; z < P; ++z, ++stage) {
        clk.begin();
        W* buf = xb + (stage & 1) * XWORDS;
        if (wi == z) {
          put(bi, buf, lane);  // Reg2SMem(SmB <- BSend)
          copy_tile(br, bi);   // Reg2Reg(BRecv <- BSend)
        }
        ptx::named_bar_sync(bar, P * 32);
        if (wi != z) get(br, buf, lane);  // SMem2Reg(BRecv <- SmB)
        clk.comm_done();
        mma_tile(c, a, br, z * (KP / At::AK));  // C_i += A_i[:, z k/p:(z+1) k/p] BRecv
        clk.comp_done();
      }
    }
    clk.flush(cyc, lane);
    store_c(c, C, N, wi * MP, 0, lane);  // Reg2GMem
  }
};

// KAMI-2D, Alg. 2: sqrt(p) x sqrt(p) warp grid; warp
// (r, c) holds A_rc (m/q x k/q), B_rc (k/q x n/q).  Stage z: column z
// broadcasts its A tile along its row, row z broadcasts its B tile along
// its column.
template <class At, int M, int N, int K, int P>
struct Sched2D {
  static constexpr int Q = (P == 4) ? 2 : (P == 16) ? 4 : (P == 1 ? 1 : 0);
  static_assert(Q > 0, "2D needs p = 4 or 16");
  static constexpr int TM = M / Q, TN = N / Q, TK = K / Q;
  using TA = TileA<At, TM, TK>;
  using TB = TileB<At, TK, TN>;
  using TC = TileC<At, TM, TN>;
  static constexpr int XWORDS = Q * TA::WORDS + Q * TB::WORDS;
  static constexpr int SMEM_WORDS = 2 * XWORDS;
  static constexpr int SMEM_BYTES = SMEM_WORDS * sizeof(typename At::R);
  static_assert(TM % At::AM == 0 && TK % At::AK == 0 && TN % At::AN == 0, "2D tile shape");
  template <bool kTime>
  __device__ static void run(const typename At::E* A, const typename At::E* B, typename At::E* C, uint8_t* smem,
                             int wi, int lane, int bar, uint32_t& stage, int reps, long long* cyc) {
    using W = typename At::R;
    const int wr = wi / Q, wc = wi % Q;
    TA ai, ar;
    TB bi, br;
    TC c;
    load_a(ai, A, K, wr * TM, wc * TK, lane);
    load_b(bi, B, N, wr * TK, wc * TN, lane);
    zero(c);
    PhaseClock<kTime> clk;
#pragma unroll 1
    for (int rep = 0; rep < reps; ++rep) {
#pragma unroll
      for (int z = 0; z < Q; ++z, ++stage) {
        clk.begin();
        W* buf = reinterpret_cast<W*>(smem) + (stage & 1) * XWORDS;
        W* sa = buf + wr * TA::WORDS;                  // SmA of grid row wr
        W* sb = buf + Q * TA::WORDS + wc * TB::WORDS;  // SmB of grid column wc
        if (wc == z) {
          put(ai, sa, lane);
          copy_tile(ar, ai);
        }
        if (wr == z) {
          put(bi, sb, lane);
          copy_tile(br, bi);
        }
        ptx::named_bar_sync(bar, P * 32);
        if (wc != z) get(ar, sa, lane);
        if (wr != z) get(br, sb, lane);
        clk.comm_done();
        mma_tile(c, ar, br, 0);
        clk.comp_done();
      }
    }
    clk.flush(cyc, lane);
    store_c(c, C, N, wr * TM, wc * TN, lane);
  }
};

// KAMI-3D, Alg. 3: cbrt(p)^3 warp cube = cbrt(p) layers of
// 2D grids, layer l owning the k-range [l k/c, (l+1) k/c).  Reading R6:
// A_i is m/c x k/c^2, B_i k/c^2 x n/c.  After c stages each layer holds a
// partial C; layers 1.. write theirs to SMEM and layer 0 adds them in layer
// order (Alg. 3 line 19) before the store.
template <class At, int M, int N, int K, int P>
struct Sched3D {
  static constexpr int Cc = (P == 8) ? 2 : (P == 1 ? 1 : 0);
  static_assert(Cc > 0, "3D needs p = 8");
  static constexpr int TM = M / Cc, TN = N / Cc, TK = K / (Cc * Cc);
  using TA = TileA<At, TM, TK>;
  using TB = TileB<At, TK, TN>;
  using TC = TileC<At, TM, TN>;
  static constexpr int LWORDS = Cc * TA::WORDS + Cc * TB::WORDS;  // one layer, one stage
  static constexpr int XWORDS = Cc * LWORDS;
  static constexpr int XBYTES = 2 * XWORDS * sizeof(typename At::R);
  // reduce-scatter slots: per cell, per owner layer, per sender layer, one chunk
  static constexpr int RBYTES = Cc * Cc * Cc * TC::WORDS * sizeof(typename At::Acc);
  static constexpr int SMEM_BYTES = XBYTES + RBYTES;
  static_assert(TM % At::AM == 0 && TK % At::AK == 0 && TN % At::AN == 0, "3D tile shape");
  template <bool kTime>
  __device__ static void run(const typename At::E* A, const typename At::E* B, typename At::E* C, uint8_t* smem,
                             int wi, int lane, int bar, uint32_t& stage, int reps, long long* cyc) {
    using W = typename At::R;
    using Acc = typename At::Acc;
    const int l = wi / (Cc * Cc), wr = (wi / Cc) % Cc, wc = wi % Cc;
    const int kl = l * (K / Cc);
    TA ai, ar;
    TB bi, br;
    TC c;
    load_a(ai, A, K, wr * TM, kl + wc * TK, lane);
    load_b(bi, B, N, kl + wr * TK, wc * TN, lane);
    zero(c);
    PhaseClock<kTime> clk;
#pragma unroll 1
    for (int rep = 0; rep < reps; ++rep) {
#pragma unroll
      for (int z = 0; z < Cc; ++z, ++stage) {
        clk.begin();
        W* buf = reinterpret_cast<W*>(smem) + (stage & 1) * XWORDS + l * LWORDS;
        W* sa = buf + wr * TA::WORDS;
        W* sb = buf + Cc * TA::WORDS + wc * TB::WORDS;
        if (wc == z) {
          put(ai, sa, lane);
          copy_tile(ar, ai);
        }
        if (wr == z) {
          put(bi, sb, lane);
          copy_tile(br, bi);
        }
        ptx::named_bar_sync(bar, P * 32);
        if (wc != z) get(ar, sa, lane);
        if (wr != z) get(br, sb, lane);
        clk.comm_done();
        mma_tile(c, ar, br, 0);
        clk.comp_done();
      }
    }
    clk.flush(cyc, lane);
    // K-split reduction across layers as a reduce-scatter: the C tile's
    // fragments are split into Cc chunks, layer l owns chunk l.  Each layer
    // writes the chunks it does not own, reads the others' partials of its own
    // chunk, sums them in fixed layer order 0 + 1 + ... (Alg. 3 line 19) and
    // stores its chunk -- (Cc-1)/Cc of the tile crosses SMEM instead of all of it.
    constexpr int NF = TC::FM * TC::FN, FW = At::NC * 32;  // fragments, words per fragment
    Acc* red = reinterpret_cast<Acc*>(smem + XBYTES);
    const int cell = wr * Cc + wc;
    if constexpr (NF % Cc == 0) {
      constexpr int CS = NF / Cc;
      auto slot = [&](int owner, int sender) { return red + ((cell * Cc + owner) * Cc + sender) * CS * FW; };
#pragma unroll
      for (int f = 0; f < NF; ++f) {
        const int o = f / CS;
        if (o != l) {
          Acc* dst = slot(o, l) + (f - o * CS) * FW;
#pragma unroll
          for (int r = 0; r < At::NC; ++r) dst[r * 32 + lane] = c.v[f / TC::FN][f % TC::FN][r];
        }
      }
      ptx::named_bar_sync(bar, P * 32);
#pragma unroll
      for (int f = 0; f < NF; ++f) {
        if (f / CS == l) {
          Acc v[At::NC];
#pragma unroll
          for (int r = 0; r < At::NC; ++r) {
            Acc sum = 0;
#pragma unroll
            for (int ll = 0; ll < Cc; ++ll) {
              const Acc x =
                  (ll == l) ? c.v[f / TC::FN][f % TC::FN][r] : slot(l, ll)[(f - l * CS) * FW + r * 32 + lane];
              sum = (ll == 0) ? x : sum + x;
            }
            v[r] = sum;
          }
          At::store_c(C, N, wr * TM + (f / TC::FN) * At::AM, wc * TN + (f % TC::FN) * At::AN, lane, v);
        }
      }
    } else {
      // a single-fragment tile cannot be split: gather to layer 0
      if (l > 0) put(c, red + ((l - 1) * Cc * Cc + cell) * TC::WORDS, lane);
      ptx::named_bar_sync(bar, P * 32);
      if (l == 0) {
#pragma unroll 1
        for (int ll = 1; ll < Cc; ++ll) {
          TC t;
          get(t, red + ((ll - 1) * Cc * Cc + cell) * TC::WORDS, lane);
          Acc* f = &c.v[0][0][0];
          const Acc* g = &t.v[0][0][0];
#pragma unroll
          for (int i = 0; i < (int)(sizeof(c.v) / sizeof(Acc)); ++i) f[i] += g[i];
        }
        store_c(c, C, N, wr * TM, wc * TN, lane);
      }
    }
  }
};

// Non-CA tiled baseline (the "traditional kernel" of PAPER.md L519): the team
// stages all of A and B in SMEM (fragment order, conflict-free), then a
// W_m x W_n warp grid reads its fragments from SMEM for every MMA.
template <class At, int M, int N, int K, int P>
struct SchedNonCA {
  static constexpr int WM = (P == 4) ? 2 : (P == 8 || P == 16) ? 4 : 1, WN = P / WM;
  static constexpr int TM = M / WM, TN = N / WN;
  static constexpr int FMT = M / At::AM, FKT = K / At::AK, FNT = N / At::AN;  // whole-matrix fragment grid
  static constexpr int AWORDS = FMT * FKT * At::NA * 32, BWORDS = FKT * FNT * At::NB * 32;
  static constexpr int SMEM_BYTES = (AWORDS + BWORDS) * sizeof(typename At::R);
  static_assert(TM % At::AM == 0 && TN % At::AN == 0, "non-CA tile shape");
  template <bool kTime>
  __device__ static void run(const typename At::E* A, const typename At::E* B, typename At::E* C, uint8_t* smem,
                             int wi, int lane, int bar, uint32_t& stage, int reps, long long* cyc) {
    using W = typename At::R;
    W* sA = reinterpret_cast<W*>(smem);
    W* sB = sA + AWORDS;
    // every MMA operand passes through SMEM: stage A and B (fragment order)
#pragma unroll 1
    for (int f = wi; f < FMT * FKT; f += P) {
      const int fm = f / FKT, fk = f % FKT;
#pragma unroll
      for (int r = 0; r < At::NA; ++r) {
        int row, col;
        At::a_pos(lane, r, row, col);
        sA[(f * At::NA + r) * 32 + lane] = At::load_a(A, K, fm * At::AM + row, fk * At::AK + col);
      }
    }
#pragma unroll 1
    for (int f = wi; f < FKT * FNT; f += P) {
      const int fk = f / FNT, fn = f % FNT;
#pragma unroll
      for (int r = 0; r < At::NB; ++r) {
        int k, n;
        At::b_pos(lane, r, k, n);
        sB[(f * At::NB + r) * 32 + lane] = At::load_b(B, N, fk * At::AK + k, fn * At::AN + n);
      }
    }
    ptx::named_bar_sync(bar, P * 32);
    const int wm = wi / WN, wn = wi % WN;
    TileC<At, TM, TN> c;
    zero(c);
    PhaseClock<kTime> clk;
#pragma unroll 1
    for (int rep = 0; rep < reps; ++rep) {
#pragma unroll 1
      for (int fk = 0; fk < FKT; ++fk) {
        clk.begin();
        TileA<At, TM, At::AK> a;
        TileB<At, At::AK, TN> b;
#pragma unroll
        for (int i = 0; i < TileA<At, TM, At::AK>::FM; ++i)
#pragma unroll
          for (int r = 0; r < At::NA; ++r)
            a.v[i][0][r] = sA[(((wm * (TM / At::AM) + i) * FKT + fk) * At::NA + r) * 32 + lane];
#pragma unroll
        for (int j = 0; j < TileB<At, At::AK, TN>::FN; ++j)
#pragma unroll
          for (int r = 0; r < At::NB; ++r)
            b.v[0][j][r] = sB[((fk * FNT + wn * (TN / At::AN) + j) * At::NB + r) * 32 + lane];
        clk.comm_done();
        mma_tile(c, a, b, 0);
        clk.comp_done();
      }
    }
    clk.flush(cyc, lane);
    store_c(c, C, N, wm * TM, wn * TN, lane);
    ptx::named_bar_sync(bar, P * 32);  // SMEM is reused by the next entry
    ++stage;
  }
};

// ----------------------------------------------------------- the kernel
template <class Sched, class At, int P, int TEAMS, bool kTime>
__global__ void __launch_bounds__(P * 32 * TEAMS) kami_warp_ca_kernel(const typename At::E* __restrict__ A,
                                                                      const typename At::E* __restrict__ B,
                                                                      typename At::E* __restrict__ C,
                                                                      const void* const* A_arr,
                                                                      const void* const* B_arr, void* const* C_arr,
                                                                      long long batch, int M, int N, int K,
                                                                      int prefetch, int reps, long long* cyc) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int team = warp / P, wi = warp % P;
  uint8_t* smem = smem_raw + team * ((Sched::SMEM_BYTES + 127) / 128 * 128);
  const int bar = 1 + team;
  uint32_t stage = 0;
  const long long nteams = (long long)gridDim.x * TEAMS;
  for (long long e = (long long)blockIdx.x * TEAMS + team; e < batch; e += nteams) {
    const typename At::E* a;
    const typename At::E* b;
    typename At::E* c;
    if (A_arr) {
      a = reinterpret_cast<const typename At::E*>(A_arr[e]);
      b = reinterpret_cast<const typename At::E*>(B_arr[e]);
      c = reinterpret_cast<typename At::E*>(C_arr[e]);
    } else {
      a = A + e * (long long)M * K;
      b = B + e * (long long)K * N;
      c = C + e * (long long)M * N;
    }
    // Stream the team's NEXT entry from HBM into L2 while this one computes,
    // so its GMem2Reg loads hit L2 (the register-resident design cannot
    // double-buffer operands in registers).
    if (prefetch && wi == 0 && lane == 0 && e + nteams < batch) {
      const long long en = e + nteams;
      const void* na = A_arr ? A_arr[en] : (const void*)(A + en * (long long)M * K);
      const void* nb = A_arr ? B_arr[en] : (const void*)(B + en * (long long)K * N);
      ptx::prefetch_l2_bulk(na, (uint32_t)(M * K * sizeof(typename At::E)));
      ptx::prefetch_l2_bulk(nb, (uint32_t)(K * N * sizeof(typename At::E)));
    }
    Sched::template run<kTime>(a, b, c, smem, wi, lane, bar, stage, reps, cyc ? cyc + 2 * e : nullptr);
  }
}

// ----------------------------------------------------------- host side
struct LaunchInfo {
  const void* fn;
  const void* fn_timed;
  int p;
  int threads;
  int smem;
  const char* name;
};

template <class Sched, class At, int P, int TEAMS>
LaunchInfo info(const char* name) {
  LaunchInfo li;
  li.fn = reinterpret_cast<const void*>(&kami_warp_ca_kernel<Sched, At, P, TEAMS, false>);
  li.fn_timed = reinterpret_cast<const void*>(&kami_warp_ca_kernel<Sched, At, P, TEAMS, true>);
  li.p = P;
  li.threads = P * 32 * TEAMS;
  li.smem = TEAMS * ((Sched::SMEM_BYTES + 127) / 128 * 128);
  li.name = name;
  return li;
}

#define KAMI_TEAMS(P) ((P) >= 8 ? 1 : 8 / (P))
#define KAMI_CASE(ATOM, DT, MM, NN, KK, ALG, SCHED, P, NAME)                                     \
  if (dtype == DT && m == MM && n == NN && k == KK && algo == ALG && (p == 0 || p == P)) {      \
    *out = info<SCHED<ATOM, MM, NN, KK, P>, ATOM, P, KAMI_TEAMS(P)>(NAME);                      \
    return true;                                                                                 \
  }

#define KAMI_SIZE_CASES(ATOM, DT, S, P1, P2, P3, PN, TAG)                                         \
  KAMI_CASE(ATOM, DT, S, S, S, 1, Sched1D, P1, "kami_warp_ca_1d<" TAG "," #S ">")                 \
  KAMI_CASE(ATOM, DT, S, S, S, 2, Sched2D, P2, "kami_warp_ca_2d<" TAG "," #S ">")                 \
  KAMI_CASE(ATOM, DT, S, S, S, 3, Sched3D, P3, "kami_warp_ca_3d<" TAG "," #S ">")                 \
  KAMI_CASE(ATOM, DT, S, S, S, 4, SchedNonCA, PN, "kami_warp_nonca<" TAG "," #S ">")

using H16 = F16Atom<false>;
using B16 = F16Atom<true>;

int f64_atom_pref() {  // 16 = m16n8k8 DMMA first, 8 = m8n8k4 first (env KAMI_F64_ATOM)
  static const int v = [] {
    const char* e = getenv("KAMI_F64_ATOM");
    return e ? atoi(e) : 16;
  }();
  return v;
}

bool lookup(int m, int n, int k, kami_dtype_t dtype, int algo, int p, LaunchInfo* out) {
  if (f64_atom_pref() == 16) {
    // FP64 DMMA m16n8k8 where the register budget allows it
    KAMI_CASE(F64Atom16, KAMI_DTYPE_F64, 16, 16, 16, 1, Sched1D, 1, "kami_warp_ca_1d<f64m16,16>")
    KAMI_CASE(F64Atom16, KAMI_DTYPE_F64, 32, 32, 32, 1, Sched1D, 2, "kami_warp_ca_1d<f64m16,32>")
    KAMI_CASE(F64Atom16, KAMI_DTYPE_F64, 32, 32, 32, 2, Sched2D, 4, "kami_warp_ca_2d<f64m16,32>")
    KAMI_CASE(F64Atom16, KAMI_DTYPE_F64, 32, 32, 32, 3, Sched3D, 8, "kami_warp_ca_3d<f64m16,32>")
    KAMI_CASE(F64Atom16, KAMI_DTYPE_F64, 32, 32, 32, 4, SchedNonCA, 4, "kami_warp_nonca<f64m16,32>")
    KAMI_CASE(F64Atom16, KAMI_DTYPE_F64, 64, 64, 64, 2, Sched2D, 16, "kami_warp_ca_2d<f64m16,64>")
    KAMI_CASE(F64Atom16, KAMI_DTYPE_F64, 64, 64, 64, 3, Sched3D, 8, "kami_warp_ca_3d<f64m16,64>")
    KAMI_CASE(F64Atom16, KAMI_DTYPE_F64, 64, 64, 64, 4, SchedNonCA, 4, "kami_warp_nonca<f64m16,64>")
    KAMI_CASE(F64Atom16, KAMI_DTYPE_F64, 64, 64, 64, 4, SchedNonCA, 16, "kami_warp_nonca16<f64m16,64>")
    KAMI_CASE(F64Atom16, KAMI_DTYPE_F64, 64, 64, 64, 4, SchedNonCA, 8, "kami_warp_nonca8<f64m16,64>")
  }
  // FP64 DMMA (m8n8k4): the literal KAMI register-resident family
  KAMI_SIZE_CASES(F64Atom, KAMI_DTYPE_F64, 16, 2, 4, 8, 4, "f64")
  KAMI_SIZE_CASES(F64Atom, KAMI_DTYPE_F64, 32, 4, 16, 8, 4, "f64")
  KAMI_SIZE_CASES(F64Atom, KAMI_DTYPE_F64, 64, 8, 16, 8, 4, "f64")
  KAMI_CASE(F64Atom, KAMI_DTYPE_F64, 8, 8, 8, 1, Sched1D, 1, "kami_warp_ca_1d<f64,8>")
  KAMI_CASE(F64Atom, KAMI_DTYPE_F64, 32, 32, 32, 4, SchedNonCA, 8, "kami_warp_nonca8<f64,32>")
  KAMI_CASE(H16, KAMI_DTYPE_F16, 64, 64, 64, 4, SchedNonCA, 8, "kami_warp_nonca8<f16,64>")
  KAMI_CASE(B16, KAMI_DTYPE_BF16, 64, 64, 64, 4, SchedNonCA, 8, "kami_warp_nonca8<bf16,64>")
  KAMI_CASE(H16, KAMI_DTYPE_F16, 128, 128, 128, 4, SchedNonCA, 16, "kami_warp_nonca16<f16,128>")
  // FP16 / BF16 HMMA (m16n8k16): CA evidence family
  KAMI_CASE(H16, KAMI_DTYPE_F16, 16, 16, 16, 1, Sched1D, 1, "kami_warp_ca_1d<f16,16>")
  KAMI_CASE(B16, KAMI_DTYPE_BF16, 16, 16, 16, 1, Sched1D, 1, "kami_warp_ca_1d<bf16,16>")
  // thin tiles (k <= 32 with n = 16 or 32, and bf16/f16 16 x 128 x 16) where
  // the tcgen05 unit is mostly empty: one warp per entry, register resident.
  // Kept only where they measured faster than the tcgen05 kernel
  // (profiles/r2/variant_sweep_r2.json); the wide ones (m = 16 with n >= 64 and
  // k = 32, n >= 192, 32 x 128) lost to it and were removed.
#define KAMI_THIN_CASES(MM, NN, KK)                                                                 \
  KAMI_CASE(H16, KAMI_DTYPE_F16, MM, NN, KK, 1, Sched1D, 1, "kami_warp_ca_1d<f16," #MM "x" #NN "x" #KK ">") \
  KAMI_CASE(B16, KAMI_DTYPE_BF16, MM, NN, KK, 1, Sched1D, 1, "kami_warp_ca_1d<bf16," #MM "x" #NN "x" #KK ">")
  KAMI_THIN_CASES(16, 128, 16)
  KAMI_THIN_CASES(16, 32, 16)
  KAMI_THIN_CASES(16, 16, 32)
  KAMI_THIN_CASES(32, 16, 16)
  KAMI_THIN_CASES(64, 16, 16)
  KAMI_THIN_CASES(128, 16, 16)
  KAMI_THIN_CASES(192, 16, 16)
  KAMI_THIN_CASES(256, 16, 16)
  KAMI_THIN_CASES(192, 16, 32)
  KAMI_THIN_CASES(128, 32, 16)
  KAMI_CASE(H16, KAMI_DTYPE_F16, 32, 32, 32, 1, Sched1D, 2, "kami_warp_ca_1d<f16,32>")
  KAMI_CASE(H16, KAMI_DTYPE_F16, 32, 32, 32, 2, Sched2D, 4, "kami_warp_ca_2d<f16,32>")
  KAMI_CASE(H16, KAMI_DTYPE_F16, 32, 32, 32, 4, SchedNonCA, 4, "kami_warp_nonca<f16,32>")
  KAMI_SIZE_CASES(H16, KAMI_DTYPE_F16, 64, 4, 4, 8, 4, "f16")
  KAMI_CASE(H16, KAMI_DTYPE_F16, 128, 128, 128, 1, Sched1D, 8, "kami_warp_ca_1d<f16,128>")
  KAMI_CASE(H16, KAMI_DTYPE_F16, 128, 128, 128, 2, Sched2D, 16, "kami_warp_ca_2d<f16,128>")
  KAMI_CASE(B16, KAMI_DTYPE_BF16, 32, 32, 32, 1, Sched1D, 2, "kami_warp_ca_1d<bf16,32>")
  KAMI_CASE(B16, KAMI_DTYPE_BF16, 32, 32, 32, 2, Sched2D, 4, "kami_warp_ca_2d<bf16,32>")
  KAMI_CASE(B16, KAMI_DTYPE_BF16, 32, 32, 32, 4, SchedNonCA, 4, "kami_warp_nonca<bf16,32>")
  KAMI_SIZE_CASES(B16, KAMI_DTYPE_BF16, 64, 4, 4, 8, 4, "bf16")
  return false;
}

}  // namespace

kami_status_t warp_ca_supported(int m, int n, int k, kami_dtype_t dtype, int algo, int p) {
  LaunchInfo li;
  return lookup(m, n, k, dtype, algo, p, &li) ? KAMI_SUCCESS : KAMI_ERROR_NOT_SUPPORTED;
}

int warp_ca_default_p(int m, int n, int k, kami_dtype_t dtype, int algo) {
  for (int p : {1, 2, 4, 8, 16}) {
    LaunchInfo li;
    if (lookup(m, n, k, dtype, algo, p, &li)) return p;
  }
  return 0;
}

// Resident teams per SM for the model (occupancy API when a device is
// present; otherwise a register estimate: 64K registers / (threads x regs)).
int warp_ca_teams_per_sm(int m, int n, int k, kami_dtype_t dtype, int algo, int p) {
  LaunchInfo li;
  if (!lookup(m, n, k, dtype, algo, p, &li)) return 1;
  const int teams_per_cta = li.threads / 32 / li.p;
  // a register estimate (not the occupancy API), so the planner's choice is
  // the same with and without a device (tests/test_planner_model.py)
  // registers per thread: A_i, B_i (twice, send + receive buffers of the
  // exchange, unless p = 1) and C_i, 16-bit operands two per register, FP32 /
  // FP64 accumulators one / two (matches ptxas within ~10 % on the built
  // instantiations, _build/warp_ca.cu.log)
  const bool f64 = dtype == KAMI_DTYPE_F64;
  const double ab = ((double)m * k + (double)k * n * (li.p > 1 ? 2 : 1)) / li.p * (f64 ? 2.0 : 0.5);
  const double regs = (ab + (double)m * n / li.p * (f64 ? 2.0 : 1.0)) / 32 + 24;
  int per_sm = (int)(65536.0 / (li.threads * regs));
  if (per_sm < 1) per_sm = 1;
  if (per_sm * li.threads > 2048) per_sm = 2048 / li.threads;  // 64 warps per SM
  return per_sm * teams_per_cta;
}

kami_status_t warp_ca_launch(int m, int n, int k, long long batch, kami_dtype_t dtype, int algo, int p,
                             const void* A, const void* B, void* C, const void* const* A_arr,
                             const void* const* B_arr, void* const* C_arr, cudaStream_t stream, int reps,
                             long long* cycles) {
  LaunchInfo li;
  if (!lookup(m, n, k, dtype, algo, p, &li)) return KAMI_ERROR_NOT_SUPPORTED;
  const void* fn = cycles ? li.fn_timed : li.fn;
  if (li.smem > 48 * 1024) {
    if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, li.smem) != cudaSuccess)
      return KAMI_ERROR_CUDA;
  }
  int dev = 0, sms = 148, per_sm = 1;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, li.threads, li.smem) != cudaSuccess ||
      per_sm < 1)
    per_sm = 1;
  const long long teams = li.threads / 32 / li.p;
  const long long ctas_needed = (batch + teams - 1) / teams;
  // batched: persistent teams loop over the batch; block-level (reps > 1):
  // one entry per team, every CTA launched at once
  long long grid = reps > 1 ? ctas_needed : (long long)sms * per_sm;
  if (grid > ctas_needed) grid = ctas_needed;
  if (grid < 1) grid = 1;
  if (reps == 1) grid = apply_grid_cap(grid);  // (block-level mode: one CTA per team set)
  static const int prefetch = [] {
    const char* e = getenv("KAMI_L2_PREFETCH");
    return e ? atoi(e) : 1;
  }();
  int pf = reps > 1 ? 0 : prefetch;
  void* args[] = {(void*)&A, (void*)&B, (void*)&C, (void*)&A_arr, (void*)&B_arr, (void*)&C_arr,
                  (void*)&batch, (void*)&m, (void*)&n, (void*)&k, (void*)&pf, (void*)&reps, (void*)&cycles};
  cudaError_t err = cudaLaunchKernel(fn, dim3((unsigned)grid), dim3(li.threads), args, li.smem, stream);
  set_last_kernel(li.name);
  return err == cudaSuccess ? KAMI_SUCCESS : KAMI_ERROR_CUDA;
}

}  // namespace kami
