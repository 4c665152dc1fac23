// sched.cuh -- division-free work counters shared by the persistent tcgen05
// kernels (tc16.cu, tc16_vb.cu).
//
// The single-thread producer / MMA roles run one loop iteration per unit; with
// small units their serial instruction latency bounds the kernel (ncu: ~190
// instructions per unit in the MMA lane with 64-bit divisions before these),
// so no division or modulo is left inside the loops.
#pragma once

#include <cstdint>

namespace kami {

// unit u -> (entry group grp, m-tile mt) with u = grp * m_tiles + mt, advanced
// by a fixed stride (the grid size, or twice it for one epilogue warpgroup)
struct UnitIter {
  long long grp;
  int mt, gstep, mstep, m_tiles;
  __device__ __forceinline__ UnitIter(long long u0, long long step, int mtiles) {
    m_tiles = mtiles;
    grp = u0 / mtiles;
    mt = (int)(u0 - grp * mtiles);
    gstep = (int)(step / mtiles);
    mstep = (int)(step - (long long)gstep * mtiles);
  }
  __device__ __forceinline__ void next() {
    grp += gstep;
    mt += mstep;
    if (mt >= m_tiles) {
      mt -= m_tiles;
      ++grp;
    }
  }
};

// (slot, phase) of a ring of n mbarrier-guarded slots
struct RingPos {
  uint32_t s = 0, ph = 0;
  __device__ __forceinline__ void next(uint32_t n) {
    if (++s == n) {
      s = 0;
      ph ^= 1;
    }
  }
};

// Pointer arrays on TMA (tc16.cu, dmma_tma.cu, tc16_vb.cu).  A tensor map
// cannot follow a pointer array, but all entries live in one virtual address
// space: a view map describes that space as a tensor whose two outer
// dimensions are (16-byte offset mod 2^28, 2^28-byte offset) from kViewBase,
// so the box of the entry at byte address q has outer coordinates
// ((q - kViewBase) / 16 mod 2^24, (q - kViewBase) / 2^28).  Entries are 16-byte
// aligned (kami.h) and the view covers 2^48 bytes; the inner dimensions are the
// entry's own, and a box must never leave them (measured on sm_100a: a box
// partly out of bounds of a view faults where a strided map zero-fills).
constexpr unsigned long long kViewBase = 256;
__device__ __forceinline__ void view_coords(const void* q, int& lo, int& hi) {
  const unsigned long long off = reinterpret_cast<unsigned long long>(q) - kViewBase;
  lo = (int)((off >> 4) & 0xFFFFFFull);
  hi = (int)(off >> 28);
}

}  // namespace kami
