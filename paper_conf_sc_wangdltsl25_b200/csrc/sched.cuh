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

}  // namespace kami
