// planner.cpp -- see planner.h.
#include "planner.h"

#include <cmath>

#include "kernels.h"

namespace kami {

// PAPER.md Sec. 4.3 (Eqs. 1-4), 4.4 (Eqs. 5-8), 4.5 (Eqs. 9-12), with the
// readings of DESIGN.md: R6 (3D tiles k/cbrt(p)^2), R7 (Eq. 7 / 11
// denominators p^(3/2), p^(4/3)), R8 (p/n_tc kept without ceiling).
PaperCost paper_cost(int variant, double m, double n, double k, double p, double s_e, double L_sm, double B_sm,
                     double tr, double tw, double O_tc, double n_tc) {
  PaperCost c{};
  double stages = 1, V = 0;
  if (variant == 1) {
    stages = p;
    V = k * n * s_e;                                   // Eq. (1)
    c.T_cp = 2.0 * m * n * k / (p * p * O_tc);         // Eq. (3)
  } else if (variant == 2) {
    stages = std::sqrt(p);
    V = (m * k + k * n) * s_e;                         // Eq. (5)
    c.T_cp = 2.0 * m * n * k / (std::pow(p, 1.5) * O_tc);  // Eq. (7), R7
  } else {
    stages = std::round(std::cbrt(p));
    V = (m * k + k * n) * s_e;                         // Eq. (9)
    c.T_cp = 2.0 * m * n * k / (std::pow(p, 4.0 / 3.0) * O_tc);  // Eq. (11), R7
  }
  c.V_cm = V;
  // Eqs. (2) / (6) / (10)
  c.T_cm = L_sm + V / (tw * stages * B_sm) + (stages - 1) * V / (tr * stages * B_sm);
  // Eqs. (4) / (8) / (12)
  c.T_all = stages * (c.T_cm + (p / n_tc) * c.T_cp);
  return c;
}

namespace {

// B200 constants.  L_sm: LDS latency 29 cycles; B_sm:
// 128 B/cycle/SM crossbar; n_tc = 4 sub-partition tensor cores per SM.
// O_tc per tensor core: DMMA FP64 ~ 32 flop/cycle (37 TF / 148 SMs / 1.965
// GHz / 4); legacy HMMA ~ 256 flop/cycle (assumed 1/8 of tcgen05).
constexpr double kLsm = 29, kBsm = 128, kNtc = 4;

double b200_cost(int variant, int m, int n, int k, int p, kami_dtype_t dt) {
  const double s_e = dt == KAMI_DTYPE_F64 ? 8 : 2;
  const double O = dt == KAMI_DTYPE_F64 ? 32 : 256;
  PaperCost c = paper_cost(variant, m, n, k, p, s_e, kLsm, kBsm, 1, 1, O, kNtc);
  const double stages = variant == 1 ? p : variant == 2 ? std::sqrt((double)p) : std::round(std::cbrt((double)p));
  const double ratio = std::max(1.0, p / kNtc);
  double t = stages * (c.T_cm + ratio * c.T_cp);
  if (variant == 3) {  // reading R9: layer reduction through SMEM
    const double s_acc = dt == KAMI_DTYPE_F64 ? 8 : 4;
    t += 2 * (stages - 1) * (double)m * n * s_acc / kBsm;
  }
  return t;
}

}  // namespace

kami_status_t planner_choose(int m, int n, int k, kami_dtype_t dtype, kami_algo_t algo, int p, bool pointer_array,
                             kami_plan_t* out) {
  kami_plan_t r{};
  const bool is16 = dtype != KAMI_DTYPE_F64;
  // 16-bit strided: the tcgen05 family implements 1D with p = 4 sub-partition
  // tensor cores (tc16.cu); it covers the whole 16-bit size grid.  An explicit
  // p > 0 selects the warp-level family with p warps instead.
  if (is16 && !pointer_array && (algo == KAMI_ALGO_AUTO || (algo == KAMI_ALGO_1D && p == 0))) {
    Tc16Shape s;
    kami_status_t st = tc16_plan_shape(m, n, k, &s);
    if (st != KAMI_SUCCESS) return st;
    r.algo = KAMI_ALGO_1D;
    r.p = 4;
    r.kernel = 0;
    r.entries_per_cta = s.G * s.stages;
    r.stages = s.stages;
    r.kslice_regs_pct = 0;  // operands stream through SMEM in k-chunks of s.Wk
    r.t_all_cycles = b200_cost(1, m, n, k, 4, dtype);
    *out = r;
    return KAMI_SUCCESS;
  }
  // warp-level register-resident family
  int cand[3] = {1, 2, 3};
  if (algo != KAMI_ALGO_AUTO) {
    const int pp = p ? p : warp_ca_default_p(m, n, k, dtype, (int)algo);
    if (pp == 0 || warp_ca_supported(m, n, k, dtype, (int)algo, pp) != KAMI_SUCCESS)
      return KAMI_ERROR_NOT_SUPPORTED;
    r.algo = algo;
    r.p = pp;
    r.kernel = 1;
    r.entries_per_cta = pp >= 8 ? 1 : 8 / pp;
    r.stages = 2;
    r.kslice_regs_pct = 100;
    r.t_all_cycles = algo == KAMI_ALGO_NONCA ? 0 : b200_cost((int)algo, m, n, k, pp, dtype);
    *out = r;
    return KAMI_SUCCESS;
  }
  double best = 1e300;
  int best_v = 0, best_p = 0;
  for (int v : cand) {
    const int pp = warp_ca_default_p(m, n, k, dtype, v);
    if (pp == 0) continue;
    const double t = b200_cost(v, m, n, k, pp, dtype);
    if (t < best) {  // strict: ties keep the earlier (1D) schedule
      best = t;
      best_v = v;
      best_p = pp;
    }
  }
  if (best_v == 0) return KAMI_ERROR_NOT_SUPPORTED;
  r.algo = (kami_algo_t)best_v;
  r.p = best_p;
  r.kernel = 1;
  r.entries_per_cta = best_p >= 8 ? 1 : 8 / best_p;
  r.stages = 2;
  r.kslice_regs_pct = 100;
  r.t_all_cycles = best;
  *out = r;
  return KAMI_SUCCESS;
}

}  // namespace kami
