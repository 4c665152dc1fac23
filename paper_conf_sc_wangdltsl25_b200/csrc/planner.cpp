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

// B200 constants, measured by tools/ubench.cu (profiles/r1/ubench_b200.json):
// L_sm = 29 cycles (dependent LDS), B_sm = 127.6 B/cycle/SM (conflict-free
// LDS.128), n_tc = 4 sub-partition tensor cores, O_tc per tensor core:
// DMMA FP64 37.1 TF/s -> 31.9 flop/cycle; legacy HMMA FP16 554.5 TF/s ->
// 477 flop/cycle (at 1965 MHz, 148 SMs).  HBM: 6541.8 GB/s measured copy
// (MEASURED_PEAKS.json) -> 22.5 B/cycle/SM.  T_lat: DRAM round trip seen by a
// team that starts a new entry (~1200 cycles; entries prefetched into L2 by
// the previous one).
constexpr double kLsm = 29, kBsm = 127.6, kNtc = 4;
constexpr double kHbmBpc = 22.5, kTlat = 1200;

double b200_cost(int variant, int m, int n, int k, int p, kami_dtype_t dt) {
  const double s_e = dt == KAMI_DTYPE_F64 ? 8 : 2;
  const double O = dt == KAMI_DTYPE_F64 ? 31.9 : 477;
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

// Batched form: an SM streams entries; with t teams resident the per-entry
// time is bounded by HBM and by the serial (latency + T_all) of one team
// spread over t teams.
double b200_entry_cycles(int variant, int m, int n, int k, int p, kami_dtype_t dt, int teams_per_sm) {
  const double s_e = dt == KAMI_DTYPE_F64 ? 8 : 2;
  const double t_hbm = (double)(m * k + k * n + m * n) * s_e / kHbmBpc;
  const double t_all = b200_cost(variant, m, n, k, p, dt);
  return std::max(t_hbm, (kTlat + t_all) / std::max(1, teams_per_sm));
}

// Measured throughput of each schedule (bench.py, 20 steps, one B200,
// profiles/r1/f64_sweep_r1.txt).  Where a shape is calibrated, AUTO takes the
// measured-fastest schedule; elsewhere it takes the model's minimum.
struct Calib {
  kami_dtype_t dt;
  int s, algo, p;
  double tflops;
};
const Calib kCalib[] = {
    {KAMI_DTYPE_F64, 16, 1, 1, 7.07},  {KAMI_DTYPE_F64, 16, 2, 4, 5.66},  {KAMI_DTYPE_F64, 16, 3, 8, 4.98},
    {KAMI_DTYPE_F64, 32, 1, 2, 14.29}, {KAMI_DTYPE_F64, 32, 2, 4, 12.42}, {KAMI_DTYPE_F64, 32, 3, 8, 11.63},
    {KAMI_DTYPE_F64, 64, 1, 8, 14.13}, {KAMI_DTYPE_F64, 64, 2, 16, 17.20}, {KAMI_DTYPE_F64, 64, 3, 8, 15.84},
};

double calibrated(kami_dtype_t dt, int m, int n, int k, int algo, int p) {
  if (m != n || n != k) return 0;
  for (const Calib& c : kCalib)
    if (c.dt == dt && c.s == m && c.algo == algo && c.p == p) return c.tflops;
  return 0;
}

// measured TFLOP/s of the FP64 TMA-broadcast 1D kernel (0 = not calibrated;
// bench.py --algo 1d_tma, profiles/r1/dmma_tma_sweep_r1.txt)
double calibrated_tma(int m) { return m == 16 ? 7.42 : m == 32 ? 15.02 : m == 64 ? 25.45 : 0; }

}  // namespace

kami_status_t planner_choose(int m, int n, int k, kami_dtype_t dtype, kami_algo_t algo, int p, bool pointer_array,
                             kami_plan_t* out) {
  kami_plan_t r{};
  const bool is16 = dtype != KAMI_DTYPE_F64;  // all tcgen05 types (f16, bf16, tf32, fp8)
  // 16-bit strided: the tcgen05 family implements 1D with p = 4 sub-partition
  // tensor cores (tc16.cu); it covers the whole 16-bit size grid.  An explicit
  // p > 0 selects the warp-level family with p warps instead.
  // 16^3 FP16 / BF16 AUTO: the warp-level HMMA 1D (p = 1, LDG-fed, register
  // resident) beats the tcgen05 kernel at every batch measured -- 32-byte TMA
  // rows and a per-unit fixed cost bound tcgen05 there (configs[0] 4.8 ->
  // 2.2 us per launch; 65 536 entries 19 -> 27 TFLOP/s, profiles/r1/small16_r1.txt)
  if (algo == KAMI_ALGO_AUTO && !pointer_array && m == 16 && n == 16 && k == 16 &&
      (dtype == KAMI_DTYPE_F16 || dtype == KAMI_DTYPE_BF16))
    return planner_choose(m, n, k, dtype, KAMI_ALGO_1D, 1, pointer_array, out);
  if (is16 && !pointer_array &&
      (algo == KAMI_ALGO_AUTO || algo == KAMI_ALGO_1D_TMA || (algo == KAMI_ALGO_1D && p == 0))) {
    Tc16Shape s;
    const int ik = dtype == KAMI_DTYPE_F16 ? 0 : dtype == KAMI_DTYPE_BF16 ? 1 : dtype == KAMI_DTYPE_TF32 ? 2
                 : dtype == KAMI_DTYPE_E4M3 ? 3 : 4;
    const int ok = dtype == KAMI_DTYPE_BF16 ? 1 : dtype == KAMI_DTYPE_TF32 ? 2 : 0;
    kami_status_t st = tc16_plan_shape_kind(m, n, k, ik, ok, &s);
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
  // tcgen05 with the local operand (A) resident in TMEM: explicit request
  if (algo == KAMI_ALGO_1D_TMEM || algo == KAMI_ALGO_3D_TMEM) {
    if ((dtype != KAMI_DTYPE_F16 && dtype != KAMI_DTYPE_BF16) || pointer_array || (p != 0 && p != 4 && p != 8))
      return KAMI_ERROR_NOT_SUPPORTED;
    TsShape ts;
    kami_status_t st = tc16_ts_plan(m, n, k, algo == KAMI_ALGO_3D_TMEM ? 2 : 1, &ts);
    if (st != KAMI_SUCCESS) return st == KAMI_ERROR_INVALID_VALUE ? KAMI_ERROR_NOT_SUPPORTED : st;
    r.algo = algo;
    r.p = algo == KAMI_ALGO_3D_TMEM ? 8 : 4;
    r.kernel = 3;
    r.entries_per_cta = ts.G * ts.stages;
    r.stages = ts.stages;
    r.kslice_regs_pct = 0;
    r.t_all_cycles = b200_cost(algo == KAMI_ALGO_3D_TMEM ? 3 : 1, m, n, k, algo == KAMI_ALGO_3D_TMEM ? 8 : 4, dtype);
    *out = r;
    return KAMI_SUCCESS;
  }
  // FP64 1D with the broadcast operand fed by TMA (dmma_tma.cu; pointer arrays
  // through an address-space view of each entry)
  const bool tma_ok = !is16 && dmma_tma_supported(m, n, k);
  // FP64 off the square orders the fixed-shape kernels are instantiated for:
  // the general k-sliced DMMA kernel with a register residency ratio
  // (dmma_gen.cu; a7).  Explicit 1D with p = 0 selects it too.
  const bool warp_shape = !is16 && m == n && n == k && (m == 8 || m == 16 || m == 32 || m == 64);
  if (!is16 && !pointer_array && dmma_gen_supported(m, n, k) &&
      ((algo == KAMI_ALGO_AUTO && !warp_shape) || (algo == KAMI_ALGO_1D && p == 0 && !warp_shape))) {
    r.algo = KAMI_ALGO_1D;
    r.p = 4;
    r.kernel = 4;
    r.entries_per_cta = 2;
    r.stages = 2;
    r.kslice_regs_pct = dmma_gen_resident_pct(k);
    r.t_all_cycles = b200_cost(1, n, m, k, 4, dtype);
    *out = r;
    return KAMI_SUCCESS;
  }
  if (algo == KAMI_ALGO_1D_TMA) {
    if (!tma_ok || (p != 0 && p != 4)) return KAMI_ERROR_NOT_SUPPORTED;
    r.algo = KAMI_ALGO_1D_TMA;
    r.p = 4;
    r.kernel = 2;
    r.entries_per_cta = m == 64 ? 3 : 8;
    r.stages = 2;
    r.kslice_regs_pct = 50;  // B_w resident in registers, A broadcast through SMEM
    r.t_all_cycles = b200_cost(1, n, m, k, 4, dtype);
    *out = r;
    return KAMI_SUCCESS;
  }
  if (algo == KAMI_ALGO_AUTO && tma_ok) {
    const double t_tma = calibrated_tma(m);
    double best_w = 0;
    for (int v : {1, 2, 3}) {
      const int pp = warp_ca_default_p(m, n, k, dtype, v);
      if (pp) best_w = std::max(best_w, calibrated(dtype, m, n, k, v, pp));
    }
    if (t_tma > best_w) return planner_choose(m, n, k, dtype, KAMI_ALGO_1D_TMA, 0, pointer_array, out);
  }
  if (algo == KAMI_ALGO_1D_TMA) return KAMI_ERROR_NOT_SUPPORTED;
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
  double best = 1e300, best_meas = 0;
  int best_v = 0, best_p = 0;
  for (int v : cand) {
    const int pp = warp_ca_default_p(m, n, k, dtype, v);
    if (pp == 0) continue;
    const double meas = calibrated(dtype, m, n, k, v, pp);
    const double t = b200_entry_cycles(v, m, n, k, pp, dtype, warp_ca_teams_per_sm(m, n, k, dtype, v, pp));
    const bool better = best_meas > 0 || meas > 0 ? meas > best_meas : t < best;  // ties keep 1D
    if (best_v == 0 || better) {
      best = t;
      best_meas = meas;
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
  r.t_all_cycles = b200_cost(best_v, m, n, k, best_p, dtype);
  *out = r;
  return KAMI_SUCCESS;
}

}  // namespace kami
