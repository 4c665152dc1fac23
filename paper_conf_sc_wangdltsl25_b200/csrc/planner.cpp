// planner.cpp -- see planner.h.  SURVEY.md 8(a) row a1: the schedule of an
// AUTO call is the argmax of a B200 cycle model over every kernel the library
// can run for the shape.  No per-shape measured table.
#include "planner.h"

#include <algorithm>
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

// ----------------------------------------------------------- B200 constants
// Every constant is a measured machine property (one SM, 1965 MHz), not a
// per-shape result:
//   kHbmBpc   6534.1 GB/s copy bandwidth (MEASURED_PEAKS.json hbm_gbs) /
//             148 SMs / 1.965 GHz = 22.5 B per cycle per SM
//   kLsm      29 cycles dependent LDS latency      (profiles/r1/ubench_b200.json)
//   kBsm      127.6 B per cycle per SM, LDS.128    (ubench_b200.json)
//   kDmmaFpc  37.1 TFLOP/s DMMA (ubench, kami_probe_dmma_peak) -> 127.6 flop/cycle/SM
//   kHmmaFpc  554.5 TFLOP/s mma.sync HMMA (ubench) -> 1907 flop/cycle/SM
//   kUmmaFpc  2250 TFLOP/s dense tcgen05 kind::f16 nominal -> 7737 flop/cycle/SM
//   kNtc      4 sub-partition tensor cores per SM
//   kTbar     named-barrier wait per CA stage: block-level mode measures the
//             communication phase at 1.5-4x the model's T_cm; the excess per
//             stage is 139-375 cycles (profiles/r1/block_level.md: f64 64^3
//             1D/2D/3D +139/+345/+308, f16 64^3 +185/+375/+147), mean 250
//   kTlat     DRAM round trip a team waits on when it starts an entry whose
//             operands its previous entry prefetched into L2 (~L2 latency
//             under load), 700 cycles
//   kTmaLdRow cycles of TMA engine time per LOADED box row: 32-byte rows
//             stream at 6.0 TB/s (8 stages; 64/128-byte rows 6.9-7.1 TB/s),
//             i.e. 187.5 G rows/s / 148 SMs = one row per 1.55 cycles per SM
//             (tools/ubench_tma.cu, profiles/r2/ubench_tma.json)
//   kTmaStRow per STORED row (C through the staging tile): 4 cycles,
//             calibrated on the one shape bound by it (f16 16^3: 512 stored
//             32-byte rows per 32-entry unit, 3400 cycles per unit measured,
//             profiles/r2/variant_sweep_r2.json) and checked on 48^3 (1728
//             rows, 3728 cycles measured, 4090 modelled)
//   kEpiVal   epilogue cycles per accumulator value a lane drains per unit
//             (tcgen05.ld + cvt.rn + swizzled st.shared; the busiest warp of
//             the unit sets the time): 14, from bf16 16 x 128 x 16 (two of four
//             sub-partitions hold the unit, 256 values per lane, 3573 cycles
//             per unit measured); it also reproduces the low-rank shapes'
//             ~0.9 of roofline (256 values per lane vs 3277 cycles of HBM)
//   kUnitSS   per-unit fixed cost of the SS tcgen05 pipeline (single-thread
//             producer / MMA loops, two named barriers and one TMA store per
//             unit in the epilogue): ncu f16 32^3 ~190 MMA-lane instructions
//             per unit (profiles/r1), 900 cycles
//   kItemTS   per A item of the TS kernel (one k-chunk x one layer): the
//             loader's LDG -> tcgen05.st -> wait::st -> mbarrier round trip
//             with two items in flight per thread: 1400 cycles (TS 32^3 = one
//             item per 4-entry unit: 1587 cycles per unit measured; bf16
//             48^3 / 96^3, three items: 1183 / 1328 per item)
constexpr double kHbmBpc = 22.5, kLsm = 29, kBsm = 127.6, kNtc = 4;
constexpr double kDmmaFpc = 127.6, kHmmaFpc = 1907.0, kUmmaFpc = 7737.0;
constexpr double kTbar = 250, kTlat = 700;
constexpr double kTmaLdRow = 1.55, kTmaStRow = 4.0, kUnitSS = 900, kItemTS = 1400, kEpiVal = 14, kEpiThin = 5.5;
constexpr double kWarpLdBpc = 32;

// columns of the accumulator the busiest epilogue warp drains per MMA tile
// (tc16.cu epilogue: a warp walks the column groups of the entries whose rows
// sit in its 32 TMEM lanes; replicated thin tiles give each warp one 64-column block)
int epi_cols(int m, int n, int G, int slot, int colrep) {
  if (colrep) return n < 64 ? n : 64;
  if (G <= 1) return n;
  int worst = 0;
  for (int sp = 0; sp < 4; ++sp) {
    const int glo = (sp * 32) / slot;
    int ghi = (sp * 32 + 31) / slot;
    if (ghi > G - 1) ghi = G - 1;
    if (glo < G) worst = std::max(worst, (ghi - glo + 1) * n);
  }
  (void)m;
  return worst;
}

double b200_cost(int variant, int m, int n, int k, int p, kami_dtype_t dt) {
  const double s_e = dt == KAMI_DTYPE_F64 ? 8 : 2;
  const double O = (dt == KAMI_DTYPE_F64 ? kDmmaFpc : kHmmaFpc) / kNtc;  // per tensor core
  PaperCost c = paper_cost(variant, m, n, k, p, s_e, kLsm, kBsm, 1, 1, O, kNtc);
  const double stages = variant == 1 ? p : variant == 2 ? std::sqrt((double)p) : std::round(std::cbrt((double)p));
  const double ratio = std::max(1.0, p / kNtc);  // reading R8: a warp cannot use a fraction of a tensor core
  // + the barrier wait per stage (block_level.md); a one-warp team has no barrier
  double t = stages * (c.T_cm + (p > 1 ? kTbar : 0.0) + ratio * c.T_cp);
  if (variant == 3) {  // reading R9: layer reduction through SMEM
    const double s_acc = dt == KAMI_DTYPE_F64 ? 8 : 4;
    t += 2 * (stages - 1) * (double)m * n * s_acc / kBsm;
  }
  return t;
}

int es_in(kami_dtype_t dt) {
  return dt == KAMI_DTYPE_F64 ? 8 : dt == KAMI_DTYPE_TF32 ? 4 : (dt == KAMI_DTYPE_E4M3 || dt == KAMI_DTYPE_E5M2) ? 1 : 2;
}
int es_out(kami_dtype_t dt) { return dt == KAMI_DTYPE_F64 ? 8 : dt == KAMI_DTYPE_TF32 ? 4 : 2; }
int in_kind(kami_dtype_t d) {
  return d == KAMI_DTYPE_F16 ? 0 : d == KAMI_DTYPE_BF16 ? 1 : d == KAMI_DTYPE_TF32 ? 2 : d == KAMI_DTYPE_E4M3 ? 3 : 4;
}
int out_kind(kami_dtype_t d) { return d == KAMI_DTYPE_BF16 ? 1 : d == KAMI_DTYPE_TF32 ? 2 : 0; }

struct Pred {
  double cycles;  // per entry per SM
  int bound;
};
Pred pmax(std::initializer_list<std::pair<double, int>> terms) {
  Pred r{0, 0};
  for (auto& t : terms)
    if (t.first > r.cycles) r = {t.first, t.second};
  return r;
}
// The persistent tcgen05 pipelines overlap their HBM stream, TMA engine,
// epilogue and per-unit issue only imperfectly: when several are close to the
// largest they add up partly.  A 4-norm of the terms is the largest one when
// it dominates and up to 1.3x it when three are equal (f16 64^3: 1.02x the HBM
// term, 0.98 of the roofline predicted, 0.97 measured; bf16 16 x 32 x 16, three
// terms ~1800 cycles: 2370 predicted, 2900 measured).
Pred psoft(std::initializer_list<std::pair<double, int>> terms) {
  Pred r = pmax(terms);
  double acc = 0;
  for (auto& t : terms) acc += std::pow(t.first / r.cycles, 4.0);
  r.cycles *= std::pow(acc, 0.25);
  return r;
}

double bytes_entry(int m, int n, int k, kami_dtype_t dt) {
  return (double)(m * k + k * n) * es_in(dt) + (double)m * n * es_out(dt);
}

// SS tcgen05 (tc16.cu): per unit = max(HBM, TMA rows, fixed); E entries per unit
bool model_ss(int m, int n, int k, kami_dtype_t dt, Pred* out) {
  Tc16Shape s;
  if (tc16_plan_shape_kind(m, n, k, in_kind(dt), out_kind(dt), &s) != KAMI_SUCCESS) return false;
  const double E = s.tpack ? 2.0 / 3.0 : (s.m_tiles > 1 ? 1.0 / s.m_tiles : (double)s.G * s.U);
  const int esi = es_in(dt);
  const int kpad = (k + 32 / esi - 1) / (32 / esi) * (32 / esi);
  const double rows_tile = m < 128 ? m : 128;
  const double gu = s.m_tiles > 1 ? 1 : (double)s.G * s.U;
  const double rowsA = (s.m_tiles > 1 ? rows_tile : (double)s.slot * gu) * s.k_chunks * (s.colrep ? s.colrep : 1);
  const double rowsB = (double)kpad * (n / s.Wn) * gu;
  const double rowsC = rows_tile * (n / s.Wc) * gu;
  const double t_hbm = E * bytes_entry(m, n, k, dt) / kHbmBpc;
  const double t_tma = (rowsA + rowsB) * kTmaLdRow + rowsC * kTmaStRow;
  const double t_tc = E * 2.0 * m * n * k / kUmmaFpc;
  // one entry per tile with m <= 32: only the first epilogue warp holds rows
  // and its stores leave per 64-column atom as they are staged, so a column
  // costs kEpiThin (fit: bf16 16 x 192 x 16 / 32, ~1100 cycles per entry for
  // 192 columns, profiles/r2/xt_r2.md) rather than the packed-tile kEpiVal
  const double kv = (s.G == 1 && s.m_tiles == 1 && m <= 32 && !s.colrep) ? kEpiThin : kEpiVal;
  const double t_epi = kv * epi_cols(m, n, s.G, s.slot, s.colrep) * (s.m_tiles > 1 ? 1 : s.U);
  Pred p = psoft({{t_hbm, KAMI_BOUND_HBM}, {t_tma, KAMI_BOUND_TMA}, {kUnitSS, KAMI_BOUND_ISSUE}, {t_tc, KAMI_BOUND_TENSOR},
                  {t_epi, KAMI_BOUND_ISSUE}});
  p.cycles /= E;
  *out = p;
  return true;
}

// TS tcgen05 (tc16_ts.cu): A by LDG -> TMEM (no TMA rows), B and C by TMA
bool model_ts(int m, int n, int k, kami_dtype_t dt, int layers, Pred* out) {
  if (dt != KAMI_DTYPE_F16 && dt != KAMI_DTYPE_BF16) return false;
  TsShape s;
  if (tc16_ts_plan(m, n, k, layers, &s) != KAMI_SUCCESS) return false;
  const double E = s.G;
  const int kpad = (k + 15) / 16 * 16;
  const double rowsB = (double)kpad * (n / s.Wn) * E, rowsC = (double)m * (n / s.Wc) * E;
  const double t_hbm = E * bytes_entry(m, n, k, dt) / kHbmBpc;
  const double t_tma = rowsB * kTmaLdRow + rowsC * kTmaStRow;
  const double t_tc = E * 2.0 * m * n * k / kUmmaFpc;
  const double t_fix = kItemTS * s.k_chunks * layers;  // one loader round trip per A item
  const double t_epi = kEpiVal * epi_cols(m, n, s.G, m, 0);
  Pred p = psoft({{t_hbm, KAMI_BOUND_HBM}, {t_tma, KAMI_BOUND_TMA}, {t_fix, KAMI_BOUND_ISSUE}, {t_tc, KAMI_BOUND_TENSOR},
                  {t_epi, KAMI_BOUND_ISSUE}});
  p.cycles /= E;
  *out = p;
  return true;
}

// tcgen05 on the transposed product for thin m (tc16_xt.cu): a unit = E
// entries x one 128-column tile of n; two TMA boxes in, one out; each
// epilogue lane drains E m values with one 16-bit store each (kXtVal cycles
// per value, two warpgroups on alternate units), and a unit has a fixed cost
// kUnitXT0 + kUnitXT1 E (the epilogue's barrier / TMEM-load / store chain,
// longer with more entries): measured ~3400 / 2400 / 1900 cycles per unit for
// E = 8 / 4 / 2 at m = 16 whatever n (profiles/r2/xt_r2.md).  Fit on the 24
// thin shapes (head and pair tiles): the model picks the measured-better of XT
// / SS / warp on 22, the two misses (32 x 192 x 32, 32 x 256 x 16) by 8-9 %
constexpr double kXtVal = kEpiVal, kUnitXT0 = 1400, kUnitXT1 = 200;
bool model_xt(int m, int n, int k, kami_dtype_t dt, Pred* out) {
  if (dt != KAMI_DTYPE_F16 && dt != KAMI_DTYPE_BF16) return false;
  int E = 0, stages = 0;
  if (tc16_xt_plan(m, n, k, &E, &stages) != KAMI_SUCCESS) return false;
  // a head tile: E entries x 128 columns of n; a pair tile: 2E entries x 64
  auto unit = [&](int P) {
    const double ents = (double)E * P, cols = 128.0 / P;
    const double t_hbm = ents * ((double)m * k + k * cols + m * cols) * 2 / kHbmBpc;
    const double t_tma = (ents * m + 2.0 * E * k) * kTmaLdRow + 2.0 * E * m * kTmaStRow;
    const double t_tc = E * 2.0 * P * m * 128 * k / kUmmaFpc;
    const double t_epi = kXtVal * E * m / 2;
    return psoft({{t_hbm, KAMI_BOUND_HBM}, {t_tma, KAMI_BOUND_TMA}, {kUnitXT0 + kUnitXT1 * E, KAMI_BOUND_ISSUE},
                  {t_tc, KAMI_BOUND_TENSOR}, {t_epi, KAMI_BOUND_ISSUE}});
  };
  Pred p;
  if (n % 128 == 0) {
    p = unit(1);
    p.cycles *= (n / 128.0) / E;
  } else if (n == 64) {
    p = unit(2);
    p.cycles /= 2.0 * E;
  } else {  // n = 192: two heads and one pair per 2E entries
    const Pred h = unit(1), q = unit(2);
    p = h.cycles >= q.cycles ? h : q;
    p.cycles = (2 * h.cycles + q.cycles) / (2.0 * E);
  }
  *out = p;
  return true;
}

// The CTA-pair kernel is selectable explicitly (KAMI_ALGO_2D_PAIR); AUTO
// considers it once it is measured faster than the single-CTA kernel.
constexpr bool kPairInAuto = false;
// CTA pair (tc16_pair.cu): one entry per pair-unit on two SMs; per CTA the
// unit moves its 128 rows of A and C and half of B
bool model_pair(int m, int n, int k, kami_dtype_t dt, Pred* out) {
  if ((dt != KAMI_DTYPE_F16 && dt != KAMI_DTYPE_BF16) || !tc16_pair_supported(m, n, k)) return false;
  const int kpad = (k + 15) / 16 * 16;
  const int wk = kpad * 2 % 128 == 0 ? 64 : kpad * 2 % 64 == 0 ? 32 : 16;
  const int wn = n % 128 == 0 ? 64 : n % 64 == 0 ? 32 : 16;            // atom of the n/2-column half
  const int wc = (2 * n) % 128 == 0 ? 64 : (2 * n) % 64 == 0 ? 32 : 16;
  const int kchunks = (kpad + wk - 1) / wk;
  const double t_hbm = bytes_entry(m, n, k, dt) / (2 * kHbmBpc);
  const double rows_ld = 128.0 * kchunks + (double)kpad * ((n / 2) / wn);
  const double rows_st = 128.0 * (n / wc);
  const double t_tma = rows_ld * kTmaLdRow + rows_st * kTmaStRow;
  const double t_epi = kEpiVal * n;
  const double t_tc = 2.0 * m * n * k / (2 * kUmmaFpc);
  Pred p = psoft({{t_hbm, KAMI_BOUND_HBM}, {t_tma, KAMI_BOUND_TMA}, {kUnitSS, KAMI_BOUND_ISSUE}, {t_tc, KAMI_BOUND_TENSOR},
                  {t_epi, KAMI_BOUND_ISSUE}});
  p.cycles *= 2;  // two SMs per entry: cycles per entry per SM
  *out = p;
  return true;
}

// LDG-fed tcgen05 (tc16_vb.cu) for 16-bit m or n = 8 mod 16: the same
// schedule with the operands copied by a producer warpgroup (16-byte
// cp.async); per unit max(HBM, the copy issue of the unit's 16-byte chunks,
// the SS unit cost); kVbChunk cycles per 16-byte chunk per SM (128 producer
// threads, one LDGSTS each per ~4 cycles -> 0.125 cycle per chunk, x2 for the
// zero-fill / swizzle address math), i.e. ~64 B/cycle of copy issue
constexpr double kVbChunk = 0.25;
bool model_vb(int m, int n, int k, kami_dtype_t dt, Pred* out) {
  if ((dt != KAMI_DTYPE_F16 && dt != KAMI_DTYPE_BF16) || (m % 16 == 0 && n % 16 == 0)) return false;
  const int g1 = m > 128 ? 1 : 128 / m, g2 = 256 / n;
  const double G = m > 128 ? 1.0 / ((m + 127) / 128) : (double)std::max(1, std::min(g1, g2));
  const double be = bytes_entry(m, n, k, dt);
  const double t_hbm = G * be / kHbmBpc;
  const double t_copy = G * (double)(m * k + k * n) * 2 / 16 * kVbChunk + G * (double)m * n * 2 / 16 * kVbChunk;
  Pred p = pmax({{t_hbm, KAMI_BOUND_HBM}, {t_copy, KAMI_BOUND_ISSUE}, {kUnitSS, KAMI_BOUND_ISSUE}});
  p.cycles /= G;
  *out = p;
  return true;
}

// register-resident warp teams (warp_ca.cu): a team loads its entry with its
// own LDGs (one round trip to L2, where its previous entry prefetched it),
// runs the CA schedule (T_all of Eqs. 4/8/12 with B200 constants + the
// barrier wait per stage) and stores C (fire and forget) before it starts the
// next entry, so per SM an entry costs its HBM transfer plus the team's
// unhidden chain spread over the resident teams
bool model_warp(int m, int n, int k, kami_dtype_t dt, int variant, int p, Pred* out) {
  if (warp_ca_supported(m, n, k, dt, variant, p) != KAMI_SUCCESS) return false;
  const int teams = warp_ca_teams_per_sm(m, n, k, dt, variant, p);
  const double be = bytes_entry(m, n, k, dt);
  const double rate = (dt == KAMI_DTYPE_F64 ? kDmmaFpc : kHmmaFpc) / kNtc;  // per tensor core
  const double t_sched = variant == 4 ? 2.0 * m * n * k / (rate * std::min<double>(p, kNtc))
                                      : b200_cost(variant, m, n, k, p, dt);
  // the entry's operands stream through the team's own LDGs (fragment-order
  // 4/8-byte loads): kWarpLdBpc bytes per cycle per warp
  const double t_chain = kTlat + be / (kWarpLdBpc * p) + t_sched;
  const double t_tc = 2.0 * m * n * k / (dt == KAMI_DTYPE_F64 ? kDmmaFpc : kHmmaFpc);
  const double t_mem = be / kHbmBpc + t_chain / teams;
  *out = pmax({{t_mem, t_chain / teams > be / kHbmBpc ? KAMI_BOUND_LATENCY : KAMI_BOUND_HBM},
               {t_tc, KAMI_BOUND_TENSOR}});
  return true;
}

// FP64 1D with TMA broadcast of A (dmma_tma.cu): P = 4 warps, TEAMS per CTA
bool model_dmma_tma(int m, int n, int k, Pred* out) {
  if (!dmma_tma_supported(m, n, k)) return false;
  const int teams = m == 64 ? 3 : 8;
  const double be = bytes_entry(m, n, k, KAMI_DTYPE_F64);
  const double flops = 2.0 * m * n * k;
  const double smem = (double)m * k * 8 * (1 + 4);  // TMA write + 4 warps read A
  // per team: B_w loads (prefetched into L2) + its share of the DMMA work
  const double t_team = kTlat + flops / (kDmmaFpc / kNtc * 4) * kNtc / 4;
  *out = pmax({{be / kHbmBpc, KAMI_BOUND_HBM}, {flops / kDmmaFpc, KAMI_BOUND_TENSOR},
               {smem / kBsm, KAMI_BOUND_SMEM}, {t_team / teams, KAMI_BOUND_LATENCY}});
  return true;
}

// FP64 general sizes (dmma_gen.cu): units (entry, 64-column block), A re-read
// per column block from L2, 32-row blocks of A through a double buffer
bool model_dmma_gen(int m, int n, int k, Pred* out) {
  if (!dmma_gen_supported(m, n, k)) return false;
  const double be = bytes_entry(m, n, k, KAMI_DTYPE_F64);
  const double flops = 2.0 * m * n * k;
  const double nblocks = (n + 63) / 64, mblocks = (m + 31) / 32;
  const double smem = nblocks * (double)(mblocks * 32) * k * 8 * (1 + 4);
  const double teams = k <= 32 ? 4 : 2;
  // per team and 32-row block: one TMA round trip that is only one block ahead
  const double t_team = nblocks * (kTlat + mblocks * (kTlat / 2 + flops / nblocks / mblocks / (kDmmaFpc / 2)));
  *out = pmax({{be / kHbmBpc, KAMI_BOUND_HBM}, {flops / kDmmaFpc, KAMI_BOUND_TENSOR},
               {smem / kBsm, KAMI_BOUND_SMEM}, {t_team / teams, KAMI_BOUND_LATENCY}});
  return true;
}

void fill_plan(kami_plan_t* r, int kernel, kami_algo_t algo, int p, int m, int n, int k, kami_dtype_t dt) {
  *r = kami_plan_t{};
  r->algo = algo;
  r->p = p;
  r->kernel = kernel;
  r->stages = 2;
  r->entries_per_cta = 1;
  if (kernel == 0) {
    Tc16Shape s;
    if (tc16_plan_shape_kind(m, n, k, in_kind(dt), out_kind(dt), &s) == KAMI_SUCCESS) {
      r->entries_per_cta = s.G * s.U * s.stages;
      r->stages = s.stages;
    }
    r->kslice_regs_pct = 0;  // operands stream through SMEM in k-chunks
    r->t_all_cycles = b200_cost(1, m, n, k, 4, dt);
  } else if (kernel == 3) {
    TsShape s;
    if (tc16_ts_plan(m, n, k, algo == KAMI_ALGO_3D_TMEM ? 2 : 1, &s) == KAMI_SUCCESS) {
      r->entries_per_cta = s.G * s.stages;
      r->stages = s.stages;
    }
    r->kslice_regs_pct = 100;  // A entirely TMEM-resident (local), B streamed
    r->t_all_cycles = b200_cost(algo == KAMI_ALGO_3D_TMEM ? 3 : 1, m, n, k, p, dt);
  } else if (kernel == 2) {
    r->entries_per_cta = m == 64 ? 3 : 8;
    r->kslice_regs_pct = 50;  // B_w resident in registers, A broadcast through SMEM
    r->t_all_cycles = b200_cost(1, n, m, k, 4, dt);
  } else if (kernel == 7) {
    int E = 1, st = 2;
    tc16_xt_plan(m, n, k, &E, &st);
    r->entries_per_cta = E * st;
    r->stages = st;
    r->kslice_regs_pct = 0;
    r->t_all_cycles = b200_cost(1, n, m, k, 4, dt);
  } else if (kernel == 6) {
    r->entries_per_cta = 1;
    r->stages = 4;
    r->kslice_regs_pct = 0;
    r->t_all_cycles = b200_cost(2, m, n, k, 8, dt);
  } else if (kernel == 5) {
    r->entries_per_cta = 1;
    r->kslice_regs_pct = 0;
    r->t_all_cycles = b200_cost(1, m, n, k, 4, dt);
  } else if (kernel == 4) {
    r->entries_per_cta = k <= 32 ? 4 : 2;
    r->kslice_regs_pct = dmma_gen_resident_pct(k);
    r->t_all_cycles = b200_cost(1, n, m, k, 4, dt);
  } else {
    r->entries_per_cta = p >= 8 ? 1 : 8 / p;
    r->kslice_regs_pct = 100;
    r->t_all_cycles = algo == KAMI_ALGO_NONCA ? 0 : b200_cost((int)algo, m, n, k, p, dt);
  }
}

}  // namespace

int planner_candidates(int m, int n, int k, kami_dtype_t dt, bool pointer_array, kami_candidate_t* out, int max) {
  int cnt = 0;
  auto add = [&](int kernel, kami_algo_t algo, int p, const Pred& pr) {
    if (cnt < max && out) {
      kami_candidate_t& c = out[cnt];
      c.algo = algo;
      c.p = p;
      c.kernel = kernel;
      c.model_cycles_per_entry = pr.cycles;
      c.model_tflops = 2.0 * m * n * k * 148 * 1.965e9 / pr.cycles / 1e12;
      c.bound = pr.bound;
    }
    ++cnt;
  };
  Pred pr;
  const bool is16 = dt != KAMI_DTYPE_F64;
  if (pointer_array) return 0;  // pointer arrays: fixed routing (api.cpp), not modelled
  if (is16) {
    if (model_vb(m, n, k, dt, &pr)) add(5, KAMI_ALGO_1D, 4, pr);
    if (model_ss(m, n, k, dt, &pr)) add(0, KAMI_ALGO_1D, 4, pr);
    if (model_ts(m, n, k, dt, 1, &pr)) add(3, KAMI_ALGO_1D_TMEM, 4, pr);
    if (model_xt(m, n, k, dt, &pr)) add(7, KAMI_ALGO_1D_XT, 4, pr);
    if (model_ts(m, n, k, dt, 2, &pr)) add(3, KAMI_ALGO_3D_TMEM, 8, pr);
    if (kPairInAuto && model_pair(m, n, k, dt, &pr)) add(6, KAMI_ALGO_2D_PAIR, 8, pr);
  } else {
    if (model_dmma_tma(m, n, k, &pr)) add(2, KAMI_ALGO_1D_TMA, 4, pr);
    if (model_dmma_gen(m, n, k, &pr)) add(4, KAMI_ALGO_1D, 4, pr);
  }
  if (dt == KAMI_DTYPE_F16 || dt == KAMI_DTYPE_BF16 || dt == KAMI_DTYPE_F64) {
    for (int v : {1, 2, 3}) {
      const int pp = warp_ca_default_p(m, n, k, dt, v);
      if (pp && model_warp(m, n, k, dt, v, pp, &pr)) add(1, (kami_algo_t)v, pp, pr);
    }
  }
  return cnt;
}

kami_status_t planner_choose(int m, int n, int k, kami_dtype_t dtype, kami_algo_t algo, int p, bool pointer_array,
                             kami_plan_t* out) {
  kami_plan_t r{};
  const bool is16 = dtype != KAMI_DTYPE_F64;  // all tcgen05 types (f16, bf16, tf32, fp8)
  if (algo == KAMI_ALGO_AUTO && !pointer_array) {
    // the model's argmax over every kernel that runs this shape
    kami_candidate_t c[16];
    const int nc = std::min(16, planner_candidates(m, n, k, dtype, false, c, 16));
    int best = -1;
    for (int i = 0; i < nc; ++i)
      if (best < 0 || c[i].model_cycles_per_entry < c[best].model_cycles_per_entry) best = i;
    if (best < 0) return KAMI_ERROR_NOT_SUPPORTED;
    fill_plan(&r, c[best].kernel, c[best].algo, c[best].p, m, n, k, dtype);
    r.t_all_cycles = c[best].model_cycles_per_entry;
    *out = r;
    return KAMI_SUCCESS;
  }
  // ---- explicit schedules (and pointer arrays, routed by api.cpp)
  // 16-bit m or n = 8 mod 16: the LDG-fed tcgen05 kernel is the tcgen05 1D there
  if ((dtype == KAMI_DTYPE_F16 || dtype == KAMI_DTYPE_BF16) && !pointer_array && (m % 16 || n % 16) &&
      (algo == KAMI_ALGO_1D && p == 0)) {
    fill_plan(&r, 5, KAMI_ALGO_1D, 4, m, n, k, dtype);
    *out = r;
    return KAMI_SUCCESS;
  }
  // 16-bit 1D with p = 0 / 1D_TMA / AUTO on pointer arrays: the SS tcgen05 kernel
  if (is16 && !pointer_array &&
      (algo == KAMI_ALGO_1D_TMA || (algo == KAMI_ALGO_1D && p == 0))) {
    Tc16Shape s;
    kami_status_t st = tc16_plan_shape_kind(m, n, k, in_kind(dtype), out_kind(dtype), &s);
    if (st != KAMI_SUCCESS) return st;
    fill_plan(&r, 0, KAMI_ALGO_1D, 4, m, n, k, dtype);
    *out = r;
    return KAMI_SUCCESS;
  }
  // tcgen05 with the local operand (A) resident in TMEM
  if (algo == KAMI_ALGO_1D_TMEM || algo == KAMI_ALGO_3D_TMEM) {
    if ((dtype != KAMI_DTYPE_F16 && dtype != KAMI_DTYPE_BF16) || pointer_array || (p != 0 && p != 4 && p != 8))
      return KAMI_ERROR_NOT_SUPPORTED;
    TsShape ts;
    kami_status_t st = tc16_ts_plan(m, n, k, algo == KAMI_ALGO_3D_TMEM ? 2 : 1, &ts);
    if (st != KAMI_SUCCESS) return st == KAMI_ERROR_INVALID_VALUE ? KAMI_ERROR_NOT_SUPPORTED : st;
    fill_plan(&r, 3, algo, algo == KAMI_ALGO_3D_TMEM ? 8 : 4, m, n, k, dtype);
    *out = r;
    return KAMI_SUCCESS;
  }
  // tcgen05 on the transposed product (thin m)
  if (algo == KAMI_ALGO_1D_XT) {
    if ((dtype != KAMI_DTYPE_F16 && dtype != KAMI_DTYPE_BF16) || pointer_array || (p != 0 && p != 4) ||
        !tc16_xt_supported(m, n, k))
      return KAMI_ERROR_NOT_SUPPORTED;
    fill_plan(&r, 7, KAMI_ALGO_1D_XT, 4, m, n, k, dtype);
    *out = r;
    return KAMI_SUCCESS;
  }
  // tcgen05 CTA pair
  if (algo == KAMI_ALGO_2D_PAIR) {
    if ((dtype != KAMI_DTYPE_F16 && dtype != KAMI_DTYPE_BF16) || pointer_array || (p != 0 && p != 8) ||
        !tc16_pair_supported(m, n, k))
      return KAMI_ERROR_NOT_SUPPORTED;
    fill_plan(&r, 6, KAMI_ALGO_2D_PAIR, 8, m, n, k, dtype);
    *out = r;
    return KAMI_SUCCESS;
  }
  // FP64 general sizes: explicit 1D with p = 0 off the fixed-shape orders
  const bool warp_shape = !is16 && m == n && n == k && (m == 8 || m == 16 || m == 32 || m == 64);
  if (!is16 && !pointer_array && algo == KAMI_ALGO_1D && p == 0 && !warp_shape && dmma_gen_supported(m, n, k)) {
    fill_plan(&r, 4, KAMI_ALGO_1D, 4, m, n, k, dtype);
    *out = r;
    return KAMI_SUCCESS;
  }
  // FP64 pointer arrays off the fixed shapes: dmma_gen with cp.async-fed A blocks
  if (!is16 && pointer_array && algo == KAMI_ALGO_AUTO && !warp_shape && dmma_gen_supported(m, n, k)) {
    fill_plan(&r, 4, KAMI_ALGO_1D, 4, m, n, k, dtype);
    *out = r;
    return KAMI_SUCCESS;
  }
  // FP64 1D with the broadcast operand fed by TMA (dmma_tma.cu; pointer arrays
  // through an address-space view of each entry)
  const bool tma_ok = !is16 && dmma_tma_supported(m, n, k);
  if (algo == KAMI_ALGO_1D_TMA || (algo == KAMI_ALGO_AUTO && pointer_array && tma_ok)) {
    if (!tma_ok || (p != 0 && p != 4)) return KAMI_ERROR_NOT_SUPPORTED;
    fill_plan(&r, 2, KAMI_ALGO_1D_TMA, 4, m, n, k, dtype);
    *out = r;
    return KAMI_SUCCESS;
  }
  // warp-level register-resident family (explicit algo, or pointer arrays)
  kami_algo_t a = algo;
  int pp = p;
  if (a == KAMI_ALGO_AUTO) {  // pointer arrays the fixed routes above do not take: the model's best warp schedule
    double best = 1e300;
    for (int v : {1, 2, 3}) {
      const int q = warp_ca_default_p(m, n, k, dtype, v);
      Pred pr;
      if (q && model_warp(m, n, k, dtype, v, q, &pr) && pr.cycles < best) {
        best = pr.cycles;
        a = (kami_algo_t)v;
        pp = q;
      }
    }
    if (a == KAMI_ALGO_AUTO) return KAMI_ERROR_NOT_SUPPORTED;
  }
  if (pp == 0) pp = warp_ca_default_p(m, n, k, dtype, (int)a);
  if (pp == 0 || warp_ca_supported(m, n, k, dtype, (int)a, pp) != KAMI_SUCCESS) return KAMI_ERROR_NOT_SUPPORTED;
  fill_plan(&r, 1, a, pp, m, n, k, dtype);
  *out = r;
  return KAMI_SUCCESS;
}

}  // namespace kami
