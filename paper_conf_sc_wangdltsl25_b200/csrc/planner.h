// planner.h -- variant selection for the KAMI kernels (SURVEY.md Sec. 8(a)
// row a1).  Two forms of the paper's cycle model (Eqs. 1-12):
//   paper_cost  -- paper-faithful, p/n_tc without a ceiling (reading R8);
//                  reproduces the worked examples 60 / 68 / 68 cycles.
//   b200 model  -- the same equations with B200 constants and
//                  max(1, p/n_tc) (a warp cannot use a fraction of a
//                  tensor core), plus the 3D layer-reduction term that
//                  Eq. 12 omits (reading R9).
#pragma once
#include "../../include/kami.h"

namespace kami {

struct PaperCost {
  double V_cm, T_cm, T_cp, T_all;
};

PaperCost paper_cost(int variant, double m, double n, double k, double p, double s_e, double L_sm, double B_sm,
                     double theta_r, double theta_w, double O_tc, double n_tc);

kami_status_t planner_choose(int m, int n, int k, kami_dtype_t dtype, kami_algo_t algo, int p, bool pointer_array,
                             kami_plan_t* out);

// every candidate schedule with the model's prediction (kami_plan_candidates)
int planner_candidates(int m, int n, int k, kami_dtype_t dt, bool pointer_array, kami_candidate_t* out, int max);

int warp_ca_default_p(int m, int n, int k, kami_dtype_t dtype, int algo);
int warp_ca_teams_per_sm(int m, int n, int k, kami_dtype_t dtype, int algo, int p);

}  // namespace kami
