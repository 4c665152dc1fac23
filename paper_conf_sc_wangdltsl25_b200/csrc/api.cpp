// api.cpp -- the C ABI of libkami.so (include/kami.h): argument validation
// (all before any launch), layout handling, planner, dispatch to the kernel
// families, the chunked host-memory entry point, status strings.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>

#include "../../include/kami.h"
#include "kernels.h"
#include "planner.h"

namespace kami {

static thread_local const char* g_last_kernel = "";
void set_last_kernel(const char* name) { g_last_kernel = name; }
static thread_local int g_last_cuda = 0;
int launch_status(int e) {
  if (e != 0) g_last_cuda = e;
  return e == 0 ? KAMI_SUCCESS : KAMI_ERROR_CUDA;
}
static std::atomic<int> g_grid_cap{0};
int grid_cap() { return g_grid_cap.load(std::memory_order_relaxed); }

PFN_encodeTiled get_encode_tiled() {
  static PFN_encodeTiled fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_encodeTiled>(p);
  });
  return fn;
}

namespace {

bool is16(kami_dtype_t d) { return d == KAMI_DTYPE_F16 || d == KAMI_DTYPE_BF16; }
bool is_tc(kami_dtype_t d) { return d != KAMI_DTYPE_F64; }  // tcgen05 types
int in_kind(kami_dtype_t d) {  // tc16.cu input kinds
  return d == KAMI_DTYPE_F16 ? 0 : d == KAMI_DTYPE_BF16 ? 1 : d == KAMI_DTYPE_TF32 ? 2 : d == KAMI_DTYPE_E4M3 ? 3 : 4;
}
int out_kind(kami_dtype_t d) { return d == KAMI_DTYPE_BF16 ? 1 : d == KAMI_DTYPE_TF32 ? 2 : 0; }
bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

// Size grid (R5).  Checked before anything touches the device.
kami_status_t check_sizes(int m, int n, int k, kami_dtype_t dtype) {
  if (m > 256 || n > 256 || k > 256) return KAMI_ERROR_NOT_SUPPORTED;
  if (is16(dtype)) return (m % 8 || n % 8 || k % 8) ? KAMI_ERROR_NOT_SUPPORTED : KAMI_SUCCESS;
  if (dtype == KAMI_DTYPE_TF32) return (m % 16 || n % 16 || k % 4) ? KAMI_ERROR_NOT_SUPPORTED : KAMI_SUCCESS;
  if (dtype == KAMI_DTYPE_E4M3 || dtype == KAMI_DTYPE_E5M2)
    return (m % 32 || n % 32 || k % 16) ? KAMI_ERROR_NOT_SUPPORTED : KAMI_SUCCESS;
  // FP64: multiples of 8 in [8, 256] (dmma_gen.cu covers the whole grid)
  return (m % 8 || n % 8 || k % 8) ? KAMI_ERROR_NOT_SUPPORTED : KAMI_SUCCESS;
}

kami_status_t check_common(int m, int n, int k, int64_t batch, int dtype, int layout, int algo) {
  if (m <= 0 || n <= 0 || k <= 0 || batch < 0) return KAMI_ERROR_INVALID_VALUE;
  if (dtype < KAMI_DTYPE_F16 || dtype > KAMI_DTYPE_E5M2) return KAMI_ERROR_INVALID_VALUE;
  if (layout != KAMI_ROW_MAJOR && layout != KAMI_COL_MAJOR) return KAMI_ERROR_INVALID_VALUE;
  if (algo < KAMI_ALGO_AUTO || algo > KAMI_ALGO_1D_XT) return KAMI_ERROR_INVALID_VALUE;
  return check_sizes(m, n, k, (kami_dtype_t)dtype);
}

// Row-major problem after the layout transform.  Column-major C = A B is the
// row-major problem C^T = B^T A^T on the same buffers: (m, n, A, B) ->
// (n, m, B, A)  (pinned by the transpose identity).
struct RowProblem {
  int m, n, k;
  const void* A;
  const void* B;
  const void* const* Aa;
  const void* const* Ba;
};

RowProblem to_row(int m, int n, int k, kami_layout_t layout, const void* A, const void* B, const void* const* Aa,
                  const void* const* Ba) {
  if (layout == KAMI_ROW_MAJOR) return {m, n, k, A, B, Aa, Ba};
  return {n, m, k, B, A, Ba, Aa};
}

// Experiment knob for A/B runs (unset in production): KAMI_PTR_ROUTE = tma | vb | warp
// forces the kernel 16-bit pointer arrays take (1 / 2 / 3; 0 = planner rule).
int ptr_route() {
  static const int r = [] {
    const char* e = getenv("KAMI_PTR_ROUTE");
    if (!e) return 0;
    return !strcmp(e, "tma") ? 1 : !strcmp(e, "vb") ? 2 : !strcmp(e, "warp") ? 3 : 0;
  }();
  return r;
}

kami_status_t dispatch(const RowProblem& rp, int64_t batch, kami_dtype_t dtype, kami_algo_t algo, int p, void* C,
                       void* const* Ca, cudaStream_t stream, double alpha = 1.0, double beta = 0.0) {
  const bool update = alpha != 1.0 || beta != 0.0;
  if (!is16(dtype) && dtype != KAMI_DTYPE_F64) {  // TF32 / FP8: tcgen05 1D only, strided only
    if (Ca || (algo != KAMI_ALGO_AUTO && algo != KAMI_ALGO_1D && algo != KAMI_ALGO_1D_TMA) || p)
      return KAMI_ERROR_NOT_SUPPORTED;
    return tc16_launch_kind(rp.m, rp.n, rp.k, batch, in_kind(dtype), out_kind(dtype), rp.A, rp.B, C, (float)alpha,
                            (float)beta, stream, 0);
  }
  // 16-bit pointer arrays: the TMA tcgen05 kernel over address-space views
  // (tc16.cu kPtr; f16 x 65 536: 32^3 58.0, 64^3 140.3, 128^3 280.9, 256x256x16
  // 77.7 TFLOP/s vs 26.6 / 109.5 / 279.4 / 56.1 on the LDG-fed kernel), except
  // k = 8 mod 16 (LDG-fed, see tc16.cu) and 16^3, where the warp-level HMMA
  // 1D is faster (21.7 vs 10.9 TFLOP/s), profiles/r1/ptr_ab_r1.txt
  const int route = ptr_route();
  const bool ptr_warp = Ca && is16(dtype) && algo == KAMI_ALGO_AUTO && rp.m == rp.n && rp.n == rp.k &&
                        rp.m <= 16 && warp_ca_default_p(rp.m, rp.n, rp.k, dtype, 1) != 0;
  if (((ptr_warp && route == 0) || route == 3) && !update)
    return warp_ca_launch(rp.m, rp.n, rp.k, batch, dtype, 1, warp_ca_default_p(rp.m, rp.n, rp.k, dtype, 1), rp.A,
                          rp.B, C, rp.Aa, rp.Ba, Ca, stream);
  if (Ca && is16(dtype) && algo == KAMI_ALGO_AUTO) {
    // the TMA kernel over address-space views (tc16.cu kPtr), else the LDG-fed one
    if (route != 2 && rp.m % 16 == 0 && rp.n % 16 == 0) {
      kami_status_t st = tc16_launch_kind(rp.m, rp.n, rp.k, batch, in_kind(dtype), out_kind(dtype), nullptr,
                                          nullptr, nullptr, 1.0f, 0.0f, stream, 0, rp.Aa, rp.Ba, Ca);
      if (st != KAMI_ERROR_NOT_SUPPORTED) return st;
    }
    return tc16_vb_launch(batch, dtype == KAMI_DTYPE_BF16, rp.m, rp.n, rp.k, nullptr, nullptr, nullptr, rp.m, rp.n,
                          rp.Aa, rp.Ba, Ca, stream);
  }
  kami_plan_t plan;
  kami_status_t st = planner_choose(rp.m, rp.n, rp.k, dtype, algo, p, /*pointer_array=*/Ca != nullptr, &plan);
  if (st != KAMI_SUCCESS) return st;
  if (plan.kernel == 7 && !update && !Ca)  // thin m: tcgen05 on C^T = B^T A^T (strided C = A B)
    return tc16_xt_launch(rp.m, rp.n, rp.k, batch, dtype == KAMI_DTYPE_BF16, rp.A, rp.B, C, stream);
  if (plan.kernel == 7) {
    if (algo != KAMI_ALGO_AUTO) return KAMI_ERROR_NOT_SUPPORTED;
    plan.kernel = 0;  // the update form / pointer arrays: the SS tcgen05 kernel
  }
  if (plan.kernel == 6) {  // tcgen05 CTA pair (strided C = A B)
    if (update || Ca) return KAMI_ERROR_NOT_SUPPORTED;
    return tc16_pair_launch(rp.m, rp.n, rp.k, batch, dtype == KAMI_DTYPE_BF16, rp.A, rp.B, C, stream);
  }
  if (plan.kernel == 5) {  // 16-bit m or n = 8 mod 16: the LDG-fed tcgen05 kernel on packed entries
    if (update || Ca) return KAMI_ERROR_NOT_SUPPORTED;
    return tc16_vb_strided_launch(rp.m, rp.n, rp.k, batch, dtype == KAMI_DTYPE_BF16, rp.A, rp.B, C, stream);
  }
  if (plan.kernel == 4) {  // FP64 general sizes: k-sliced DMMA with a residency ratio (C = A B)
    if (update) return KAMI_ERROR_NOT_SUPPORTED;
    return dmma_gen_launch(rp.m, rp.n, rp.k, batch, rp.A, rp.B, C, stream, rp.Aa, rp.Ba, Ca);
  }
  if (plan.kernel == 3) {  // tcgen05 with A resident in TMEM (strided C = A B only)
    if (update || Ca) return KAMI_ERROR_NOT_SUPPORTED;
    return tc16_ts_launch(rp.m, rp.n, rp.k, batch, dtype == KAMI_DTYPE_BF16, plan.algo == KAMI_ALGO_3D_TMEM ? 2 : 1,
                          rp.A, rp.B, C, stream);
  }
  if ((plan.kernel == 1 || plan.kernel == 3 || plan.kernel == 6) && update && is16(dtype) && algo == KAMI_ALGO_AUTO &&
      !Ca)
    plan.kernel = 0;  // the update form (C read) exists on the SS tcgen05 kernel only
  if ((plan.kernel == 4 || plan.kernel == 1) && update && algo == KAMI_ALGO_AUTO && !Ca &&
      dmma_tma_supported(rp.m, rp.n, rp.k))
    plan.kernel = 2;  // FP64 update form: the TMA-broadcast DMMA kernel
  if (plan.kernel == 0) {
    return tc16_launch_kind(rp.m, rp.n, rp.k, batch, in_kind(dtype), out_kind(dtype), rp.A, rp.B, C, (float)alpha,
                            (float)beta, stream, 0);
  }
  if (plan.kernel == 2) {
    if (Ca) {  // pointer arrays: the TMA view, else the register-resident family
      kami_status_t st = dmma_tma_launch(rp.m, rp.n, rp.k, batch, nullptr, nullptr, nullptr, stream, 1.0, 0.0,
                                         rp.Aa, rp.Ba, Ca);
      if (st != KAMI_ERROR_NOT_SUPPORTED || update) return st;
      if (planner_choose(rp.m, rp.n, rp.k, dtype, KAMI_ALGO_2D, 0, true, &plan) != KAMI_SUCCESS) return st;
    } else {
      return dmma_tma_launch(rp.m, rp.n, rp.k, batch, rp.A, rp.B, C, stream, alpha, beta);
    }
  }
  if (update) return KAMI_ERROR_NOT_SUPPORTED;  // the warp-level family has no update form
  return warp_ca_launch(rp.m, rp.n, rp.k, batch, dtype, (int)plan.algo, plan.p, rp.A, rp.B, C, rp.Aa, rp.Ba, Ca,
                        stream);
}

}  // namespace
}  // namespace kami

using namespace kami;

extern "C" {

kami_status_t kami_gemm_strided_batched_ex(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                           kami_layout_t layout, const void* A, const void* B, void* C,
                                           kami_algo_t algo, int p, kami_stream_t stream) {
  kami_status_t st = check_common(m, n, k, batch, dtype, layout, algo);
  if (st != KAMI_SUCCESS) return st;
  if (p < 0) return KAMI_ERROR_INVALID_VALUE;
  if (batch == 0) return KAMI_SUCCESS;
  if (!A || !B || !C) return KAMI_ERROR_INVALID_VALUE;
  if (!aligned16(A) || !aligned16(B) || !aligned16(C)) return KAMI_ERROR_MISALIGNED;
  if (batch > (int64_t)INT32_MAX) return KAMI_ERROR_NOT_SUPPORTED;
  RowProblem rp = to_row(m, n, k, layout, A, B, nullptr, nullptr);
  return dispatch(rp, batch, dtype, algo, p, C, nullptr, reinterpret_cast<cudaStream_t>(stream));
}

kami_status_t kami_gemm_strided_batched_axpby(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                              kami_layout_t layout, double alpha, const void* A, const void* B,
                                              double beta, void* C, kami_stream_t stream) {
  kami_status_t st = check_common(m, n, k, batch, dtype, layout, KAMI_ALGO_AUTO);
  if (st != KAMI_SUCCESS) return st;
  if (batch == 0) return KAMI_SUCCESS;
  if (!A || !B || !C) return KAMI_ERROR_INVALID_VALUE;
  if (!aligned16(A) || !aligned16(B) || !aligned16(C)) return KAMI_ERROR_MISALIGNED;
  if (batch > (int64_t)INT32_MAX) return KAMI_ERROR_NOT_SUPPORTED;
  // column-major: C^T = alpha B^T A^T + beta C^T on the same buffers
  RowProblem rp = to_row(m, n, k, layout, A, B, nullptr, nullptr);
  return dispatch(rp, batch, dtype, KAMI_ALGO_AUTO, 0, C, nullptr, reinterpret_cast<cudaStream_t>(stream), alpha,
                  beta);
}

kami_status_t kami_gemm_strided_batched(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                        kami_layout_t layout, const void* A, const void* B, void* C,
                                        kami_stream_t stream) {
  return kami_gemm_strided_batched_ex(m, n, k, batch, dtype, layout, A, B, C, KAMI_ALGO_AUTO, 0, stream);
}

kami_status_t kami_gemm(int m, int n, int k, int64_t batch, kami_dtype_t dtype, kami_layout_t layout,
                        const void* A, const void* B, void* C, kami_stream_t stream) {
  if (batch != 1) return KAMI_ERROR_INVALID_VALUE;
  return kami_gemm_strided_batched(m, n, k, 1, dtype, layout, A, B, C, stream);
}

kami_status_t kami_gemm_batched(int m, int n, int k, int64_t batch, kami_dtype_t dtype, kami_layout_t layout,
                                const void* const* A_array, const void* const* B_array, void* const* C_array,
                                kami_stream_t stream) {
  kami_status_t st = check_common(m, n, k, batch, dtype, layout, KAMI_ALGO_AUTO);
  if (st != KAMI_SUCCESS) return st;
  if (batch == 0) return KAMI_SUCCESS;
  if (!A_array || !B_array || !C_array) return KAMI_ERROR_INVALID_VALUE;
  if (!aligned16(A_array) || !aligned16(B_array) || !aligned16(C_array)) return KAMI_ERROR_MISALIGNED;
  if (batch > (int64_t)INT32_MAX) return KAMI_ERROR_NOT_SUPPORTED;
  RowProblem rp = to_row(m, n, k, layout, nullptr, nullptr, A_array, B_array);
  return dispatch(rp, batch, dtype, KAMI_ALGO_AUTO, 0, nullptr, C_array, reinterpret_cast<cudaStream_t>(stream));
}

kami_status_t kami_gemm_vbatched(int64_t batch, const int* m_array, const int* n_array, const int* k_array,
                                 int max_m, int max_n, int max_k, kami_dtype_t dtype, kami_layout_t layout,
                                 const void* const* A_array, const void* const* B_array, void* const* C_array,
                                 kami_stream_t stream) {
  kami_status_t st = check_common(max_m, max_n, max_k, batch, dtype, layout, KAMI_ALGO_AUTO);
  if (st != KAMI_SUCCESS) return st;
  if (!is16(dtype) && dtype != KAMI_DTYPE_F64) return KAMI_ERROR_NOT_SUPPORTED;
  if (batch == 0) return KAMI_SUCCESS;
  if (!m_array || !n_array || !k_array || !A_array || !B_array || !C_array) return KAMI_ERROR_INVALID_VALUE;
  if (!aligned16(A_array) || !aligned16(B_array) || !aligned16(C_array)) return KAMI_ERROR_MISALIGNED;
  if (batch > (int64_t)INT32_MAX) return KAMI_ERROR_NOT_SUPPORTED;
  // column-major: C^T = B^T A^T per entry -> swap m<->n and A<->B
  const bool col = layout == KAMI_COL_MAJOR;
  if (dtype == KAMI_DTYPE_F64)  // the k-sliced DMMA kernel with per-entry sizes
    return dmma_gen_vb_launch(batch, col ? n_array : m_array, col ? m_array : n_array, k_array, col ? max_n : max_m,
                              col ? max_m : max_n, max_k, col ? B_array : A_array, col ? A_array : B_array, C_array,
                              reinterpret_cast<cudaStream_t>(stream));
  return tc16_vb_launch(batch, dtype == KAMI_DTYPE_BF16, 0, 0, 0, col ? n_array : m_array, col ? m_array : n_array,
                        k_array, col ? max_n : max_m, col ? max_m : max_n, col ? B_array : A_array,
                        col ? A_array : B_array, C_array, reinterpret_cast<cudaStream_t>(stream));
}

kami_status_t kami_spmm_bsr_strided_batched(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                            const int* row_ptr, const int* col_blk, const void* vals,
                                            int max_nnzb, const void* B, void* C, kami_stream_t stream) {
  kami_status_t st = check_common(m, n, k, batch, dtype, KAMI_ROW_MAJOR, KAMI_ALGO_AUTO);
  if (st != KAMI_SUCCESS) return st;
  if (!is16(dtype) || k % 16) return KAMI_ERROR_NOT_SUPPORTED;
  if (max_nnzb < 0 || max_nnzb > (m / 16) * (k / 16)) return KAMI_ERROR_INVALID_VALUE;
  if (batch == 0) return KAMI_SUCCESS;
  if (!row_ptr || !col_blk || !vals || !B || !C || max_nnzb == 0) return KAMI_ERROR_INVALID_VALUE;
  if (!aligned16(vals) || !aligned16(B) || !aligned16(C)) return KAMI_ERROR_MISALIGNED;
  if (batch > (int64_t)INT32_MAX) return KAMI_ERROR_NOT_SUPPORTED;
  return tc16_spmm_bsr_launch(m, n, k, batch, dtype == KAMI_DTYPE_BF16, row_ptr, col_blk, vals, max_nnzb, B, C,
                              reinterpret_cast<cudaStream_t>(stream));
}

kami_status_t kami_spmm_zmorton_strided_batched_ex(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                                   const int* nnzb, const int* zcode, const void* vals,
                                                   int max_nnzb, const void* B, void* C, kami_algo_t algo,
                                                   kami_stream_t stream) {
  kami_status_t st = check_common(m, n, k, batch, dtype, KAMI_ROW_MAJOR, KAMI_ALGO_AUTO);
  if (st != KAMI_SUCCESS) return st;
  if (!is16(dtype) || k % 16 || m % 16) return KAMI_ERROR_NOT_SUPPORTED;
  if (max_nnzb < 0 || max_nnzb > (m / 16) * (k / 16)) return KAMI_ERROR_INVALID_VALUE;
  const bool two_d = algo == KAMI_ALGO_2D || algo == KAMI_ALGO_2D_PAIR;
  if (!(algo == KAMI_ALGO_AUTO || algo == KAMI_ALGO_1D || two_d)) return KAMI_ERROR_NOT_SUPPORTED;
  if (two_d && !tc16_pair_supported(m, n, k)) return KAMI_ERROR_NOT_SUPPORTED;
  if (batch == 0) return KAMI_SUCCESS;
  if (!nnzb || !zcode || !vals || !B || !C || max_nnzb == 0) return KAMI_ERROR_INVALID_VALUE;
  if (!aligned16(vals) || !aligned16(B) || !aligned16(C)) return KAMI_ERROR_MISALIGNED;
  if (batch > (int64_t)INT32_MAX) return KAMI_ERROR_NOT_SUPPORTED;
  // 2D: the schedule across a CTA pair, each CTA finding its block rows as
  // one contiguous Morton range (tc16_pair.cu).  AUTO / 1D: the 1D kernel,
  // which decodes each block's position from its code (tc16_vb.cu) -- on
  // B200 the faster of the two since its A blocks arrive by TMA
  if (two_d)
    return tc16_pair_launch(m, n, k, batch, dtype == KAMI_DTYPE_BF16, nullptr, B, C,
                            reinterpret_cast<cudaStream_t>(stream), nnzb, zcode, vals, max_nnzb);
  return tc16_spmm_bsr_launch(m, n, k, batch, dtype == KAMI_DTYPE_BF16, nnzb, zcode, vals, max_nnzb, B, C,
                              reinterpret_cast<cudaStream_t>(stream), /*zorder=*/true);
}

kami_status_t kami_spmm_zmorton_strided_batched(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                                const int* nnzb, const int* zcode, const void* vals, int max_nnzb,
                                                const void* B, void* C, kami_stream_t stream) {
  return kami_spmm_zmorton_strided_batched_ex(m, n, k, batch, dtype, nnzb, zcode, vals, max_nnzb, B, C,
                                              KAMI_ALGO_AUTO, stream);
}

kami_status_t kami_gemm_block_level(int m, int n, int k, int64_t batch, kami_dtype_t dtype, kami_layout_t layout,
                                    kami_algo_t algo, int p, int reps, const void* A, const void* B, void* C,
                                    int64_t* cycles, kami_stream_t stream) {
  kami_status_t st = check_common(m, n, k, batch, dtype, layout, algo);
  if (st != KAMI_SUCCESS) return st;
  if (p < 0 || reps < 1 || algo == KAMI_ALGO_1D_TMA || algo >= KAMI_ALGO_1D_TMEM) return KAMI_ERROR_INVALID_VALUE;
  if (batch == 0) return KAMI_SUCCESS;
  if (!A || !B || !C) return KAMI_ERROR_INVALID_VALUE;
  if (!aligned16(A) || !aligned16(B) || !aligned16(C)) return KAMI_ERROR_MISALIGNED;
  if (batch > (int64_t)INT32_MAX) return KAMI_ERROR_NOT_SUPPORTED;
  RowProblem rp = to_row(m, n, k, layout, A, B, nullptr, nullptr);
  const int a = algo == KAMI_ALGO_AUTO ? (int)KAMI_ALGO_1D : (int)algo;
  const int pp = p ? p : warp_ca_default_p(rp.m, rp.n, rp.k, dtype, a);
  if (pp == 0) return KAMI_ERROR_NOT_SUPPORTED;
  return warp_ca_launch(rp.m, rp.n, rp.k, batch, dtype, a, pp, rp.A, rp.B, C, nullptr, nullptr, nullptr,
                        reinterpret_cast<cudaStream_t>(stream), reps, reinterpret_cast<long long*>(cycles));
}

kami_status_t kami_plan(int m, int n, int k, kami_dtype_t dtype, kami_layout_t layout, kami_algo_t algo, int p,
                        kami_plan_t* out) {
  kami_status_t st = check_common(m, n, k, 1, dtype, layout, algo);
  if (st != KAMI_SUCCESS) return st;
  if (!out || p < 0) return KAMI_ERROR_INVALID_VALUE;
  RowProblem rp = to_row(m, n, k, layout, nullptr, nullptr, nullptr, nullptr);
  return planner_choose(rp.m, rp.n, rp.k, dtype, algo, p, false, out);
}

kami_status_t kami_plan_candidates(int m, int n, int k, kami_dtype_t dtype, kami_layout_t layout,
                                   kami_candidate_t* out, int max, int* count) {
  kami_status_t st = check_common(m, n, k, 1, dtype, layout, KAMI_ALGO_AUTO);
  if (st != KAMI_SUCCESS) return st;
  if (!count || max < 0 || (max > 0 && !out)) return KAMI_ERROR_INVALID_VALUE;
  RowProblem rp = to_row(m, n, k, layout, nullptr, nullptr, nullptr, nullptr);
  *count = planner_candidates(rp.m, rp.n, rp.k, dtype, false, out, max);
  return KAMI_SUCCESS;
}

kami_status_t kami_paper_cost(kami_algo_t variant, double m, double n, double k, double p, double s_e,
                              double L_sm, double B_sm, double theta_r, double theta_w, double O_tc, double n_tc,
                              double out[4]) {
  if (!out) return KAMI_ERROR_INVALID_VALUE;
  if (variant != KAMI_ALGO_1D && variant != KAMI_ALGO_2D && variant != KAMI_ALGO_3D)
    return KAMI_ERROR_INVALID_VALUE;
  if (m <= 0 || n <= 0 || k <= 0 || p <= 0 || s_e <= 0 || B_sm <= 0 || theta_r <= 0 || theta_w <= 0 ||
      O_tc <= 0 || n_tc <= 0)
    return KAMI_ERROR_INVALID_VALUE;
  PaperCost c = paper_cost((int)variant, m, n, k, p, s_e, L_sm, B_sm, theta_r, theta_w, O_tc, n_tc);
  out[0] = c.V_cm;
  out[1] = c.T_cm;
  out[2] = c.T_cp;
  out[3] = c.T_all;
  return KAMI_SUCCESS;
}

const char* kami_status_string(kami_status_t s) {
  switch (s) {
    case KAMI_SUCCESS: return "KAMI_SUCCESS";
    case KAMI_ERROR_INVALID_VALUE: return "KAMI_ERROR_INVALID_VALUE";
    case KAMI_ERROR_NOT_SUPPORTED: return "KAMI_ERROR_NOT_SUPPORTED";
    case KAMI_ERROR_MISALIGNED: return "KAMI_ERROR_MISALIGNED";
    case KAMI_ERROR_CUDA: return "KAMI_ERROR_CUDA";
  }
  return "KAMI_ERROR_UNKNOWN";
}

const char* kami_last_kernel(void) { return g_last_kernel; }
const char* kami_last_cuda_error(void) { return cudaGetErrorString((cudaError_t)g_last_cuda); }

int kami_version(void) { return (KAMI_VERSION_MAJOR << 16) | KAMI_VERSION_MINOR; }

kami_status_t kami_set_grid_cap(int max_ctas) {
  if (max_ctas < 0) return KAMI_ERROR_INVALID_VALUE;
  g_grid_cap.store(max_ctas, std::memory_order_relaxed);
  return KAMI_SUCCESS;
}

}  // extern "C"
