// kernels.h -- host-side interface between the C ABI (api.cpp) and the
// kernel families (tc16.cu: tcgen05 16-bit; warp_ca.cu: register-resident
// warp-level CA family with DMMA/HMMA).  Internal; not installed.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "../../include/kami.h"

namespace kami {

// cuTensorMapEncodeTiled fetched through the runtime (no link-time libcuda)
typedef CUresult (*PFN_encodeTiled)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                    const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                    CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
PFN_encodeTiled get_encode_tiled();
void set_last_kernel(const char* name);
// records e for kami_last_cuda_error(); returns KAMI_SUCCESS iff e == cudaSuccess
int launch_status(int cuda_error);
// kami_set_grid_cap (tests): every persistent launcher clamps its grid to this (0 = no cap)
int grid_cap();
inline long long apply_grid_cap(long long grid) {
  const int c = grid_cap();
  return (c > 0 && grid > c) ? c : grid;
}

// ---------------------------------------------------------------- tcgen05
struct Tc16Shape {
  int G, m_tiles, rows_tile, Wk, Wn, Wc, k_chunks, N_mma;
  int slot;    // A-tile rows / TMEM lanes per packed entry
  int colrep;  // thin m, G = 1: number of 32-lane slots the A box is replicated into (0 = off)
  int write_heavy;  // a unit writes at least as many bytes as it reads
  int tpack;        // 128 < m <= 192, n <= 128: two entries' tail rows share a tile (3 units per pair)
  int U;  // MMA sub-tiles per unit (G U entries per unit)
  uint32_t stage_bytes, c_buf_bytes;
  int c_bufs, stages, acc_cols, acc_bufs;
  uint32_t smem_bytes;
  long long units;
};
kami_status_t tc16_plan_shape(int m, int n, int k, Tc16Shape* s);
kami_status_t tc16_launch(int m, int n, int k, long long batch, bool bf16, const void* A, const void* B, void* C,
                          cudaStream_t stream, int max_ctas);
// in_kind: 0 f16, 1 bf16, 2 tf32, 3 e4m3, 4 e5m2; out_kind: 0 f16, 1 bf16, 2 f32.
// C = alpha A B + beta C (C is read iff beta != 0).
// no_tp: no tail packing (pointer arrays, the C-update form)
kami_status_t tc16_plan_shape_kind(int m, int n, int k, int in_kind, int out_kind, Tc16Shape* s, bool no_tp = false);
// Aa/Ba/Ca != nullptr: device pointer arrays (kami_gemm_batched; f16/bf16, C = AB only), A/B/C unused.
kami_status_t tc16_launch_kind(int m, int n, int k, long long batch, int in_kind, int out_kind, const void* A,
                               const void* B, void* C, float alpha, float beta, cudaStream_t stream, int max_ctas,
                               const void* const* Aa = nullptr, const void* const* Ba = nullptr,
                               void* const* Ca = nullptr);

// ------------------------------- tcgen05 with A resident in TMEM (tc16_ts.cu)
struct TsShape {
  int G, N_mma, Wk, Wn, Wc, k_chunks, ksteps_full, ksteps_last;
  int layers, item_cols, slot_cols, a_slots, loader_wgs, acc_cols;
  uint32_t stage_bytes, c_buf_bytes;
  int c_bufs, stages;
  uint32_t smem_bytes;
};
// layers: 1 = KAMI_ALGO_1D_TMEM, 2 = KAMI_ALGO_3D_TMEM
kami_status_t tc16_ts_plan(int m, int n, int k, int layers, TsShape* s);
kami_status_t tc16_ts_launch(int m, int n, int k, long long batch, bool bf16, int layers, const void* A,
                             const void* B, void* C, cudaStream_t stream);

// ------------- tcgen05 on the transposed product for thin m (tc16_xt.cu)
bool tc16_xt_supported(int m, int n, int k);
kami_status_t tc16_xt_plan(int m, int n, int k, int* E, int* stages);
kami_status_t tc16_xt_launch(int m, int n, int k, long long batch, bool bf16, const void* A, const void* B, void* C,
                             cudaStream_t stream);

// ------------------------ tcgen05 CTA pair, KAMI-2D over 2 SMs (tc16_pair.cu)
bool tc16_pair_supported(int m, int n, int k);
// zcode != nullptr: A in Z-Morton block storage (nnzb, zcode, vals as kami_spmm_zmorton_strided_batched)
kami_status_t tc16_pair_launch(int m, int n, int k, long long batch, bool bf16, const void* A, const void* B, void* C,
                               cudaStream_t stream, const int* nnzb = nullptr, const int* zcode = nullptr,
                               const void* vals = nullptr, int max_nnzb = 0);

// ------------------------------------------------ warp-level CA (literal KAMI)
// algo: 1 = 1D, 2 = 2D, 3 = 3D, 4 = non-CA tiled.  dtype: KAMI_DTYPE_*.
// Entry pointers: if A_arr != nullptr they are device arrays of per-entry
// pointers (kami_gemm_batched); else strided from A/B/C.
kami_status_t warp_ca_supported(int m, int n, int k, kami_dtype_t dtype, int algo, int p);
// reps > 1: block-level mode (operands loaded once, the CA schedule repeated
// reps times on chip, C = reps * A B stored once).  cycles != nullptr: per-entry
// [comm, compute] clock64 sums over the team's warps (int64 device array).
kami_status_t warp_ca_launch(int m, int n, int k, long long batch, kami_dtype_t dtype, int algo, int p,
                             const void* A, const void* B, void* C, const void* const* A_arr,
                             const void* const* B_arr, void* const* C_arr, cudaStream_t stream, int reps = 1,
                             long long* cycles = nullptr);

// ------------------------------------------- FP64 1D with TMA-fed broadcast
bool dmma_tma_supported(int m, int n, int k);
// Aa/Ba/Ca != nullptr: device pointer arrays (kami_gemm_batched, C = AB only), A/B/C unused.
kami_status_t dmma_tma_launch(int m, int n, int k, long long batch, const void* A, const void* B, void* C,
                              cudaStream_t stream, double alpha = 1.0, double beta = 0.0,
                              const void* const* Aa = nullptr, const void* const* Ba = nullptr,
                              void* const* Ca = nullptr);

// --------------- FP64, whole size grid, k-slicing + residency ratio (dmma_gen.cu)
bool dmma_gen_supported(int m, int n, int k);
int dmma_gen_resident_pct(int k);  // share of B_w's k-steps kept in registers (rest parked in SMEM)
// Aa/Ba/Ca != nullptr: device pointer arrays (kami_gemm_batched), A/B/C unused
kami_status_t dmma_gen_launch(int m, int n, int k, long long batch, const void* A, const void* B, void* C,
                              cudaStream_t stream, const void* const* Aa = nullptr, const void* const* Ba = nullptr,
                              void* const* Ca = nullptr);

// FP64 variable sizes: the pointer-array dmma_gen kernel with per-entry sizes (device arrays)
kami_status_t dmma_gen_vb_launch(long long batch, const int* dm, const int* dn, const int* dk, int max_m, int max_n,
                                 int max_k, const void* const* Aa, const void* const* Ba, void* const* Ca,
                                 cudaStream_t stream);

// ------------------------- 16-bit pointer-array / variable-size (tc16_vb.cu)
// dm/dn/dk: device arrays of per-entry sizes, or nullptr for uniform m, n, k.
kami_status_t tc16_vb_launch(long long batch, bool bf16, int m, int n, int k, const int* dm, const int* dn,
                             const int* dk, int max_m, int max_n, const void* const* A, const void* const* B,
                             void* const* C, cudaStream_t stream);

// strided batches with m or n = 8 mod 16 (16-bit): the same LDG-fed kernel on packed entries
kami_status_t tc16_vb_strided_launch(int m, int n, int k, long long batch, bool bf16, const void* A, const void* B,
                                     void* C, cudaStream_t stream);

// SpMM: block-sparse A (BSR, 16x16 blocks) x dense B on tcgen05 (densify on load)
// zorder: A in Z-Morton block storage (row_ptr = per-entry block counts, col_blk = Morton codes)
kami_status_t tc16_spmm_bsr_launch(int m, int n, int k, long long batch, bool bf16, const int* row_ptr,
                                   const int* col_blk, const void* vals, int max_nnzb, const void* B, void* C,
                                   cudaStream_t stream, bool zorder = false);

}  // namespace kami
