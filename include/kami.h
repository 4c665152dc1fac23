/*
 * kami.h -- C ABI of the B200-native KAMI batched small-GEMM library
 * (libkami.so, built from paper_conf_sc_wangdltsl25_b200/csrc).
 *
 * Operation (Sec. 2.1 "Matrix Multiplication"; batched form
 * L69 and Sec. 5.4): for every batch entry b,
 *
 *     C_b = A_b * B_b,   A_b m-by-k,  B_b k-by-n,  C_b m-by-n,
 *
 * computed with the thread-block-level communication-avoiding schedules of
 * KAMI (1D Alg. 1, 2D Alg. 2, 3D Alg. 3) re-designed for
 * sm_100a.  C is overwritten, never read (reading R1).
 * FP16 / BF16 inputs accumulate in FP32 and C is rounded to the input type
 * with round-to-nearest-even; FP64 is FP64 end to end (R2).
 *
 * Layout (R4; "aligned to cuBLAS/MAGMA"): one
 * flag for all three matrices, entries packed back to back, no leading
 * dimensions:
 *     KAMI_ROW_MAJOR: X_b(r, c) at  X + b*R*C + r*C + c
 *     KAMI_COL_MAJOR: X_b(r, c) at  X + b*R*C + c*R + r
 *
 * Sizes supported (R5): 16-bit and FP64 types: m, n, k multiples
 * of 8 in [8, 256] (the SURVEY.md 8(b) grid); TF32 m, n multiples of 16, k of
 * 4; FP8 m, n multiples of 32 and k of 16 (all <= 256).  Anything else
 * returns KAMI_ERROR_NOT_SUPPORTED.  Some entry points narrow this (the
 * update form, pointer arrays of FP64, SpMM): see each declaration.
 *
 * Ownership and threading: the caller owns every buffer.  Device entry points
 * never allocate device memory, never synchronise and enqueue on `stream`
 * (NULL = legacy default stream) of the current device.  They are
 * thread-safe.  C must not alias A or B; entries of C must not overlap.
 * All argument errors are detected before any launch; device faults surface
 * at the caller's next synchronisation (as in cuBLAS).
 */
#ifndef KAMI_H_
#define KAMI_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define KAMI_VERSION_MAJOR 0
#define KAMI_VERSION_MINOR 1

typedef enum {
  KAMI_SUCCESS = 0,
  KAMI_ERROR_INVALID_VALUE = 1, /* bad size/enum/pointer, batch < 0, ... */
  KAMI_ERROR_NOT_SUPPORTED = 2, /* outside the supported size grid        */
  KAMI_ERROR_MISALIGNED = 3,    /* base pointer not 16-byte aligned       */
  KAMI_ERROR_CUDA = 4           /* a CUDA runtime call failed             */
} kami_status_t;

/* Element types.  F16/BF16: A, B, C in that type, FP32 accumulation, C
 * rounded RNE.  F64: FP64 end to end.  TF32: A, B, C are FP32
 * arrays, the tensor core reads A and B at TF32 precision (10-bit fraction),
 * FP32 accumulation, C FP32.  E4M3 / E5M2 (f4): A, B are OCP FP8 bytes, FP32
 * accumulation, C FP16 (RNE). */
typedef enum {
  KAMI_DTYPE_F16 = 0,
  KAMI_DTYPE_BF16 = 1,
  KAMI_DTYPE_F64 = 2,
  KAMI_DTYPE_TF32 = 3,
  KAMI_DTYPE_E4M3 = 4,
  KAMI_DTYPE_E5M2 = 5
} kami_dtype_t;

typedef enum { KAMI_ROW_MAJOR = 0, KAMI_COL_MAJOR = 1 } kami_layout_t;

/* Which schedule runs (Sec. 4.3-4.5).  AUTO = the planner's choice
 * (kami_plan).  NONCA = the non-communication-avoiding tiled baseline.
 * 1D_TMA = KAMI-1D whose broadcast operand is written to shared memory by the
 * TMA engine (16-bit: the tcgen05 kernel; FP64: the DMMA kernel of
 * dmma_tma.cu, m = n = k in {32, 64}). */
typedef enum {
  KAMI_ALGO_AUTO = 0,
  KAMI_ALGO_1D = 1,
  KAMI_ALGO_2D = 2,
  KAMI_ALGO_3D = 3,
  KAMI_ALGO_NONCA = 4,
  KAMI_ALGO_1D_TMA = 5,
  /* 16-bit only, tcgen05 with the LOCAL operand resident in tensor memory
   * (Table 1: local storage never passes through shared
   * memory): A is loaded global -> registers -> TMEM, only B is broadcast
   * through shared memory.  m, n multiples of 16 in
   * [16, 128], k a multiple of 8 in [8, 256]; NOT_SUPPORTED otherwise. */
  KAMI_ALGO_1D_TMEM = 6,
  /* as 1D_TMEM with the k-chunks split into cbrt(p) = 2 k-layers (Alg. 3,
   * L338-380), each layer's A rows written by its own loader warpgroup, and
   * the layer partials summed inside ONE TMEM accumulator (the Alg. 3
   * reduction costs no shared-memory traffic).  Needs every k-chunk to hold
   * an even number of K = 16 steps (k a multiple of 32 in practice). */
  KAMI_ALGO_3D_TMEM = 7,
  /* 16-bit only, 192 < m <= 256: KAMI-2D across a CTA pair (tcgen05
   * cta_group::2, M = 256): CTA r owns rows [128r, 128r+128) of A and C and
   * columns [r n/2, (r+1) n/2) of B in its shared memory; the pair's MMA
   * broadcasts each B column block to the other CTA's rows (Alg. 2).
   * n a multiple of 32 in [32,256], k a multiple of 8; NOT_SUPPORTED
   * otherwise. */
  KAMI_ALGO_2D_PAIR = 8,
  /* 16-bit only, thin m (m in {16, 32}, n a multiple of 64 in [64, 256], k in
   * {16, 32, 64}): tcgen05 1D on the transposed product C^T = B^T A^T, n on
   * the 128 TMEM lanes and m on the columns, so E entries share one
   * accumulator side by side.  Strided C = A B; NOT_SUPPORTED
   * otherwise. */
  KAMI_ALGO_1D_XT = 9
} kami_algo_t;

/* Opaque CUDA stream; binary compatible with cudaStream_t. */
typedef struct CUstream_st* kami_stream_t;

/* Single GEMM (block-level interface).  `batch` must be 1. */
kami_status_t kami_gemm(int m, int n, int k, int64_t batch, kami_dtype_t dtype, kami_layout_t layout,
                        const void* A, const void* B, void* C, kami_stream_t stream);

/* Pointer-array batched GEMM (cuBLAS *gemmBatched convention): A_array,
 * B_array, C_array are DEVICE arrays of `batch` DEVICE pointers, each
 * 16-byte aligned, each pointing at one packed matrix in `layout`.  Same
 * operation, sizes, types and errors as kami_gemm_strided_batched (PAPER.md
 * L523: batched functions "aligned to" cuBLAS / MAGMA); entries may lie
 * anywhere in the device's address space, C entries must not overlap.  A
 * misaligned entry pointer cannot be detected before launch (the arrays are
 * device memory): its result is undefined.  16-bit types run on the same
 * tcgen05 kernel as the strided form, fed by TMA boxes over an address-space
 * view of each entry; m or n = 8 mod 16 on the LDG-fed
 * tcgen05 kernel.  FP64: m = n = k in {16, 32, 64} on the TMA-broadcast
 * DMMA kernel, 8^3 on the warp-level one, every other shape of the grid on
 * the k-sliced DMMA kernel with cp.async-fed A blocks. */
kami_status_t kami_gemm_batched(int m, int n, int k, int64_t batch, kami_dtype_t dtype, kami_layout_t layout,
                                const void* const* A_array, const void* const* B_array, void* const* C_array,
                                kami_stream_t stream);

/* Variable-size batched GEMM (MAGMA *_vbatched convention; "various matrix
 * orders in a batch"): entry b is m_array[b] x k_array[b]
 * times k_array[b] x n_array[b].  m_array, n_array, k_array are DEVICE int
 * arrays; A_array, B_array, C_array are DEVICE arrays of DEVICE pointers (each
 * 16-byte aligned, packed matrices in `layout`).  max_m/max_n/max_k are host
 * upper bounds used for planning and validated against the size grid; every
 * entry must itself be on the grid (16-bit: m, n multiples of 16 <= 256, k a
 * multiple of 8 <= 256; FP64: m, n, k multiples of 8 <= 256) and within the
 * max bounds -- entries off the grid are undefined behaviour for 16-bit and
 * skipped (C untouched) for FP64 (the sizes live on the device and are not
 * read by the host).  FP16 / BF16 run the class-sorted tcgen05 kernel, FP64
 * the k-sliced DMMA kernel with per-entry sizes; TF32 / FP8 return
 * KAMI_ERROR_NOT_SUPPORTED. */
kami_status_t kami_gemm_vbatched(int64_t batch, const int* m_array, const int* n_array, const int* k_array,
                                 int max_m, int max_n, int max_k, kami_dtype_t dtype, kami_layout_t layout,
                                 const void* const* A_array, const void* const* B_array, void* const* C_array,
                                 kami_stream_t stream);

/* Strided-batched GEMM: entry b of A at A + b*m*k elements, of B at
 * B + b*k*n, of C at C + b*m*n.  The hot path of BASELINE.json. */
kami_status_t kami_gemm_strided_batched(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                        kami_layout_t layout, const void* A, const void* B, void* C,
                                        kami_stream_t stream);

/* C <- alpha * A B + beta * C (the C-update form of Alg. 1-3, whose
 * GMem2Reg loads C).  C is read iff beta != 0.  alpha and beta are
 * applied in FP32 for the tensor-core types (FP64 for F64).  Strided batches,
 * planner-chosen kernel; NOT_SUPPORTED where that kernel has no update form
 * (FP64 order 8). */
kami_status_t kami_gemm_strided_batched_axpby(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                              kami_layout_t layout, double alpha, const void* A, const void* B,
                                              double beta, void* C, kami_stream_t stream);

/* Same with an explicit schedule and warp count p.  p = 0 takes the planner
 * default; for 16-bit KAMI_ALGO_1D with p = 0 that is the tcgen05 kernel
 * (whose compute units are the 4 sub-partition tensor cores of an SM), while
 * p > 0 selects the register-resident warp-level kernel with p warps per
 * entry.  Bench/test surface: lets the 1D/2D/3D/non-CA variants be compared. */
kami_status_t kami_gemm_strided_batched_ex(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                           kami_layout_t layout, const void* A, const void* B, void* C,
                                           kami_algo_t algo, int p, kami_stream_t stream);

/* Host-memory entry point (end-to-end): A, B, C are HOST pointers (pinned
 * memory recommended).  The library streams the batch through device
 * workspace in chunks, overlapping host->device copies, the kernel and
 * device->host copies on internal streams, and returns after C is complete
 * on the host (synchronous).  Workspace is allocated on first use per device
 * and kept until kami_release_workspace(). */
kami_status_t kami_gemm_strided_batched_host(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                             kami_layout_t layout, const void* A, const void* B, void* C);
kami_status_t kami_release_workspace(void);

/* SpMM: C_b = A_b * B_b with block-sparse A_b (Sec. 4.6):
 * A is stored as 16 x 16 dense blocks in block-row order (the 1D storage of
 * Fig. 7(a), i.e. BSR): for entry b, block row i owns blocks
 * row_ptr[b*(m/16+1) + i] .. row_ptr[b*(m/16+1) + i + 1] - 1 (indices local to
 * the entry), block j has block column col_blk[b*max_nnzb + j] and values
 * vals[(b*max_nnzb + j)*256 + r*16 + c] (row-major block).  B (k x n) and C
 * (m x n) are dense, row-major, packed strided batches.  All arrays are
 * DEVICE memory.  m, n, k multiples of 16 in [16, 256]; 16-bit types only.
 * Absent blocks are zero; the kernel densifies A on load (HBM traffic is the
 * nonzero blocks only) and runs the dense tcgen05 1D schedule. */
kami_status_t kami_spmm_bsr_strided_batched(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                            const int* row_ptr, const int* col_blk, const void* vals,
                                            int max_nnzb, const void* B, void* C, kami_stream_t stream);

/* SpMM with A in multi-level Z-Morton block storage (Sec. 4.6,
 * Fig. 7(b): the storage of the 2D / 3D algorithms, "to facilitate efficient
 * submatrix indexing").  Entry b holds nnzb[b] dense 16 x 16 blocks; the j-th
 * (j < nnzb[b]) is block (i, c) of A with Morton code
 *     zcode[b*max_nnzb + j] = sum_t c_t 4^t + i_t 2 * 4^t
 * (column bits in the even positions, row bits in the odd ones: the Z curve
 * visits TL, TR, BL, BR at every level, so every aligned 2^L x 2^L submatrix
 * is one contiguous code range), codes ascending, values at
 * vals[(b*max_nnzb + j)*256 + r*16 + c'] (row-major block).  B, C dense
 * row-major packed strided batches.  All arrays DEVICE memory.  Same sizes,
 * types and errors as kami_spmm_bsr_strided_batched.  m > 128 (n a multiple
 * of 32): the 2D schedule across a CTA pair, CTA r taking block rows
 * [8r, 8r+8) = the Morton codes [128r, 128r+128), one contiguous range of the
 * sorted codes; otherwise the 1D kernel, which decodes each block's position
 * from its code.  (This entry point is the _ex form with KAMI_ALGO_AUTO.) */
kami_status_t kami_spmm_zmorton_strided_batched(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                                const int* nnzb, const int* zcode, const void* vals, int max_nnzb,
                                                const void* B, void* C, kami_stream_t stream);

/* Same with an explicit schedule: KAMI_ALGO_1D runs the 1D kernel (every
 * CTA decodes its tile's block positions from the codes); KAMI_ALGO_2D /
 * KAMI_ALGO_2D_PAIR the 2D schedule across a CTA pair (m > 128, n a multiple
 * of 32; NOT_SUPPORTED otherwise), each CTA taking the contiguous Morton
 * range of its block rows (Sec. 4.6).  KAMI_ALGO_AUTO = the faster
 * on B200, the 1D kernel (256^3 at 50 % blocks 0.75 vs 0.48
 * of the roofline).  Other algos: NOT_SUPPORTED. */
kami_status_t kami_spmm_zmorton_strided_batched_ex(int m, int n, int k, int64_t batch, kami_dtype_t dtype,
                                                   const int* nnzb, const int* zcode, const void* vals,
                                                   int max_nnzb, const void* B, void* C, kami_algo_t algo,
                                                   kami_stream_t stream);

/* Block-level (on-chip-resident) mode -- the paper's block-level experiment
 * (Sec. 5.1, Sec. 5.2, Fig. 8/9): every entry is owned by one
 * team of p warps that loads A_b and B_b once and runs the CA schedule `reps`
 * times on chip, accumulating C_b = reps * A_b B_b, stored once; all entries
 * are launched at once (no persistent loop, no L2 prefetch).  It measures the
 * schedule without global I/O.  `cycles` (optional, may be NULL) is a DEVICE
 * int64 array of 2*batch that receives, per entry, the clock64 cycles spent
 * in communication (SMEM exchange + barrier) and in computation (MMA issue),
 * summed over the team's warps (Sec. 5.6.2, Fig. 15); it must be zeroed by
 * the caller.  Register-resident warp-level kernels only: algo 1D/2D/3D/NONCA
 * (AUTO = 1D) with p = 0 for the default warp count.  reps >= 1. */
kami_status_t kami_gemm_block_level(int m, int n, int k, int64_t batch, kami_dtype_t dtype, kami_layout_t layout,
                                    kami_algo_t algo, int p, int reps, const void* A, const void* B, void* C,
                                    int64_t* cycles, kami_stream_t stream);

/* Planner decision (cost model PAPER.md Eqs. 4/8/12). */
typedef struct {
  kami_algo_t algo;      /* chosen schedule                                 */
  int p;                 /* warps (or tensor-core sub-partitions) per entry */
  int kernel;            /* 0 = tcgen05 16-bit (SS), 1 = warp-level DMMA/HMMA, 2 = FP64 DMMA with TMA
                            broadcast, 3 = tcgen05 16-bit with A resident in TMEM (TS), 4 = FP64 DMMA
                            for the whole size grid (k-sliced, register residency ratio), 5 = LDG-fed
                            tcgen05 16-bit (m or n = 8 mod 16), 6 = tcgen05 CTA pair (2D, cta_group::2),
                            7 = tcgen05 16-bit on the transposed product (thin m, XT) */
  int entries_per_cta;   /* batch entries a CTA keeps in flight             */
  int stages;            /* shared-memory pipeline depth                    */
  int kslice_regs_pct;   /* share of A/B kept resident (Sec. 4.7)           */
  double t_all_cycles;   /* model cycles per entry of the chosen schedule   */
} kami_plan_t;

kami_status_t kami_plan(int m, int n, int k, kami_dtype_t dtype, kami_layout_t layout, kami_algo_t algo, int p,
                        kami_plan_t* out);

/* What bounds a candidate in the planner's B200 cycle model. */
typedef enum {
  KAMI_BOUND_HBM = 0,      /* algorithmic bytes / HBM bandwidth                       */
  KAMI_BOUND_TENSOR = 1,   /* flops / tensor-pipe rate (tcgen05, HMMA or DMMA)        */
  KAMI_BOUND_SMEM = 2,     /* shared-memory bytes / SMEM bandwidth                    */
  KAMI_BOUND_TMA = 3,      /* TMA box rows x per-row engine time                      */
  KAMI_BOUND_ISSUE = 4,    /* per-unit fixed cost of the persistent pipeline          */
  KAMI_BOUND_LATENCY = 5   /* a team's serial chain (DRAM latency + Eqs. 4/8/12 with
                              B200 constants + barriers) over the teams per SM       */
} kami_bound_t;

/* One schedule the library can run for a shape, with the model's prediction
 * (Eqs. 4/8/12 with B200 constants for the
 * register-resident schedules, a streaming roofline for the tcgen05 ones). */
typedef struct {
  kami_algo_t algo;
  int p;
  int kernel;                    /* as kami_plan_t.kernel                     */
  double model_cycles_per_entry; /* per SM, at 1965 MHz                       */
  double model_tflops;           /* whole GPU (148 SMs)                       */
  int bound;                     /* kami_bound_t of the largest term          */
} kami_candidate_t;

/* Every candidate schedule for a strided problem (row-major view after the
 * layout transform) with the model's prediction; AUTO takes the fastest.
 * Writes min(*count, max) entries to `out` (may be NULL with max = 0) and the
 * total number to *count.  Host-only (no device work); errors as kami_plan. */
kami_status_t kami_plan_candidates(int m, int n, int k, kami_dtype_t dtype, kami_layout_t layout,
                                   kami_candidate_t* out, int max, int* count);

/* Paper-faithful cost model (Eqs. 1-12, readings R6-R8): fills
 * V_cm, T_cm, T_cp, T_all for variant 1/2/3 (KAMI_ALGO_1D/2D/3D). */
kami_status_t kami_paper_cost(kami_algo_t variant, double m, double n, double k, double p, double s_e,
                              double L_sm, double B_sm, double theta_r, double theta_w, double O_tc,
                              double n_tc, double out[4]);

const char* kami_status_string(kami_status_t status);

/* Name of the last kernel this thread launched ("" if none). */
const char* kami_last_kernel(void);

/* Diagnostic: the CUDA runtime's message for the last launch error a call
 * reported as KAMI_ERROR_CUDA on this thread ("no error" if none). */
const char* kami_last_cuda_error(void);

int kami_version(void); /* (MAJOR << 16) | MINOR */

/* Diagnostic: the FP64 DMMA roofline denominator measured on this device.
 * Runs an mma.sync.m8n8k4.f64 loop (the FP64 hot path's instruction) on
 * 4 CTAs per SM, launch after launch on `stream`, for at least min_ms
 * (0 <= min_ms <= 60000) and synchronizes.  *burst = the fastest launch
 * (TFLOP/s, a kernel timed alone), *sustained = the median launch of the
 * second half of the run (clock under the power cap).  Allocates and frees
 * 64 bytes of device memory.  KAMI_ERROR_INVALID_VALUE for null outputs or
 * min_ms out of range; KAMI_ERROR_CUDA if a launch fails. */
kami_status_t kami_probe_dmma_peak(double min_ms, double* burst, double* sustained, kami_stream_t stream);

/* Test / diagnostic knob: cap the number of CTAs of every persistent kernel
 * launched afterwards by this process (0 = no cap, the default).  With a cap
 * of c, each CTA of a batch of u work units runs ceil(u / c) of them, so the
 * parity tests exercise the pipelines' steady state (ring wrap-around,
 * mbarrier phase flips, TMEM accumulator and C staging reuse) at small batch
 * sizes.  Results do not depend on the cap; only the speed does.  Not
 * thread-safe with respect to concurrent launches on other threads.
 * Returns KAMI_ERROR_INVALID_VALUE for max_ctas < 0.  No device work. */
kami_status_t kami_set_grid_cap(int max_ctas);

#ifdef __cplusplus
}
#endif

#endif /* KAMI_H_ */
