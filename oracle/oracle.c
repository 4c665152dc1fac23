/*
 * oracle.c -- KAMI batched small-GEMM reference oracle.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_sc_wangdltsl25_b200/, include/kami.h) never
 * links, imports or executes anything under oracle/, and this file includes
 * nothing from the product tree.
 *
 * What it computes (plain definitions, written out, no blocking/fusion):
 *
 *   GEMM (Sec. 2.1): C = A * B with A m-by-k, B k-by-n,
 *   C m-by-n.  Batched GEMM (Sec. 2.1, Fig. 1(e)) applies it to
 *   every entry b of a batch independently.  KAMI's 1D/2D/3D algorithms
 *   (Alg. 1-3) only reorder data movement between warps,
 *   so the exact result they approximate in floating point is
 *
 *       C_ref[b,i,j] = sum_{l=0}^{k-1} double(A[b,i,l]) * double(B[b,l,j])
 *
 *   accumulated in IEEE binary64 with l ascending.  Inputs are the already
 *   dtype-rounded fp16 / bf16 / fp64 values, decoded exactly to double.
 *
 *   Layout (reading R4; "aligned to cuBLAS"): one
 *   flag for all three matrices, packed, no leading dimensions.
 *     row-major: X[b, r, c] at b*R*C + r*C + c
 *     col-major: X[b, r, c] at b*R*C + c*R + r
 *
 *   Error scale (BASELINE.json north_star): S[b,i,j] = sum_l |A[b,i,l]| |B[b,l,j]|.
 *
 *   Round-to-nearest-even converters double -> fp16 / bf16 (used to form the
 *   bit-exact expectation for integer-valued inputs, reading R2),
 *   written with integer/bit manipulation and C99 rint() under the default
 *   FE_TONEAREST mode.  No CUDA header is used.
 *
 * Pins: tests/test_oracle.py (hand cases, identity/permutation, closed forms,
 * transpose identity, integer exactness, cross-check vs torch.matmul float64,
 * RNE converter cases vs the IEEE 754 definition).
 */
#include <fenv.h>
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_F16 0
#define ORACLE_BF16 1
#define ORACLE_F64 2
#define ORACLE_F32 3  /* IEEE binary32 storage (TF32 inputs are FP32 values with a 10-bit mantissa) */
#define ORACLE_E4M3 4 /* OCP FP8 E4M3 ("fn": no infinities, 0x7f/0xff NaN) */
#define ORACLE_E5M2 5 /* OCP FP8 E5M2 (IEEE-like) */

#define ORACLE_ROW 0
#define ORACLE_COL 1

/* ---------------------------------------------------------------- decoders */

/* IEEE 754 binary16: 1 sign, 5 exponent (bias 15), 10 fraction bits. */
double oracle_f16_to_f64(uint16_t h) {
  int s = (h >> 15) & 1;
  int e = (h >> 10) & 0x1f;
  int f = h & 0x3ff;
  double v;
  if (e == 0) {
    v = ldexp((double)f, -24); /* subnormal: f * 2^-24 */
  } else if (e == 31) {
    v = f ? NAN : INFINITY;
  } else {
    v = ldexp((double)(1024 + f), e - 25); /* (1.f) * 2^(e-15) */
  }
  return s ? -v : v;
}

/* bfloat16: the upper 16 bits of an IEEE binary32. */
double oracle_bf16_to_f64(uint16_t h) {
  uint32_t u = ((uint32_t)h) << 16;
  float f;
  memcpy(&f, &u, sizeof f);
  return (double)f;
}

/* FP8 E4M3 (bias 7, 3 fraction bits, max 448, S.1111.111 = NaN). */
double oracle_e4m3_to_f64(uint8_t h) {
  int s = (h >> 7) & 1, e = (h >> 3) & 0xf, f = h & 7;
  double v;
  if (e == 15 && f == 7) v = NAN;
  else if (e == 0) v = ldexp((double)f, -9); /* f * 2^-3 * 2^-6 */
  else v = ldexp((double)(8 + f), e - 10);   /* (1.f) * 2^(e-7) */
  return s ? -v : v;
}

/* FP8 E5M2 (bias 15, 2 fraction bits, IEEE specials). */
double oracle_e5m2_to_f64(uint8_t h) {
  int s = (h >> 7) & 1, e = (h >> 2) & 0x1f, f = h & 3;
  double v;
  if (e == 31) v = f ? NAN : INFINITY;
  else if (e == 0) v = ldexp((double)f, -16); /* f * 2^-2 * 2^-14 */
  else v = ldexp((double)(4 + f), e - 17);    /* (1.f) * 2^(e-15) */
  return s ? -v : v;
}

/* ------------------------------------------------------ RNE encoders (f64) */

/* Generic: round |a| (finite, > 0) to a binary format with `mbits` fraction
 * bits, exponent bias `bias`, max biased exponent `emax_biased` (all-ones
 * reserved).  Returns the magnitude bits. */
static uint32_t rne_encode_mag(double a, int mbits, int bias, int emax_biased) {
  int fe = 0;
  double fr = frexp(a, &fe);       /* a = fr * 2^fe, fr in [0.5, 1) */
  int E = fe - 1;                   /* a = (2 fr) * 2^E, 2fr in [1,2) */
  int emin = 1 - bias;              /* smallest normal exponent */
  uint32_t one = 1u << mbits;
  if (E < emin) {
    /* subnormal range: value = q * 2^(emin - mbits), q integer after RNE */
    double q = rint(ldexp(a, mbits - emin));
    /* q == one naturally encodes the smallest normal */
    return (uint32_t)q;
  }
  double q = rint(ldexp(a, mbits - E)); /* in [one, 2*one] */
  if (q >= (double)(2 * one)) {
    q = (double)one;
    E += 1;
  }
  int eb = E + bias;
  if (eb >= emax_biased) return ((uint32_t)emax_biased) << mbits; /* inf */
  return (((uint32_t)eb) << mbits) | ((uint32_t)q - one);
}

uint16_t oracle_f64_to_f16_rne(double x) {
  if (isnan(x)) return 0x7e00;
  uint16_t s = signbit(x) ? 0x8000 : 0;
  double a = fabs(x);
  if (a == 0.0) return s;
  if (isinf(a)) return s | 0x7c00;
  return s | (uint16_t)rne_encode_mag(a, 10, 15, 31);
}

uint16_t oracle_f64_to_bf16_rne(double x) {
  if (isnan(x)) return 0x7fc0;
  uint16_t s = signbit(x) ? 0x8000 : 0;
  double a = fabs(x);
  if (a == 0.0) return s;
  if (isinf(a)) return s | 0x7f80;
  return s | (uint16_t)rne_encode_mag(a, 7, 127, 255);
}

/* ------------------------------------------------------------ element read */

static double load_elem(const void* base, int dtype, int64_t idx) {
  switch (dtype) {
    case ORACLE_F16:
      return oracle_f16_to_f64(((const uint16_t*)base)[idx]);
    case ORACLE_BF16:
      return oracle_bf16_to_f64(((const uint16_t*)base)[idx]);
    case ORACLE_F32:
      return (double)((const float*)base)[idx];
    case ORACLE_E4M3:
      return oracle_e4m3_to_f64(((const uint8_t*)base)[idx]);
    case ORACLE_E5M2:
      return oracle_e5m2_to_f64(((const uint8_t*)base)[idx]);
    default:
      return ((const double*)base)[idx];
  }
}

/* index of X[b, r, c] for an R-by-C matrix (layout applies to all operands) */
static int64_t at(int layout, int64_t b, int64_t r, int64_t c, int64_t R, int64_t C) {
  return layout == ORACLE_ROW ? b * R * C + r * C + c : b * R * C + c * R + r;
}

/* ------------------------------------------------------------ GEMM oracle */

typedef struct {
  int m, n, k, dtype, layout;
  int64_t b0, b1;
  const void *A, *B;
  double *C, *S; /* C/S are row-major [batch][m][n] regardless of layout */
} job_t;

static void* gemm_worker(void* arg) {
  job_t* j = (job_t*)arg;
  const int64_t m = j->m, n = j->n, k = j->k;
  for (int64_t b = j->b0; b < j->b1; ++b) {
    for (int64_t i = 0; i < m; ++i) {
      for (int64_t jj = 0; jj < n; ++jj) {
        double acc = 0.0, sabs = 0.0;
        for (int64_t l = 0; l < k; ++l) { /* l ascending (R3) */
          double a = load_elem(j->A, j->dtype, at(j->layout, b, i, l, m, k));
          double bb = load_elem(j->B, j->dtype, at(j->layout, b, l, jj, k, n));
          acc += a * bb;
          sabs += fabs(a) * fabs(bb);
        }
        j->C[b * m * n + i * n + jj] = acc;
        if (j->S) j->S[b * m * n + i * n + jj] = sabs;
      }
    }
  }
  return NULL;
}

/*
 * oracle_gemm: C_ref (and optionally S) for every entry, threads over entries.
 * C and S are written row-major [batch][m][n] (a host-side convention of the
 * oracle, independent of the input layout).  Returns 0 on success.
 */
int oracle_gemm(int m, int n, int k, int64_t batch, int dtype, int layout,
                const void* A, const void* B, double* C, double* S, int nthreads) {
  if (m <= 0 || n <= 0 || k <= 0 || batch < 0) return 1;
  if (dtype < 0 || dtype > 5 || layout < 0 || layout > 1) return 1;
  if (batch == 0) return 0;
  if (fegetround() != FE_TONEAREST) fesetround(FE_TONEAREST);
  if (nthreads < 1) nthreads = 1;
  if (nthreads > batch) nthreads = (int)batch;
  pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * nthreads);
  job_t* jobs = (job_t*)malloc(sizeof(job_t) * nthreads);
  for (int t = 0; t < nthreads; ++t) {
    jobs[t].m = m; jobs[t].n = n; jobs[t].k = k;
    jobs[t].dtype = dtype; jobs[t].layout = layout;
    jobs[t].b0 = batch * t / nthreads;
    jobs[t].b1 = batch * (t + 1) / nthreads;
    jobs[t].A = A; jobs[t].B = B; jobs[t].C = C; jobs[t].S = S;
  }
  if (nthreads == 1) {
    gemm_worker(&jobs[0]);
  } else {
    for (int t = 0; t < nthreads; ++t) pthread_create(&th[t], NULL, gemm_worker, &jobs[t]);
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
  }
  free(th);
  free(jobs);
  return 0;
}

/* Round an array of doubles to fp16 / bf16 bits with RNE (expectation for the
 * bit-exact integer-valued parity cases). */
void oracle_round_f16(const double* x, uint16_t* out, int64_t n) {
  for (int64_t i = 0; i < n; ++i) out[i] = oracle_f64_to_f16_rne(x[i]);
}
void oracle_round_bf16(const double* x, uint16_t* out, int64_t n) {
  for (int64_t i = 0; i < n; ++i) out[i] = oracle_f64_to_bf16_rne(x[i]);
}
void oracle_decode_f16(const uint16_t* x, double* out, int64_t n) {
  for (int64_t i = 0; i < n; ++i) out[i] = oracle_f16_to_f64(x[i]);
}
void oracle_decode_bf16(const uint16_t* x, double* out, int64_t n) {
  for (int64_t i = 0; i < n; ++i) out[i] = oracle_bf16_to_f64(x[i]);
}

/* ---------------------------------------------------------- SpMM oracle
 * PAPER.md Sec. 4.6 (L407-418): SpMM multiplies a sparse A, stored as dense
 * blk x blk blocks in block-row order (Fig. 7(a), the 1D storage: row_ptr /
 * col_blk / vals), by a dense B into a dense C.  The plain definition: expand
 * A to its dense m x k matrix (absent blocks are zero) and run the GEMM
 * definition above.  Per entry b: row_ptr[b*(m/blk+1) + i] .. row_ptr[...+i+1]
 * index the blocks of block row i in col_blk[b*max_nnzb + j] and
 * vals[(b*max_nnzb + j)*blk*blk + r*blk + c].  B and C row-major. */
int oracle_spmm_bsr(int m, int n, int k, int blk, int64_t batch, int dtype, const int* row_ptr,
                    const int* col_blk, const void* vals, int max_nnzb, const void* B, double* C, double* S,
                    int nthreads) {
  if (m <= 0 || n <= 0 || k <= 0 || blk <= 0 || batch < 0 || m % blk || k % blk) return 1;
  const int mb = m / blk;
  double* Ad = (double*)malloc(sizeof(double) * (size_t)m * k);
  double* Bd = (double*)malloc(sizeof(double) * (size_t)k * n);
  if (!Ad || !Bd) return 2;
  int rc = 0;
  for (int64_t b = 0; b < batch && rc == 0; ++b) {
    memset(Ad, 0, sizeof(double) * (size_t)m * k);
    const int* rp = row_ptr + b * (mb + 1);
    for (int i = 0; i < mb; ++i) {
      for (int j = rp[i]; j < rp[i + 1]; ++j) {
        const int bc = col_blk[b * max_nnzb + j];
        if (bc < 0 || (bc + 1) * blk > k) { rc = 3; break; }
        for (int r = 0; r < blk; ++r)
          for (int c = 0; c < blk; ++c)
            Ad[(size_t)(i * blk + r) * k + bc * blk + c] =
                load_elem(vals, dtype, (b * max_nnzb + j) * (int64_t)blk * blk + r * blk + c);
      }
    }
    for (int64_t t = 0; t < (int64_t)k * n; ++t) Bd[t] = load_elem(B, dtype, b * (int64_t)k * n + t);
    rc = rc ? rc : oracle_gemm(m, n, k, 1, ORACLE_F64, ORACLE_ROW, Ad, Bd, C + b * (int64_t)m * n,
                               S ? S + b * (int64_t)m * n : NULL, 1);
  }
  (void)nthreads;
  free(Ad);
  free(Bd);
  return rc;
}

/* ---------------------------------------- multi-level Z-Morton block order
 * PAPER.md Sec. 4.6 L409 (Fig. 7(b)): for the 2D / 3D algorithms the dense
 * 16 x 16 blocks of a sparse matrix are stored in a multi-level Z-Morton
 * order.  Reading (R31): the Z curve visits, at every level, the
 * top-left, top-right, bottom-left, bottom-right quadrant, i.e. the code of
 * block (block row i, block column j) interleaves the bits of j (even bit
 * positions) and i (odd positions):  z = sum_t j_t 2^(2t) + i_t 2^(2t+1).
 * Every aligned 2^L x 2^L submatrix is then one contiguous code range, at
 * every level L -- the "efficient submatrix indexing".  Written bit by bit. */
int oracle_morton_encode(int i, int j) {
  int z = 0;
  for (int t = 0; t < 15; ++t) {
    z |= ((j >> t) & 1) << (2 * t);
    z |= ((i >> t) & 1) << (2 * t + 1);
  }
  return z;
}
void oracle_morton_decode(int z, int* i, int* j) {
  int a = 0, b = 0;
  for (int t = 0; t < 15; ++t) {
    b |= ((z >> (2 * t)) & 1) << t;
    a |= ((z >> (2 * t + 1)) & 1) << t;
  }
  *i = a;
  *j = b;
}

/* SpMM with A in Z-Morton block storage: entry b holds nnzb[b] blocks, the
 * j-th with Morton code zcode[b * max_nnzb + j] and values
 * vals[(b * max_nnzb + j) * blk * blk ...] (row-major block).  A is densified
 * (absent blocks are zero), then the plain GEMM definition. */
int oracle_spmm_zmorton(int m, int n, int k, int blk, int64_t batch, int dtype, const int* nnzb, const int* zcode,
                        const void* vals, int max_nnzb, const void* B, double* C, double* S) {
  if (m <= 0 || n <= 0 || k <= 0 || blk <= 0 || batch < 0 || m % blk || k % blk) return 1;
  double* Ad = (double*)malloc(sizeof(double) * (size_t)m * k);
  double* Bd = (double*)malloc(sizeof(double) * (size_t)k * n);
  if (!Ad || !Bd) return 2;
  int rc = 0;
  for (int64_t b = 0; b < batch && rc == 0; ++b) {
    memset(Ad, 0, sizeof(double) * (size_t)m * k);
    if (nnzb[b] < 0 || nnzb[b] > max_nnzb) { rc = 3; break; }
    for (int j = 0; j < nnzb[b]; ++j) {
      int bi, bj;
      oracle_morton_decode(zcode[b * max_nnzb + j], &bi, &bj);
      if ((bi + 1) * blk > m || (bj + 1) * blk > k) { rc = 3; break; }
      for (int r = 0; r < blk; ++r)
        for (int c = 0; c < blk; ++c)
          Ad[(size_t)(bi * blk + r) * k + bj * blk + c] =
              load_elem(vals, dtype, (b * max_nnzb + j) * (int64_t)blk * blk + r * blk + c);
    }
    for (int64_t t = 0; t < (int64_t)k * n; ++t) Bd[t] = load_elem(B, dtype, b * (int64_t)k * n + t);
    rc = rc ? rc : oracle_gemm(m, n, k, 1, ORACLE_F64, ORACLE_ROW, Ad, Bd, C + b * (int64_t)m * n,
                               S ? S + b * (int64_t)m * n : NULL, 1);
  }
  free(Ad);
  free(Bd);
  return rc;
}

/* ------------------------------------------------- alpha A B + beta C_in
 * The GEMM-update form the algorithms' GMem2Reg(C_i <- C) implies (Alg. 1-3
 * load C, R1/f4):  C_ref = alpha * (A B)_ref + beta * C_in, both
 * terms in binary64; C_in given as doubles (already decoded, row-major
 * [batch][m][n]).  Writes the result in place over C (which holds (A B)_ref). */
void oracle_axpby(double* C, const double* Cin, double alpha, double beta, int64_t count) {
  for (int64_t i = 0; i < count; ++i) C[i] = alpha * C[i] + beta * Cin[i];
}
void oracle_decode_fp8(const uint8_t* x, double* out, int64_t n, int e5m2) {
  for (int64_t i = 0; i < n; ++i) out[i] = e5m2 ? oracle_e5m2_to_f64(x[i]) : oracle_e4m3_to_f64(x[i]);
}
