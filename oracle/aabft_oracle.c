/*
 * aabft_oracle.c -- plain, slow, obviously-correct CPU oracle for the A-ABFT hot path
 * (Braun, Halder, Wunderlich, "A-ABFT: Autonomous Algorithm-Based Fault Tolerance for
 * Matrix Multiplications on GPUs", DSN'14).  P:Lnn = line nn of /root/reference/PAPER.md.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load or call this library.  It shares no
 * code, header, table or constant generator with the CUDA path
 * (paper_conf_dsn_braunhw14_b200/csrc); neither side includes the other.
 *
 * Build: gcc -O2 -std=c11 -ffp-contract=off -fno-fast-math -pthread -shared -fPIC
 *        (no FMA contraction; FMA only where fma_model = 1 asks for it, via fma()/fmaf()).
 *
 * Everything is row-major.  dtype 0 = double (FP64), 1 = float (FP32).  Working precision
 * w is the dtype; bounds, reference sums and differences are always double (R12).
 * Readings of the paper where it is silent/garbled are DESIGN.md R1..R22 (= SURVEY G1..G22).
 *
 * Pins (tests/test_oracle_*.py): closed forms of Eq 28 / P:L287, integer-exact checksum
 * identities (Eq 5), brute-force top-p and y invariants (§IV-E), the Table II/III
 * "AVG. A-ABFT" and "AVG. Rnd. Error" columns, brute-force single-fault
 * locate/correct on tiny integer inputs; the NEXT-3 comparators (external-eps check/correct,
 * SEA-ABFT bound O11) and the Alg 3 product site (site 4) in tests/test_oracle_comparators.py,
 * the SEA bound against Table II/III "AVG. SEA-ABFT".  No function here is
 * "parity unpinned".
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OR_F64 0
#define OR_F32 1

static double ld(int dtype, const void *p, int64_t idx) {
  return dtype == OR_F64 ? ((const double *)p)[idx] : (double)((const float *)p)[idx];
}

/* ------------------------------------------------------------------------------------
 * O2 Encode.  Eq 1: a_{m+1,j} = sum_i a_{i,j}; partitioned per BS x BS block
 * (ref [20]); Alg 1: each thread sums its column top -> bottom, i.e.
 * sequential ascending order, in the working precision.
 *   Acs[I][k] = ((A[I*bs][k] + A[I*bs+1][k]) + ...) + A[I*bs+bs-1][k]
 * Eq 2 (index garbled): b_{i,q+1} = sum_j b_{i,j}, per BS-column block:
 *   Bcs[k][J] = sequential ascending sum over j in block J of B[k][j]
 * ------------------------------------------------------------------------------------ */
void oracle_encode_cols(int dtype, int64_t M, int64_t K, int bs, const void *A, int64_t lda,
                        void *Acs, int64_t ld_acs) {
  for (int64_t I = 0; I < M / bs; ++I)
    for (int64_t k = 0; k < K; ++k) {
      if (dtype == OR_F64) {
        double s = 0.0;
        for (int64_t i = I * bs; i < I * bs + bs; ++i) s = s + ((const double *)A)[i * lda + k];
        ((double *)Acs)[I * ld_acs + k] = s;
      } else {
        float s = 0.0f;
        for (int64_t i = I * bs; i < I * bs + bs; ++i) s = s + ((const float *)A)[i * lda + k];
        ((float *)Acs)[I * ld_acs + k] = s;
      }
    }
}

void oracle_encode_rows(int dtype, int64_t K, int64_t N, int bs, const void *B, int64_t ldb,
                        void *Bcs, int64_t ld_bcs) {
  for (int64_t k = 0; k < K; ++k)
    for (int64_t J = 0; J < N / bs; ++J) {
      if (dtype == OR_F64) {
        double s = 0.0;
        for (int64_t j = J * bs; j < J * bs + bs; ++j) s = s + ((const double *)B)[k * ldb + j];
        ((double *)Bcs)[k * ld_bcs + J] = s;
      } else {
        float s = 0.0f;
        for (int64_t j = J * bs; j < J * bs + bs; ++j) s = s + ((const float *)B)[k * ldb + j];
        ((float *)Bcs)[k * ld_bcs + J] = s;
      }
    }
}

/* ------------------------------------------------------------------------------------
 * O3 Top-p.  §IV-E: "For each vector a_i from matrix A and each vector b_j from
 * matrix B, the p elements with the largest absolute values and the corresponding indices
 * are determined."  Alg 1: p rounds; each round scans for the maximum |x|,
 * records value and index, and excludes it from the next round.  Reading R13/R14: ties go
 * to the lowest index (strict '>' while scanning ascending); excluded = already chosen
 * index (zeros remain selectable); p <= length.
 * The vector is x[0], x[stride], ..., x[(len-1)*stride].
 * ------------------------------------------------------------------------------------ */
void oracle_topp_vector(int dtype, const void *x, int64_t len, int64_t stride, int p,
                        double *val, int32_t *idx) {
  for (int m = 0; m < p; ++m) {
    double best = -1.0;
    int64_t best_k = -1;
    for (int64_t k = 0; k < len; ++k) {
      int taken = 0;
      for (int r = 0; r < m; ++r)
        if (idx[r] == k) taken = 1;
      if (taken) continue;
      double v = fabs(ld(dtype, x, k * stride));
      if (v > best) { best = v; best_k = k; }
    }
    val[m] = best;
    idx[m] = (int32_t)best_k;
  }
}

/* Top-p of every data row of A (M rows) then every checksum row of Acs (M/bs rows):
 * topA_val / topA_idx are (M + M/bs) x p.  Reading R4: checksum vectors are in the
 * top-p (Alg 1 localSums/maxSum). */
void oracle_topp_rows(int dtype, int64_t M, int64_t K, int bs, int p, const void *A, int64_t lda,
                      const void *Acs, int64_t ld_acs, double *topA_val, int32_t *topA_idx) {
  size_t es = dtype == OR_F64 ? 8 : 4;
  for (int64_t i = 0; i < M; ++i)
    oracle_topp_vector(dtype, (const char *)A + (size_t)(i * lda) * es, K, 1, p,
                       topA_val + i * p, topA_idx + i * p);
  for (int64_t I = 0; I < M / bs; ++I)
    oracle_topp_vector(dtype, (const char *)Acs + (size_t)(I * ld_acs) * es, K, 1, p,
                       topA_val + (M + I) * p, topA_idx + (M + I) * p);
}

/* Top-p of every data column of B (N cols) then every checksum column of Bcs (N/bs cols):
 * topB_val / topB_idx are (N + N/bs) x p. */
void oracle_topp_cols(int dtype, int64_t K, int64_t N, int bs, int p, const void *B, int64_t ldb,
                      const void *Bcs, int64_t ld_bcs, double *topB_val, int32_t *topB_idx) {
  size_t es = dtype == OR_F64 ? 8 : 4;
  for (int64_t j = 0; j < N; ++j)
    oracle_topp_vector(dtype, (const char *)B + (size_t)j * es, K, ldb, p,
                       topB_val + j * p, topB_idx + j * p);
  for (int64_t J = 0; J < N / bs; ++J)
    oracle_topp_vector(dtype, (const char *)Bcs + (size_t)J * es, K, ld_bcs, p,
                       topB_val + (N + J) * p, topB_idx + (N + J) * p);
}

/* ------------------------------------------------------------------------------------
 * O4 GEMM.  Eq 15: c_ij = sum_{k=1..n} a_ik b_kj, accumulated in ascending k
 * (Alg 3 inner loop).  fma_model = 1: c = fma(a, b, c) (§IV-D, one
 * rounding per step); fma_model = 0: c = c + a*b with the product rounded separately
 * (§IV-C).  The same routine produces C = A.B, Ccol = Acs.B and Crow = A.Bcs (Eq 3).
 * Parallel over row ranges only (no reordering of any element's arithmetic).
 * ------------------------------------------------------------------------------------ */
typedef struct {
  int dtype, fma_model;
  int64_t r0, r1, N, K;
  const void *A; int64_t lda;
  const void *B; int64_t ldb;
  void *C; int64_t ldc;
} gemm_job;

static void gemm_rows(const gemm_job *g) {
  for (int64_t i = g->r0; i < g->r1; ++i)
    for (int64_t j = 0; j < g->N; ++j) {
      if (g->dtype == OR_F64) {
        const double *a = (const double *)g->A + i * g->lda;
        const double *b = (const double *)g->B + j;
        double c = 0.0;
        for (int64_t k = 0; k < g->K; ++k)
          c = g->fma_model ? fma(a[k], b[k * g->ldb], c) : c + a[k] * b[k * g->ldb];
        ((double *)g->C)[i * g->ldc + j] = c;
      } else {
        const float *a = (const float *)g->A + i * g->lda;
        const float *b = (const float *)g->B + j;
        float c = 0.0f;
        for (int64_t k = 0; k < g->K; ++k)
          c = g->fma_model ? fmaf(a[k], b[k * g->ldb], c) : c + a[k] * b[k * g->ldb];
        ((float *)g->C)[i * g->ldc + j] = c;
      }
    }
}

static void *gemm_thread(void *arg) { gemm_rows((const gemm_job *)arg); return NULL; }

void oracle_gemm(int dtype, int fma_model, int64_t M, int64_t N, int64_t K, const void *A,
                 int64_t lda, const void *B, int64_t ldb, void *C, int64_t ldc, int nthreads) {
  if (nthreads < 1) nthreads = 1;
  if (nthreads > 256) nthreads = 256;
  if ((int64_t)nthreads > M) nthreads = M > 0 ? (int)M : 1;
  gemm_job jobs[256];
  pthread_t th[256];
  for (int t = 0; t < nthreads; ++t) {
    gemm_job g = {dtype, fma_model, M * t / nthreads, M * (t + 1) / nthreads, N, K,
                  A, lda, B, ldb, C, ldc};
    jobs[t] = g;
  }
  if (nthreads == 1) { gemm_rows(&jobs[0]); return; }
  for (int t = 0; t < nthreads; ++t) pthread_create(&th[t], NULL, gemm_thread, &jobs[t]);
  for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
}

/* O9 (Alg 3): one element of C_fc recomputed with a fault.
 * site 0: XOR xor_mask into the bits of the final value ("errorVecAdd2")
 * site 1: XOR xor_mask into the partial sum right after step k_step ("errorVecAdd1")
 * site 2: add `add` to the final value (additive magnitude fault; R23)
 * site 3: add `add` to the partial sum right after step k_step (additive accumulator fault)
 * site 4: "errorVecMul" (Alg 3 inner loop: accum += (rA*rB) XOR errorVecMult):
 *         at step k_step the product is rounded on its own, XOR-ed with xor_mask and then
 *         added (c = c + (fl(a_k*b_k) ^ mask)); every other step as fma_model says
 * The row a (len K, stride 1) and column b (len K, stride ldb) are passed directly. */
static uint64_t bits_of(double x) { uint64_t u; memcpy(&u, &x, 8); return u; }
static double of_bits(uint64_t u) { double x; memcpy(&x, &u, 8); return x; }
static uint32_t bits_of_f(float x) { uint32_t u; memcpy(&u, &x, 4); return u; }
static float of_bits_f(uint32_t u) { float x; memcpy(&x, &u, 4); return x; }

double oracle_dot_fault(int dtype, int fma_model, int64_t K, const void *a, const void *b,
                        int64_t ldb, int site, int64_t k_step, uint64_t xor_mask, double add) {
  if (dtype == OR_F64) {
    const double *x = (const double *)a, *y = (const double *)b;
    double c = 0.0;
    for (int64_t k = 0; k < K; ++k) {
      if (site == 4 && k == k_step) {
        double prod = x[k] * y[k * ldb];
        c = c + of_bits(bits_of(prod) ^ xor_mask);
      } else {
        c = fma_model ? fma(x[k], y[k * ldb], c) : c + x[k] * y[k * ldb];
      }
      if (site == 1 && k == k_step) c = of_bits(bits_of(c) ^ xor_mask);
      if (site == 3 && k == k_step) c = c + add;
    }
    if (site == 0) c = of_bits(bits_of(c) ^ xor_mask);
    if (site == 2) c = c + add;
    return c;
  } else {
    const float *x = (const float *)a, *y = (const float *)b;
    float c = 0.0f;
    for (int64_t k = 0; k < K; ++k) {
      if (site == 4 && k == k_step) {
        float prod = x[k] * y[k * ldb];
        c = c + of_bits_f(bits_of_f(prod) ^ (uint32_t)xor_mask);
      } else {
        c = fma_model ? fmaf(x[k], y[k * ldb], c) : c + x[k] * y[k * ldb];
      }
      if (site == 1 && k == k_step) c = of_bits_f(bits_of_f(c) ^ (uint32_t)xor_mask);
      if (site == 3 && k == k_step) c = (float)((double)c + add);
    }
    if (site == 0) c = of_bits_f(bits_of_f(c) ^ (uint32_t)xor_mask);
    if (site == 2) c = (float)((double)c + add);
    return (double)c;
  }
}

/* ------------------------------------------------------------------------------------
 * O5 y.  §IV-E: y = maximum of the three cases; reading R3: always the max
 * of all three terms (case 1 only when S = A_idx ∩ B_idx is non-empty):
 *   y = max( max_{s in S} |a_s||b_s| , max(va)*min(vb) , max(vb)*min(va) )
 * va/vb are the p largest |values| (descending), ia/ib their indices.
 * ------------------------------------------------------------------------------------ */
double oracle_y(int p, const double *va, const int32_t *ia, const double *vb, const int32_t *ib) {
  double case1 = 0.0;
  for (int r = 0; r < p; ++r)
    for (int s = 0; s < p; ++s)
      if (ia[r] == ib[s]) {
        double prod = va[r] * vb[s];
        if (prod > case1) case1 = prod;
      }
  double amax = va[0], amin = va[0], bmax = vb[0], bmin = vb[0];
  for (int r = 1; r < p; ++r) {
    if (va[r] > amax) amax = va[r];
    if (va[r] < amin) amin = va[r];
    if (vb[r] > bmax) bmax = vb[r];
    if (vb[r] < bmin) bmin = vb[r];
  }
  double case2 = amax * bmin;
  double case3 = bmax * amin;
  double y = case1;
  if (case2 > y) y = case2;
  if (case3 > y) y = case3;
  return y;
}

/* O6 sigma coefficient sqrt(F(n)):
 *  fma_model = 1: Eq 28  sigma <= sqrt(n(n+1)(2n+1)/48) * y * 2^-t
 *  fma_model = 0: P:L287          sigma <= sqrt((n(n+1)(n+1/2) + 2n)/24) * 2^-t * y
 * n = logical inner dimension K (Eq 15, reading R5).  Evaluation order is normative. */
double oracle_sigma_coeff(int64_t n, int fma_model) {
  double dn = (double)n;
  double F;
  if (fma_model)
    F = ((dn * (dn + 1.0)) * (2.0 * dn + 1.0)) / 48.0;
  else
    F = ((dn * (dn + 1.0)) * (dn + 0.5) + 2.0 * dn) / 24.0;
  return sqrt(F);
}

/* sigma and eps for one carried checksum element.  Eq 7: interval EV +- omega*sigma;
 * summation EV = 0 (Eq 27); non-FMA adds the product mean EV_Prod <= n/3 * 2^-2t * y
 * (Eq 43; reading R7) as |EV|.  */
void oracle_bound(int64_t n, int fma_model, int t, double omega, double y, double *sig,
                  double *eps) {
  double s = oracle_sigma_coeff(n, fma_model);
  double sg = s * ldexp(y, -t);
  double e = omega * sg;
  if (!fma_model) e = e + ((double)n / 3.0) * ldexp(y, -2 * t);
  *sig = sg;
  *eps = e;
}

/* All bounds of the carried checksums (§IV-E last paragraph; reading R4):
 *   column checksum (I, j): y(topA[checksum row I], topB[column j])   -> eps_col[(M/bs) x N]
 *   row checksum    (i, J): y(topA[row i],          topB[checksum col J]) -> eps_row[M x (N/bs)]
 * sig_* may be NULL. */
void oracle_bounds_all(int64_t M, int64_t N, int64_t K, int bs, int p, double omega, int t,
                       int fma_model, const double *topA_val, const int32_t *topA_idx,
                       const double *topB_val, const int32_t *topB_idx, double *eps_col,
                       double *sig_col, double *eps_row, double *sig_row) {
  int64_t nI = M / bs, nJ = N / bs;
  for (int64_t I = 0; I < nI; ++I)
    for (int64_t j = 0; j < N; ++j) {
      double y = oracle_y(p, topA_val + (M + I) * p, topA_idx + (M + I) * p, topB_val + j * p,
                          topB_idx + j * p);
      double sg, e;
      oracle_bound(K, fma_model, t, omega, y, &sg, &e);
      eps_col[I * N + j] = e;
      if (sig_col) sig_col[I * N + j] = sg;
    }
  for (int64_t i = 0; i < M; ++i)
    for (int64_t J = 0; J < nJ; ++J) {
      double y = oracle_y(p, topA_val + i * p, topA_idx + i * p, topB_val + (N + J) * p,
                          topB_idx + (N + J) * p);
      double sg, e;
      oracle_bound(K, fma_model, t, omega, y, &sg, &e);
      eps_row[i * nJ + J] = e;
      if (sig_row) sig_row[i * nJ + J] = sg;
    }
}

/* ------------------------------------------------------------------------------------
 * O7 Check + classify.  Eq 4: c*_{m+1,j} = sum_i c_ij, c*_{i,q+1} = sum_j c_ij per
 * block (sequential ascending, in double: reading R11/R12); Eq 6 with reading R9:
 * consistent iff |d| <= eps, so NaN/Inf are critical.  Three classes (R10):
 *   0 ROUNDING |d| <= sig; 1 TOLERABLE sig < |d| <= eps; 2 CRITICAL !(|d| <= eps).
 * O8 block verdict ("Errors can be located at the intersection of mismatching
 * checksum rows and columns"; R15/R16):
 *   nr = #critical row checks, nc = #critical column checks in the block
 *   (0,0) CLEAN(0); (1,1) SINGLE(4) -> located, corrected by oracle_correct;
 *   exactly one of nr,nc nonzero -> CHECKSUM_ONLY(2); otherwise UNCORRECTABLE(3).
 *
 * Outputs (per block b = I*nJ + J), flat arrays:
 *   rep_status[b], rep_worst[b], rep_nrows[b], rep_ncols[b], rep_row[b], rep_col[b]
 *   rep_ratio[b] = max |d|/eps over the block's checks (inf when eps = 0 and d != 0, or d NaN)
 *   counts[8] = blocks, clean, corrected, checksum_only, uncorrectable, rounding, tolerable,
 *   critical; *max_ratio.  d_col / d_row (may be NULL) receive the differences.
 * ------------------------------------------------------------------------------------ */
static int classify(double d, double sig, double eps) {
  double a = fabs(d);
  if (a <= sig) return 0;
  if (a <= eps) return 1;
  return 2; /* includes NaN: !(|d| <= eps) */
}

static double ratio_of(double d, double eps) {
  double a = fabs(d);
  if (a != a) return INFINITY;
  if (eps > 0.0) return a / eps;
  return a == 0.0 ? 0.0 : INFINITY;
}

/* Where eps (and sigma) of a carried checksum come from.  A-ABFT (the method): the bound of
 * §IV-E from the top-p tables.  External (NEXT-3 comparators, reading R26): a caller-given
 * eps per checksum (eps_col / eps_row, e.g. the SEA-ABFT bound) or, when those are NULL, one
 * fixed eps for every check ("ABFT with manually set error bounds", Table I);
 * external bounds carry no sigma, so sigma = eps (classes ROUNDING / CRITICAL only). */
typedef struct {
  int external;
  int64_t M, N, K;
  int bs, p, t, fma_model;
  double omega;
  const double *topA_val, *topB_val;
  const int32_t *topA_idx, *topB_idx;
  const double *eps_col, *eps_row;
  double eps_fixed;
} eps_source;

static void col_bound(const eps_source *s, int64_t I, int64_t j, double *sg, double *e) {
  if (s->external) {
    *e = s->eps_col ? s->eps_col[I * s->N + j] : s->eps_fixed;
    *sg = *e;
    return;
  }
  int p = s->p;
  double y = oracle_y(p, s->topA_val + (s->M + I) * p, s->topA_idx + (s->M + I) * p,
                      s->topB_val + j * p, s->topB_idx + j * p);
  oracle_bound(s->K, s->fma_model, s->t, s->omega, y, sg, e);
}

static void row_bound(const eps_source *s, int64_t i, int64_t J, double *sg, double *e) {
  if (s->external) {
    *e = s->eps_row ? s->eps_row[i * (s->N / s->bs) + J] : s->eps_fixed;
    *sg = *e;
    return;
  }
  int p = s->p;
  double y = oracle_y(p, s->topA_val + i * p, s->topA_idx + i * p, s->topB_val + (s->N + J) * p,
                      s->topB_idx + (s->N + J) * p);
  oracle_bound(s->K, s->fma_model, s->t, s->omega, y, sg, e);
}

static void check_core(int dtype, const eps_source *src, const void *C, int64_t ldc,
                       const void *Ccol, int64_t ld_ccol, const void *Crow, int64_t ld_crow,
                       int32_t *rep_status, int32_t *rep_worst, int32_t *rep_nrows,
                       int32_t *rep_ncols, int32_t *rep_row, int32_t *rep_col, double *rep_ratio,
                       int64_t *counts, double *max_ratio, double *d_col, double *d_row) {
  int64_t M = src->M, N = src->N;
  int bs = src->bs;
  int64_t nI = M / bs, nJ = N / bs;
  for (int c = 0; c < 8; ++c) counts[c] = 0;
  *max_ratio = 0.0;
  for (int64_t I = 0; I < nI; ++I)
    for (int64_t J = 0; J < nJ; ++J) {
      int64_t b = I * nJ + J;
      int nr = 0, nc = 0, worst = 0, crit_row = -1, crit_col = -1;
      double bratio = 0.0;
      /* column checks j in J: reference sum down the BS rows of block-row I */
      for (int64_t j = J * bs; j < J * bs + bs; ++j) {
        double ref = 0.0;
        for (int64_t i = I * bs; i < I * bs + bs; ++i) ref = ref + ld(dtype, C, i * ldc + j);
        double d = ref - ld(dtype, Ccol, I * ld_ccol + j);
        double sg, e;
        col_bound(src, I, j, &sg, &e);
        int cl = classify(d, sg, e);
        counts[5 + cl] += 1;
        if (cl > worst) worst = cl;
        if (cl == 2) { nc += 1; crit_col = (int)j; }
        double r = ratio_of(d, e);
        if (r > bratio) bratio = r;
        if (d_col) d_col[I * N + j] = d;
      }
      /* row checks i in I: reference sum across the BS columns of block-column J */
      for (int64_t i = I * bs; i < I * bs + bs; ++i) {
        double ref = 0.0;
        for (int64_t j = J * bs; j < J * bs + bs; ++j) ref = ref + ld(dtype, C, i * ldc + j);
        double d = ref - ld(dtype, Crow, i * ld_crow + J);
        double sg, e;
        row_bound(src, i, J, &sg, &e);
        int cl = classify(d, sg, e);
        counts[5 + cl] += 1;
        if (cl > worst) worst = cl;
        if (cl == 2) { nr += 1; crit_row = (int)i; }
        double r = ratio_of(d, e);
        if (r > bratio) bratio = r;
        if (d_row) d_row[i * nJ + J] = d;
      }
      int status;
      if (nr == 0 && nc == 0) status = 0;
      else if (nr == 1 && nc == 1) status = 4;
      else if (nr == 0 || nc == 0) status = 2;
      else status = 3;
      counts[0] += 1;
      if (status == 0) counts[1] += 1;
      if (status == 2) counts[3] += 1;
      if (status == 3) counts[4] += 1;
      rep_status[b] = status;
      rep_worst[b] = worst;
      rep_nrows[b] = nr;
      rep_ncols[b] = nc;
      rep_row[b] = status == 4 ? crit_row : -1;
      rep_col[b] = status == 4 ? crit_col : -1;
      rep_ratio[b] = bratio;
      if (bratio > *max_ratio) *max_ratio = bratio;
    }
}

void oracle_check(int dtype, int64_t M, int64_t N, int64_t K, int bs, int p, double omega, int t,
                  int fma_model, const void *C, int64_t ldc, const void *Ccol, int64_t ld_ccol,
                  const void *Crow, int64_t ld_crow, const double *topA_val,
                  const int32_t *topA_idx, const double *topB_val, const int32_t *topB_idx,
                  int32_t *rep_status, int32_t *rep_worst, int32_t *rep_nrows,
                  int32_t *rep_ncols, int32_t *rep_row, int32_t *rep_col, double *rep_ratio,
                  int64_t *counts, double *max_ratio, double *d_col, double *d_row) {
  eps_source src = {0, M, N, K, bs, p, t, fma_model, omega, topA_val, topB_val, topA_idx,
                    topB_idx, NULL, NULL, 0.0};
  check_core(dtype, &src, C, ldc, Ccol, ld_ccol, Crow, ld_crow, rep_status, rep_worst, rep_nrows,
             rep_ncols, rep_row, rep_col, rep_ratio, counts, max_ratio, d_col, d_row);
}

/* The same check against an external eps (NEXT-3 comparators; reading R26): eps_col
 * ((M/bs) x N) and eps_row (M x (N/bs)) or, when both are NULL, eps_fixed everywhere. */
void oracle_check_ext(int dtype, int64_t M, int64_t N, int bs, const void *C, int64_t ldc,
                      const void *Ccol, int64_t ld_ccol, const void *Crow, int64_t ld_crow,
                      const double *eps_col, const double *eps_row, double eps_fixed,
                      int32_t *rep_status, int32_t *rep_worst, int32_t *rep_nrows,
                      int32_t *rep_ncols, int32_t *rep_row, int32_t *rep_col, double *rep_ratio,
                      int64_t *counts, double *max_ratio, double *d_col, double *d_row) {
  eps_source src = {1, M, N, 0, bs, 0, 0, 0, 0.0, NULL, NULL, NULL, NULL, eps_col, eps_row,
                    eps_fixed};
  check_core(dtype, &src, C, ldc, Ccol, ld_ccol, Crow, ld_crow, rep_status, rep_worst, rep_nrows,
             rep_ncols, rep_row, rep_col, rep_ratio, counts, max_ratio, d_col, d_row);
}

/* O8 correction (reading R15, Huang-Abraham [10]; Alg 2 "start correction"):
 * for every SINGLE(4) block with located (i, j):
 *   C[i][j] <- Ccol[I][j] - sum_{i' in I, i' != i} C[i'][j]   (double, ascending i'; stored in w)
 * then re-check row i against Crow[i][J] with its own eps: CORRECTED(1) if |d| <= eps,
 * else UNCORRECTABLE(3).  Updates counts[2] / counts[4]. */
static void correct_core(int dtype, const eps_source *src, void *C, int64_t ldc,
                         const void *Ccol, int64_t ld_ccol, const void *Crow, int64_t ld_crow,
                         int32_t *rep_status, const int32_t *rep_row, const int32_t *rep_col,
                         int64_t *counts) {
  int64_t M = src->M, N = src->N;
  int bs = src->bs;
  int64_t nI = M / bs, nJ = N / bs;
  (void)M;
  for (int64_t I = 0; I < nI; ++I)
    for (int64_t J = 0; J < nJ; ++J) {
      int64_t b = I * nJ + J;
      if (rep_status[b] != 4) continue;
      int64_t i = rep_row[b], j = rep_col[b];
      double v = ld(dtype, Ccol, I * ld_ccol + j);
      for (int64_t ii = I * bs; ii < I * bs + bs; ++ii)
        if (ii != i) v = v - ld(dtype, C, ii * ldc + j);
      if (dtype == OR_F64) ((double *)C)[i * ldc + j] = v;
      else ((float *)C)[i * ldc + j] = (float)v;
      double ref = 0.0;
      for (int64_t jj = J * bs; jj < J * bs + bs; ++jj) ref = ref + ld(dtype, C, i * ldc + jj);
      double d = ref - ld(dtype, Crow, i * ld_crow + J);
      double sg, e;
      row_bound(src, i, J, &sg, &e);
      if (fabs(d) <= e) { rep_status[b] = 1; counts[2] += 1; }
      else { rep_status[b] = 3; counts[4] += 1; }
    }
}

void oracle_correct(int dtype, int64_t M, int64_t N, int64_t K, int bs, int p, double omega, int t,
                    int fma_model, void *C, int64_t ldc, const void *Ccol, int64_t ld_ccol,
                    const void *Crow, int64_t ld_crow, const double *topA_val,
                    const int32_t *topA_idx, const double *topB_val, const int32_t *topB_idx,
                    int32_t *rep_status, const int32_t *rep_row, const int32_t *rep_col,
                    int64_t *counts) {
  eps_source src = {0, M, N, K, bs, p, t, fma_model, omega, topA_val, topB_val, topA_idx,
                    topB_idx, NULL, NULL, 0.0};
  correct_core(dtype, &src, C, ldc, Ccol, ld_ccol, Crow, ld_crow, rep_status, rep_row, rep_col,
               counts);
}

/* Correction with the external eps of oracle_check_ext (the re-verified row uses eps_row, or
 * eps_fixed when eps_row is NULL). */
void oracle_correct_ext(int dtype, int64_t M, int64_t N, int bs, void *C, int64_t ldc,
                        const void *Ccol, int64_t ld_ccol, const void *Crow, int64_t ld_crow,
                        const double *eps_row, double eps_fixed, int32_t *rep_status,
                        const int32_t *rep_row, const int32_t *rep_col, int64_t *counts) {
  eps_source src = {1, M, N, 0, bs, 0, 0, 0, 0.0, NULL, NULL, NULL, NULL, NULL, eps_row,
                    eps_fixed};
  correct_core(dtype, &src, C, ldc, Ccol, ld_ccol, Crow, ld_crow, rep_status, rep_row, rep_col,
               counts);
}

/* ------------------------------------------------------------------------------------
 * O11 SEA-ABFT bound (NEXT-3 comparator, reporting only).  §III, the simplified
 * error analysis bound of ref [28] for the column checksum of an (m+1) x n column-checksum
 * matrix A times a column b:
 *   |c_{n+1} - c*_{n+1}| < ((n + 2m - 2) ||b||_2 sum_{i=1..m} ||a_i||_2
 *                          + n ||a_{m+1}||_2 ||b||_2) eps_M,          eps_M = 2^-t
 * Partitioned encoding: m = bs rows of block-row I, a_{m+1} = Acs[I] (the checksum
 * row), b = column j of B, n = K.  A row checksum (i, J) is the transposed statement (A, b)
 * -> (B^T, a_i): the BS columns b_j of block-column J play a_1..a_m, Bcs[:, J] plays a_{m+1}
 * and row a_i of A plays b.  The corner (I, J) (reading R25, only for the Table II/III
 * average): a_{m+1} = Acs[I], b = Bcs[:, J].
 * Norms: ||x||_2 = sqrt of the sequential ascending sum of x_k^2 in double.
 * ------------------------------------------------------------------------------------ */
static double norm_seq(int dtype, const void *X, int64_t off, int64_t len, int64_t stride) {
  double s = 0.0;
  for (int64_t k = 0; k < len; ++k) {
    double v = ld(dtype, X, off + k * stride);
    s = s + v * v;
  }
  return sqrt(s);
}

/* ||row r||_2 of an R x L row-major matrix (ld) -> out[r] */
void oracle_norms_rows(int dtype, int64_t R, int64_t L, const void *X, int64_t ldx, double *out) {
  for (int64_t r = 0; r < R; ++r) out[r] = norm_seq(dtype, X, r * ldx, L, 1);
}

/* ||column c||_2 of an L x Cn row-major matrix (ld) -> out[c] */
void oracle_norms_cols(int dtype, int64_t L, int64_t Cn, const void *X, int64_t ldx, double *out) {
  for (int64_t c = 0; c < Cn; ++c) out[c] = norm_seq(dtype, X, c, L, ldx);
}

/* nA[M] row norms of A, nAcs[M/bs] of the checksum rows, nB[N] column norms of B, nBcs[N/bs]
 * of the checksum columns.  Outputs eps_col (M/bs) x N, eps_row M x (N/bs), eps_corner
 * (M/bs) x (N/bs) (any may be NULL).  Evaluation: ((n+2m-2) * ||b|| * S + n * ||a_{m+1}|| *
 * ||b||) * 2^-t with S = sequential ascending sum of the m norms. */
void oracle_sea_bounds(int64_t M, int64_t N, int64_t K, int bs, int t, const double *nA,
                       const double *nAcs, const double *nB, const double *nBcs, double *eps_col,
                       double *eps_row, double *eps_corner) {
  int64_t nI = M / bs, nJ = N / bs;
  double n = (double)K, c1 = (double)K + 2.0 * bs - 2.0;
  for (int64_t I = 0; I < nI; ++I) {
    double SA = 0.0;
    for (int64_t i = I * bs; i < I * bs + bs; ++i) SA = SA + nA[i];
    for (int64_t j = 0; j < N; ++j)
      if (eps_col) eps_col[I * N + j] = ldexp(c1 * nB[j] * SA + n * nAcs[I] * nB[j], -t);
    for (int64_t J = 0; J < nJ; ++J)
      if (eps_corner) eps_corner[I * nJ + J] = ldexp(c1 * nBcs[J] * SA + n * nAcs[I] * nBcs[J], -t);
  }
  for (int64_t J = 0; J < nJ; ++J) {
    double SB = 0.0;
    for (int64_t j = J * bs; j < J * bs + bs; ++j) SB = SB + nB[j];
    for (int64_t i = 0; i < M; ++i)
      if (eps_row) eps_row[i * nJ + J] = ldexp(c1 * nA[i] * SB + n * nBcs[J] * nA[i], -t);
  }
}

