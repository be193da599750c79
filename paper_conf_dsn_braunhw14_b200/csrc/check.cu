// check.cu -- steps 4a-4c and the correction of Alg 2 on sm_100a.
//
// Bound (§IV-E): per carried checksum element, y from the top-p lists of the two
// vectors of its inner product (three cases, reading R3), sigma = sqrt(F(K)) y 2^-t
// (Eq 28 P:L219 / P:L287), eps = omega sigma (Eq 7) (+ |EV_Prod| Eq 43 when
// fma_model = 0).  Evaluated in double with explicit round-to-nearest intrinsics so no FMA
// contraction can change a bit (bit-identical to the definition).
//
// Check (Eq 4-6): one CTA per BS x BS sub-matrix of C (as Alg 2).  The block is
// streamed in 32-row strips through padded shared memory: a thread per column keeps the
// reference column sum in a register (ascending i) and a thread per row sums its strip row
// (ascending j); both in double (readings R11/R12).  Classification (R9/R10):
// ROUNDING |d| <= sigma, TOLERABLE <= eps, CRITICAL otherwise (NaN/Inf included).
#include <algorithm>
#include <atomic>
#include <cfloat>
#include <math_constants.h>

#include "common.cuh"

namespace aabft {
namespace {


template <int P>
__device__ __forceinline__ double y_bound(const double *__restrict__ va, const int *__restrict__ ia,
                                          const double *__restrict__ vb,
                                          const int *__restrict__ ib) {
  double a[P], b[P];
  int ai[P], bi[P];
#pragma unroll
  for (int r = 0; r < P; ++r) { a[r] = va[r]; b[r] = vb[r]; ai[r] = ia[r]; bi[r] = ib[r]; }
  double case1 = 0.0;
#pragma unroll
  for (int r = 0; r < P; ++r)
#pragma unroll
    for (int s = 0; s < P; ++s)
      if (ai[r] == bi[s]) case1 = fmax(case1, __dmul_rn(a[r], b[s]));
  double amax = a[0], amin = a[0], bmax = b[0], bmin = b[0];
#pragma unroll
  for (int r = 1; r < P; ++r) {
    amax = fmax(amax, a[r]); amin = fmin(amin, a[r]);
    bmax = fmax(bmax, b[r]); bmin = fmin(bmin, b[r]);
  }
  return fmax(case1, fmax(__dmul_rn(amax, bmin), __dmul_rn(bmax, amin)));
}

struct Bound {
  double sig, eps;
};
__device__ __forceinline__ Bound bound_of(const BoundParams &bp, double y) {
  Bound b;
  b.sig = __dmul_rn(bp.s, __dmul_rn(y, bp.two_mt));
  b.eps = __dmul_rn(bp.omega, b.sig);
  if (!bp.fma_model) b.eps = __dadd_rn(b.eps, __dmul_rn(bp.ev_coeff, __dmul_rn(y, bp.two_m2t)));
  return b;
}

__device__ __forceinline__ int classify(double d, const Bound &b) {
  const double a = fabs(d);
  if (a <= b.sig) return 0;
  if (a <= b.eps) return 1;
  return 2;  // !(|d| <= eps): NaN and Inf are critical (reading R9)
}
__device__ __forceinline__ double ratio_of(double d, double eps) {
  const double a = fabs(d);
  if (a != a) return CUDART_INF;
  if (eps > 0.0) return a / eps;
  return a == 0.0 ? 0.0 : CUDART_INF;
}

// |d| / eps for the report (a diagnostic: single-precision division is enough, no DDIV)
__device__ __forceinline__ double ratio_fast(double d, double eps) {
  const double a = fabs(d);
  if (a != a) return CUDART_INF;
  if (eps > 0.0) return (double)__fdividef((float)a, (float)eps);
  return a == 0.0 ? 0.0 : CUDART_INF;
}

// atomic max on non-negative doubles (bit pattern order == value order)
__device__ __forceinline__ void atomic_max_nonneg(double *addr, double v) {
  atomicMax(reinterpret_cast<unsigned long long *>(addr),
            (unsigned long long)__double_as_longlong(v));
}

// --------------------------------------------------------------------------- bound only
template <int P>
__global__ void bound_kernel(int64_t M, int64_t N, int bs, BoundParams bp,
                             const double *__restrict__ tav, const int *__restrict__ tai,
                             const double *__restrict__ tbv, const int *__restrict__ tbi,
                             double *eps_col, double *sig_col, double *eps_row,
                             double *sig_row) {
  const int64_t ncol = (M / bs) * N, nrow = M * (N / bs);
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < ncol + nrow;
       e += (int64_t)gridDim.x * blockDim.x) {
    if (e < ncol) {
      const int64_t I = e / N, j = e % N;
      const double y = y_bound<P>(tav + (M + I) * P, tai + (M + I) * P, tbv + j * P, tbi + j * P);
      const Bound b = bound_of(bp, y);
      if (eps_col) eps_col[e] = b.eps;
      if (sig_col) sig_col[e] = b.sig;
    } else {
      const int64_t f = e - ncol, nJ = N / bs, i = f / nJ, J = f % nJ;
      const double y = y_bound<P>(tav + i * P, tai + i * P, tbv + (N + J) * P, tbi + (N + J) * P);
      const Bound b = bound_of(bp, y);
      if (eps_row) eps_row[f] = b.eps;
      if (sig_row) sig_row[f] = b.sig;
    }
  }
}

// bound of arbitrary C_fc elements (row / col index straight into the top-p tables, whose
// data vectors come first and checksum vectors after)
template <int P>
__global__ void bound_elements_kernel(int64_t M, int64_t N, int bs, BoundParams bp,
                                      const double *__restrict__ tav, const int *__restrict__ tai,
                                      const double *__restrict__ tbv, const int *__restrict__ tbi,
                                      const int64_t *__restrict__ rows,
                                      const int64_t *__restrict__ cols, int64_t n, double *sig,
                                      double *eps) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = rows[e], c = cols[e];
    double sg = CUDART_NAN, ep = CUDART_NAN;
    if (r >= 0 && r < M + M / bs && c >= 0 && c < N + N / bs) {
      const Bound b = bound_of(bp, y_bound<P>(tav + r * P, tai + r * P, tbv + c * P, tbi + c * P));
      sg = b.sig;
      ep = b.eps;
    }
    if (sig) sig[e] = sg;
    if (eps) eps[e] = ep;
  }
}

// --------------------------------------------------------------------------- check
struct CheckArgs {
  int64_t M, N;
  int bs;
  const void *C;
  int64_t ldc;
  const void *Ccol;
  int64_t ld_ccol;
  const void *Crow;
  int64_t ld_crow;
  const double *tav;
  const int *tai;
  const double *tbv;
  const int *tbi;
  aabft_block_report *rep;
  aabft_counts *cnt;
  const double *Rcol;  // fused reference sums from the GEMM epilogue (NULL = re-sum C)
  const double *Rrow;
  const double *Rcol2;  // further partial reference sums from the epilogue, added in order
  const double *Rrow2;  // (Rrow2 holds row_parts - 1 planes of M x N/bs)
  int col_parts, row_parts;
  // external eps (NEXT-3 comparators, reading R26): per-checksum arrays or one fixed value
  const double *eps_col;  // (M/bs) x N dense, or NULL
  const double *eps_row;  // M x (N/bs) dense, or NULL
  double eps_fixed;
  // counters: CTAs add into the workspace accumulator `acc` (zeroed by aabft_gemm, re-armed by
  // the last CTA, which writes the totals to `cnt`), so no memset sits between the GEMM and
  // the check; NULL = add straight into `cnt` after a memset (no workspace given)
  unsigned long long *acc;  // [9]: n[8], max_ratio bits; [9]: CTA ticket
  int correct;              // AABFT_FLAG_CHECK_CORRECTS: correct SINGLE blocks in place
};

// Bound of column check (I, j) / row check (i, J): the A-ABFT bound from the top-p tables, or
// (EXT) the caller's eps with sigma = eps (an external bound carries no sigma: classes
// ROUNDING / CRITICAL only, as the oracle's check_ext)
template <bool EXT, int P>
__device__ __forceinline__ Bound col_bound(const CheckArgs &a, const BoundParams &bp, int64_t I,
                                           int64_t j) {
  if (EXT) {
    Bound b;
    b.eps = a.eps_col ? a.eps_col[I * a.N + j] : a.eps_fixed;
    b.sig = b.eps;
    return b;
  }
  return bound_of(bp, y_bound<P>(a.tav + (a.M + I) * P, a.tai + (a.M + I) * P, a.tbv + j * P,
                                 a.tbi + j * P));
}
template <bool EXT, int P>
__device__ __forceinline__ Bound row_bound(const CheckArgs &a, const BoundParams &bp, int64_t i,
                                           int64_t J) {
  if (EXT) {
    Bound b;
    b.eps = a.eps_row ? a.eps_row[i * (a.N / a.bs) + J] : a.eps_fixed;
    b.sig = b.eps;
    return b;
  }
  return bound_of(bp, y_bound<P>(a.tav + i * P, a.tai + i * P, a.tbv + (a.N + J) * P,
                                 a.tbi + (a.N + J) * P));
}

// block verdict + report + aggregated counter update (shared by both check kernels)
__device__ __forceinline__ void finish_block(const CheckArgs &a, int64_t blk, int nr, int nc,
                                             int crit_row, int crit_col, const int cls[3],
                                             double br) {
  uint8_t status;
  if (nr == 0 && nc == 0) status = AABFT_BLK_CLEAN;
  else if (nr == 1 && nc == 1) status = AABFT_BLK_SINGLE;
  else if (nr == 0 || nc == 0) status = AABFT_BLK_CHECKSUM_ONLY;
  else status = AABFT_BLK_UNCORRECTABLE;
  aabft_block_report r;
  r.status = status;
  r.worst_class = (uint8_t)(cls[2] ? 2 : (cls[1] ? 1 : 0));
  r.n_bad_rows = (uint16_t)min(nr, 65535);
  r.n_bad_cols = (uint16_t)min(nc, 65535);
  r.reserved = 0;
  r.row = status == AABFT_BLK_SINGLE ? crit_row : -1;
  r.col = status == AABFT_BLK_SINGLE ? crit_col : -1;
  r.max_ratio = (float)br;
  a.rep[blk] = r;
  unsigned long long *n = reinterpret_cast<unsigned long long *>(a.cnt->n);
  atomicAdd(&n[0], 1ull);
  if (status == AABFT_BLK_CLEAN) atomicAdd(&n[1], 1ull);
  if (status == AABFT_BLK_CHECKSUM_ONLY) atomicAdd(&n[3], 1ull);
  if (status == AABFT_BLK_UNCORRECTABLE) atomicAdd(&n[4], 1ull);
  for (int c = 0; c < 3; ++c)
    if (cls[c]) atomicAdd(&n[5 + c], (unsigned long long)cls[c]);
  if (br > 0.0) atomicMax(reinterpret_cast<unsigned long long *>(&a.cnt->max_ratio),
                          (unsigned long long)__double_as_longlong(br));
}

// Alg 2's correction of one SINGLE block (row i, column j located by the check): returns
// AABFT_BLK_CORRECTED, or AABFT_BLK_UNCORRECTABLE when the re-verified row still fails
template <typename T, int P, bool EXT>
__device__ __forceinline__ uint8_t correct_block(const CheckArgs &a, const BoundParams &bp, T *C, int64_t blk,
                                 int64_t i, int64_t j) {
  const int bs = a.bs;
  const int64_t nJ = a.N / bs;
  const int64_t I = blk / nJ, J = blk % nJ;
  // c_ij <- Ccol[I][j] - sum_{i' != i} c_i'j  (reading R15; double, ascending i')
  double v = (double)static_cast<const T *>(a.Ccol)[I * a.ld_ccol + j];
  for (int64_t ii = I * bs; ii < I * bs + bs; ++ii)
    if (ii != i) v = v - (double)C[ii * a.ldc + j];
  C[i * a.ldc + j] = (T)v;
  // re-verify row i
  double ref = 0.0;
  for (int64_t jj = J * bs; jj < J * bs + bs; ++jj) ref = ref + (double)C[i * a.ldc + jj];
  const double d = ref - (double)static_cast<const T *>(a.Crow)[i * a.ld_crow + J];
  const Bound b = row_bound<EXT, P>(a, bp, i, J);
  if (a.Rcol) {
    // fused check: the epilogue reference sums still describe the faulty element; refresh
    // the two that pass through (i, j) from the corrected C so a later aabft_check of the
    // same product sees the corrected state (ascending order, double)
    double rc = 0.0;
    for (int64_t ii = I * bs; ii < I * bs + bs; ++ii) rc = rc + (double)C[ii * a.ldc + j];
    const_cast<double *>(a.Rcol)[I * a.N + j] = rc;
    const_cast<double *>(a.Rrow)[i * nJ + J] = ref;
  }
  return fabs(d) <= b.eps ? (uint8_t)AABFT_BLK_CORRECTED : (uint8_t)AABFT_BLK_UNCORRECTABLE;
}

// Block-verdict epilogue of both check kernels: AABFT_FLAG_CHECK_CORRECTS corrects a SINGLE
// block right here (the CTA owns the whole block; Alg 2 classifies and corrects in one kernel,
// P:L380-393), so the step needs no separate correction launch.
template <typename T, int P, bool EXT>
__device__ __forceinline__ uint8_t maybe_correct(const CheckArgs &a, const BoundParams &bp,
                                                 uint8_t status, int64_t blk, int row, int col) {
  if (!a.correct || status != AABFT_BLK_SINGLE) return status;
  return correct_block<T, P, EXT>(a, bp, static_cast<T *>(const_cast<void *>(a.C)), blk, row, col);
}

// CTA counters (s_n[8], s_mr: float bits) -> device totals.  With a workspace accumulator the
// CTAs add into it and the LAST CTA (ticket) moves the totals into `cnt` and re-arms the
// accumulator (threadfence-reduction pattern); otherwise straight atomics into the zeroed cnt.
template <typename CT>
__device__ __forceinline__ void publish_counts(const CheckArgs &a, const CT *s_n, unsigned s_mr,
                                               int tid) {
  unsigned long long *dst = a.acc ? a.acc : reinterpret_cast<unsigned long long *>(a.cnt->n);
  if (tid < 8 && s_n[tid]) atomicAdd(dst + tid, (unsigned long long)s_n[tid]);
  if (tid == 8 && s_mr) atomicMax(dst + 8, (unsigned long long)__double_as_longlong((double)__uint_as_float(s_mr)));
  if (!a.acc) return;
  __shared__ bool s_last;
  __threadfence();
  __syncthreads();
  if (tid == 0) {
    const unsigned total = gridDim.x * gridDim.y;
    s_last = atomicAdd(reinterpret_cast<unsigned *>(a.acc + 9), 1u) == total - 1;
  }
  __syncthreads();
  if (s_last) {
    __threadfence();
    if (tid < 9) reinterpret_cast<unsigned long long *>(a.cnt)[tid] = atomicExch(a.acc + tid, 0ull);
    if (tid == 0) atomicExch(reinterpret_cast<unsigned *>(a.acc + 9), 0u);
  }
}

// --------------------------------------------------------------------------- fused check
// The GEMM epilogue already produced the reference sums (Rcol, Rrow); compare them with the
// carried checksums: 2*bs checks per block, no pass over C.  Latency-bound work, so it is laid
// out for memory-level parallelism: one THREAD per check, every load independent and
// coalesced.  A CTA owns a unit of JB = 256/bs adjacent blocks of one block-row I: thread t
// holds column check j = J0*bs + t and row check (i = I*bs + t/JB, J = J0 + t%JB); the block
// verdicts are gathered in shared memory (atomics only for the rare non-rounding checks) and
// the device counters see one atomic per CTA.
constexpr int kFusedThreads = 256;
// grid: CTAs per SM (0 = as many as are co-resident: one wave, each CTA loops over units;
// measured at c2: resident 13.7 us vs 6 per SM (1.5 waves) 16.7 us)
#ifndef AABFT_CHECK_CTAS
#define AABFT_CHECK_CTAS 0
#endif

template <typename T, int P, bool EXT>
__global__ void __launch_bounds__(kFusedThreads) check_fused_kernel(CheckArgs a, BoundParams bp,
                                                                    int64_t nunits, int ngrp) {
  constexpr int MAXJB = kFusedThreads / 8;  // bs >= 8
  __shared__ int s_nr[MAXJB], s_nc[MAXJB], s_row[MAXJB], s_col[MAXJB], s_worst[MAXJB];
  __shared__ unsigned s_rmax[MAXJB];  // float bits (non-negative: integer order = value order)
  __shared__ unsigned s_n[8];  // 32-bit: native shared atomics
  __shared__ unsigned s_mr;
  const int tid = threadIdx.x, lane = tid & 31;
  const int bs = a.bs, JB = kFusedThreads / bs;
  const int lbs = __ffs(bs) - 1, ljb = __ffs(JB) - 1;  // bs, JB are powers of two
  const int64_t nJ = a.N / bs;
  if (tid < 8) s_n[tid] = 0u;
  if (tid == 8) s_mr = 0u;
  unsigned my_n[5] = {0, 0, 0, 0, 0};  // blocks, clean, corrected, checksum-only, uncorrectable
  unsigned cls0 = 0, cls1 = 0, cls2 = 0;  // checks per class (registers, not an indexed array)
  float mr = 0.f;
  const int cseg = bs < 32 ? bs : 32;  // lanes sharing one block among the column checks
  // unit u = I * ngrp + g, advanced by gridDim.x with a carry (no division in the loop)
  const unsigned du = gridDim.x / (unsigned)ngrp, dg = gridDim.x % (unsigned)ngrp;
  unsigned uI = blockIdx.x / (unsigned)ngrp, ug = blockIdx.x % (unsigned)ngrp;
  for (int64_t u = blockIdx.x; u < nunits; u += gridDim.x) {
    const int64_t I = uI, J0 = (int64_t)ug << ljb;
    uI += du;
    ug += dg;
    if (ug >= (unsigned)ngrp) { ug -= (unsigned)ngrp; ++uI; }
    if (tid < JB) {
      s_nr[tid] = 0; s_nc[tid] = 0; s_row[tid] = -1; s_col[tid] = -1; s_worst[tid] = 0;
      s_rmax[tid] = 0u;
    }
    __syncthreads();
    // Both checks' operands are gathered first (every load of the thread in flight together),
    // then the part sums are written back, then classified.
    const int Jc = tid >> lbs;                                 // column check: block of j
    const int64_t j = (J0 << lbs) + tid;
    const int ii = tid >> ljb, Jr = tid & (JB - 1);            // row check: (i, J)
    const int64_t J = J0 + Jr, i = (I << lbs) + ii;
    const bool hc = j < a.N, hr = J < nJ;
    double refc = 0.0, carc = 0.0, refr = 0.0, carr = 0.0, rc2 = 0.0, rp[7] = {};  // row_parts <= 64 / 8
    Bound bc{0.0, 0.0}, brw{0.0, 0.0};
    if (hc) {  // column check (I, j): Rcol (+ the epilogue's second part) vs carried Ccol[I][j]
      refc = a.Rcol[I * a.N + j];
      if (a.col_parts > 1) rc2 = a.Rcol2[I * a.N + j];
      carc = (double)static_cast<const T *>(a.Ccol)[I * a.ld_ccol + j];
      bc = col_bound<EXT, P>(a, bp, I, j);
    }
    if (hr) {  // row check (i, J): Rrow (+ parts) vs carried Crow[i][J]
      refr = a.Rrow[i * nJ + J];
      for (int q = 1; q < a.row_parts && q <= 7; ++q)
        rp[q - 1] = a.Rrow2[(q - 1) * a.M * nJ + i * nJ + J];
      carr = (double)static_cast<const T *>(a.Crow)[i * a.ld_crow + J];
      brw = row_bound<EXT, P>(a, bp, i, J);
    }
    // complete the epilogue parts in their fixed order and leave the full sums in Rcol / Rrow;
    // the consumed parts are zeroed so a second check (another bound) sees the same sums
    if (hc && a.col_parts > 1) {
      refc = refc + rc2;
      const_cast<double *>(a.Rcol)[I * a.N + j] = refc;
      const_cast<double *>(a.Rcol2)[I * a.N + j] = 0.0;
    }
    if (hr && a.row_parts > 1) {
      for (int q = 1; q < a.row_parts && q <= 7; ++q) {
        refr = refr + rp[q - 1];
        const_cast<double *>(a.Rrow2)[(q - 1) * a.M * nJ + i * nJ + J] = 0.0;
      }
      const_cast<double *>(a.Rrow)[i * nJ + J] = refr;
    }
    {
      float r = 0.f;
      if (hc) {
        const double d = refc - carc;
        const int cl = classify(d, bc);
        cls0 += cl == 0; cls1 += cl == 1; cls2 += cl == 2;
        if (cl) {
          atomicMax(&s_worst[Jc], cl);
          if (cl == 2) { atomicAdd(&s_nc[Jc], 1); s_col[Jc] = (int)j; }
        }
        r = (float)ratio_fast(d, bc.eps);
      }
      unsigned rb = __float_as_uint(r);  // r >= 0: bit order == value order
      if (cseg == 32) {
        rb = __reduce_max_sync(0xffffffffu, rb);
      } else {
#pragma unroll
        for (int m = 1; m < 32; m <<= 1)
          if (m < cseg) rb = max(rb, __shfl_xor_sync(0xffffffffu, rb, m));  // uniform condition
      }
      if ((lane & (cseg - 1)) == 0 && rb) atomicMax(&s_rmax[Jc], rb);
    }
    {
      float r = 0.f;
      if (hr) {
        const double d = refr - carr;
        const int cl = classify(d, brw);
        cls0 += cl == 0; cls1 += cl == 1; cls2 += cl == 2;
        if (cl) {
          atomicMax(&s_worst[Jr], cl);
          if (cl == 2) { atomicAdd(&s_nr[Jr], 1); s_row[Jr] = (int)i; }
        }
        r = (float)ratio_fast(d, brw.eps);
      }
      unsigned rb = __float_as_uint(r);
#pragma unroll
      for (int m = 1; m < 32; m <<= 1)
        if (m >= JB) rb = max(rb, __shfl_xor_sync(0xffffffffu, rb, m));  // uniform condition
      if (lane < JB && rb) atomicMax(&s_rmax[Jr], rb);
    }
    __syncthreads();
    // ---- block verdicts (warp 0: JB <= 32 blocks)
    if (tid < JB && J0 + tid < nJ) {
      const int nr = s_nr[tid], nc = s_nc[tid];
      uint8_t status;
      if (nr == 0 && nc == 0) status = AABFT_BLK_CLEAN;
      else if (nr == 1 && nc == 1) status = AABFT_BLK_SINGLE;
      else if (nr == 0 || nc == 0) status = AABFT_BLK_CHECKSUM_ONLY;
      else status = AABFT_BLK_UNCORRECTABLE;
      aabft_block_report rep;
      rep.status = status;
      rep.worst_class = (uint8_t)s_worst[tid];
      rep.n_bad_rows = (uint16_t)min(nr, 65535);
      rep.n_bad_cols = (uint16_t)min(nc, 65535);
      rep.reserved = 0;
      rep.row = status == AABFT_BLK_SINGLE ? s_row[tid] : -1;
      rep.col = status == AABFT_BLK_SINGLE ? s_col[tid] : -1;
      const float br = __uint_as_float(s_rmax[tid]);
      rep.max_ratio = br;
      a.rep[I * nJ + J0 + tid] = rep;
      my_n[0] += 1;
      my_n[1] += status == AABFT_BLK_CLEAN;
      my_n[3] += status == AABFT_BLK_CHECKSUM_ONLY;
      my_n[4] += status == AABFT_BLK_UNCORRECTABLE;
      mr = fmaxf(mr, br);
      s_nc[tid] = status == AABFT_BLK_SINGLE ? 1 : 0;  // (slot reused: SINGLE marker)
    }
    __syncthreads();
    // AABFT_FLAG_CHECK_CORRECTS: correct this unit's SINGLE blocks (a separate phase, so the
    // rare correction code does not add to the register pressure of the check above)
    if (a.correct && tid < JB && J0 + tid < nJ && s_nc[tid]) {
      const int64_t blk = I * nJ + J0 + tid;
      const uint8_t st = correct_block<T, P, EXT>(a, bp, static_cast<T *>(const_cast<void *>(a.C)),
                                                  blk, s_row[tid], s_col[tid]);
      a.rep[blk].status = st;
      my_n[2] += st == AABFT_BLK_CORRECTED;
      my_n[4] += st == AABFT_BLK_UNCORRECTABLE;
    }
    __syncthreads();  // the per-block slots are re-initialised by the next unit
  }
  // ---- CTA aggregation: warp reductions (REDUX), then one global atomic per non-zero counter
  // (per-thread totals are far below 2^32: a CTA handles a few units of 2 x 256 checks)
  const unsigned tot[8] = {my_n[0], my_n[1], my_n[2], my_n[3], my_n[4], cls0, cls1, cls2};
  unsigned wn[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) wn[c] = __reduce_add_sync(0xffffffffu, tot[c]);
  const unsigned wmr = __reduce_max_sync(0xffffffffu, __float_as_uint(mr));
  if (lane == 0) {
#pragma unroll
    for (int c = 0; c < 8; ++c)
      if (wn[c]) atomicAdd(&s_n[c], wn[c]);
    if (wmr) atomicMax(&s_mr, wmr);
  }
  __syncthreads();
  publish_counts(a, s_n, s_mr, tid);
}

// --------------------------------------------------------------------------- streaming check
// Unfused check (FP32, or bs > 64): re-sums C once, streaming.  A CTA owns block-row I x a
// chunk of CW = max(128, bs) columns (CW/bs blocks); thread c owns column j0 + c: its Eq 4
// column reference is a register running sum in ascending row order (double, reading R12).
// Strips of SR rows go through registers (the next strip's loads are issued before this
// strip's row-sum phase) into shared memory, where task (row r, block jb) forms the Eq 4 row
// reference by summing its bs elements in ascending j.  Block verdicts are gathered in shared
// memory; one global atomic per counter per CTA.
template <typename T, int P, bool EXT, int CW>
__global__ void __launch_bounds__(CW) check_stream_kernel(CheckArgs a, BoundParams bp) {
  constexpr int SR = (CW * sizeof(T) > 1024) ? 16 : 32;  // strip rows (static smem <= 48 KiB)
  constexpr int MAXB = CW / 8;                           // blocks per chunk (bs >= 8)
  __shared__ T tile[SR][CW + 1];  // odd pitch: row-sum lanes (one row each) hit distinct banks
  __shared__ int s_nr[MAXB], s_nc[MAXB], s_row[MAXB], s_col[MAXB], s_worst[MAXB];
  __shared__ unsigned s_rmax[MAXB];
  __shared__ unsigned long long s_n[8];
  __shared__ unsigned s_mr;
  const int c = threadIdx.x, lane = c & 31;
  const int bs = a.bs;
  const int64_t I = blockIdx.y, j0 = (int64_t)blockIdx.x * CW;
  const int ncols = (int)(a.N - j0 < CW ? a.N - j0 : CW);  // multiple of bs
  const int nbh = ncols / bs;
  const int64_t nJ = a.N / bs;
  if (c < MAXB) {
    s_nr[c] = 0; s_nc[c] = 0; s_row[c] = -1; s_col[c] = -1; s_worst[c] = 0; s_rmax[c] = 0u;
  }
  if (c < 8) s_n[c] = 0ull;
  if (c == 8) s_mr = 0u;
  const T *C = static_cast<const T *>(a.C);
  const bool jin = c < ncols;
  const T *col = C + (I * bs) * a.ldc + j0 + c;
  T vals[SR];
  auto load_strip = [&](int r0) {
    const int rows = bs - r0 < SR ? bs - r0 : SR;
    const T *src = col + (int64_t)r0 * a.ldc;
    if (rows == SR) {
#pragma unroll
      for (int rr = 0; rr < SR; ++rr) vals[rr] = jin ? src[(int64_t)rr * a.ldc] : T(0);
    } else {
#pragma unroll
      for (int rr = 0; rr < SR; ++rr) vals[rr] = (jin && rr < rows) ? src[(int64_t)rr * a.ldc] : T(0);
    }
  };
  load_strip(0);
  __syncthreads();  // slot initialisation
  double colsum = 0.0;
  int cls_tot[3] = {0, 0, 0};
  for (int r0 = 0; r0 < bs; r0 += SR) {
    const int rows = bs - r0 < SR ? bs - r0 : SR;
#pragma unroll
    for (int rr = 0; rr < SR; ++rr) {
      if (rr < rows) {
        colsum = colsum + (double)vals[rr];  // Eq 4, ascending i
        tile[rr][c] = vals[rr];
      }
    }
    if (r0 + SR < bs) load_strip(r0 + SR);
    __syncthreads();
    for (int t = c; t < rows * nbh; t += CW) {
      const int r = t % rows, jb = t / rows;
      const int64_t i = I * bs + r0 + r, J = j0 / bs + jb;
      double ref = 0.0;
      for (int jj = 0; jj < bs; ++jj) ref = ref + (double)tile[r][jb * bs + jj];  // asc j
      const double d = ref - (double)static_cast<const T *>(a.Crow)[i * a.ld_crow + J];
      const Bound b = row_bound<EXT, P>(a, bp, i, J);
      const int cl = classify(d, b);
      cls_tot[cl] += 1;
      if (cl) {
        atomicMax(&s_worst[jb], cl);
        if (cl == 2) { atomicAdd(&s_nr[jb], 1); s_row[jb] = (int)i; }
      }
      const float rt = (float)ratio_fast(d, b.eps);
      if (rt > 0.f) atomicMax(&s_rmax[jb], __float_as_uint(rt));
    }
    __syncthreads();  // tile consumed
  }
  if (jin) {
    const int jb = c / bs;
    const int64_t j = j0 + c;
    const double d = colsum - (double)static_cast<const T *>(a.Ccol)[I * a.ld_ccol + j];
    const Bound b = col_bound<EXT, P>(a, bp, I, j);
    const int cl = classify(d, b);
    cls_tot[cl] += 1;
    if (cl) {
      atomicMax(&s_worst[jb], cl);
      if (cl == 2) { atomicAdd(&s_nc[jb], 1); s_col[jb] = (int)j; }
    }
    const float rt = (float)ratio_fast(d, b.eps);
    if (rt > 0.f) atomicMax(&s_rmax[jb], __float_as_uint(rt));
  }
  __syncthreads();
  unsigned long long my_n[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  float mr = 0.f;
  if (c < nbh) {  // block verdicts (warp 0: nbh <= 16)
    const int nr = s_nr[c], nc = s_nc[c];
    uint8_t status;
    if (nr == 0 && nc == 0) status = AABFT_BLK_CLEAN;
    else if (nr == 1 && nc == 1) status = AABFT_BLK_SINGLE;
    else if (nr == 0 || nc == 0) status = AABFT_BLK_CHECKSUM_ONLY;
    else status = AABFT_BLK_UNCORRECTABLE;
    aabft_block_report rep;
    rep.status = status;
    rep.worst_class = (uint8_t)s_worst[c];
    rep.n_bad_rows = (uint16_t)min(nr, 65535);
    rep.n_bad_cols = (uint16_t)min(nc, 65535);
    rep.reserved = 0;
    rep.row = status == AABFT_BLK_SINGLE ? s_row[c] : -1;
    rep.col = status == AABFT_BLK_SINGLE ? s_col[c] : -1;
    mr = __uint_as_float(s_rmax[c]);
    rep.max_ratio = mr;
    rep.status = maybe_correct<T, P, EXT>(a, bp, status, I * nJ + j0 / bs + c, rep.row, rep.col);
    a.rep[I * nJ + j0 / bs + c] = rep;
    my_n[0] = 1;
    my_n[1] = status == AABFT_BLK_CLEAN;
    my_n[2] = rep.status == AABFT_BLK_CORRECTED;
    my_n[3] = status == AABFT_BLK_CHECKSUM_ONLY;
    my_n[4] = rep.status == AABFT_BLK_UNCORRECTABLE;
  }
  my_n[5] = cls_tot[0]; my_n[6] = cls_tot[1]; my_n[7] = cls_tot[2];
#pragma unroll
  for (int k = 0; k < 8; ++k) {
#pragma unroll
    for (int m = 16; m >= 1; m >>= 1) my_n[k] += __shfl_xor_sync(0xffffffffu, my_n[k], m);
  }
#pragma unroll
  for (int m = 16; m >= 1; m >>= 1) mr = fmaxf(mr, __shfl_xor_sync(0xffffffffu, mr, m));
  if (lane == 0) {
    for (int k = 0; k < 8; ++k)
      if (my_n[k]) atomicAdd(&s_n[k], my_n[k]);
    if (mr > 0.f) atomicMax(&s_mr, __float_as_uint(mr));
  }
  __syncthreads();
  publish_counts(a, s_n, s_mr, c);
}

// --------------------------------------------------------------------------- correct
template <typename T, int P, bool EXT>
__global__ void correct_kernel(CheckArgs a, BoundParams bp, T *C) {
  const int bs = a.bs;
  const int64_t nJ = a.N / bs, nb = (a.M / bs) * nJ;
  for (int64_t blk = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; blk < nb;
       blk += (int64_t)gridDim.x * blockDim.x) {
    aabft_block_report *r = a.rep + blk;
    if (r->status != AABFT_BLK_SINGLE) continue;
    const uint8_t st = correct_block<T, P, EXT>(a, bp, C, blk, r->row, r->col);
    r->status = st;
    unsigned long long *n = reinterpret_cast<unsigned long long *>(a.cnt->n);
    atomicAdd(&n[st == AABFT_BLK_CORRECTED ? 2 : 4], 1ull);
  }
}

CheckArgs make_args(const aabft_config *cfg, const aabft_encoded *enc, const aabft_product *prod,
                    aabft_block_report *rep, aabft_counts *cnt, void *gemm_ws = nullptr) {
  CheckArgs a;
  a.M = cfg->M; a.N = cfg->N; a.bs = cfg->bs;
  a.C = prod->C; a.ldc = prod->ldc;
  a.Ccol = prod->Ccol; a.ld_ccol = prod->ld_ccol;
  a.Crow = prod->Crow; a.ld_crow = prod->ld_crow;
  a.tav = enc ? enc->topA_val : nullptr; a.tai = enc ? enc->topA_idx : nullptr;
  a.tbv = enc ? enc->topB_val : nullptr; a.tbi = enc ? enc->topB_idx : nullptr;
  a.rep = rep; a.cnt = cnt;
  // fused reference sums exist only where aabft_gemm produces them (FP64, bs <= 64)
  const bool fused = prod->Rcol && prod->Rrow && fused_check_ok(cfg);
  a.Rcol = fused && gemm_ws ? prod->Rcol : nullptr;
  a.Rrow = fused && gemm_ws ? prod->Rrow : nullptr;
  a.Rcol2 = a.Rrow2 = nullptr;
  a.col_parts = a.row_parts = 1;
  a.eps_col = a.eps_row = nullptr;
  a.eps_fixed = 0.0;
  a.acc = nullptr;
  a.correct = (cfg->flags & AABFT_FLAG_CHECK_CORRECTS) ? 1 : 0;
  if (a.Rcol && cfg->dtype == AABFT_F64) {  // the FP32 epilogue always completes its sums
    a.col_parts = gemm_f64_fused_parts(cfg->bs, &a.row_parts);
    double *rc2, *rr2;
    gemm_f64_red_ptrs(cfg, gemm_ws, &rc2, &rr2);
    a.Rcol2 = rc2;
    a.Rrow2 = rr2;
  }
  return a;
}

// correction: the fused reference sums (complete after aabft_check) are refreshed for every
// corrected element (a second check of a corrected product must stay clean)
void set_refresh(const aabft_config *cfg, const aabft_product *prod, CheckArgs &a) {
  const bool fused = prod->Rcol && prod->Rrow && fused_check_ok(cfg);
  a.Rcol = fused ? prod->Rcol : nullptr;
  a.Rrow = fused ? prod->Rrow : nullptr;
}

template <typename T, int P, bool EXT = false>
aabft_status run_check(const aabft_config *cfg, const CheckArgs &a, BoundParams bp,
                       cudaStream_t st) {
  const int64_t nb = (cfg->M / cfg->bs) * (cfg->N / cfg->bs);
  if (nb > 0) {
    if (a.Rcol && a.Rrow) {
      // units of JB = 256/bs adjacent blocks of one block-row (bs <= 64 => JB >= 4)
      const int JB = kFusedThreads / cfg->bs;
      const int64_t ngrp = (cfg->N / cfg->bs + JB - 1) / JB;
      const int64_t nunits = (cfg->M / cfg->bs) * ngrp;
      // one wave of co-resident CTAs (per device and instantiation, computed once)
      static std::atomic<int> resident_dev[64];
      int dev = 0;
      cudaGetDevice(&dev);
      int resident = resident_dev[dev & 63].load(std::memory_order_relaxed);
      if (!resident) {
        int sms = 0, per_sm = 0;
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, check_fused_kernel<T, P, EXT>,
                                                      kFusedThreads, 0);
        resident = std::max(1, sms * (AABFT_CHECK_CTAS > 0 ? AABFT_CHECK_CTAS : std::max(1, per_sm)));
        resident_dev[dev & 63].store(resident, std::memory_order_relaxed);
      }
      const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(nunits, resident));
      check_fused_kernel<T, P, EXT><<<grid, kFusedThreads, 0, st>>>(a, bp, nunits, (int)ngrp);
    } else if (cfg->bs <= 128) {
      dim3 grid((unsigned)((cfg->N + 127) / 128), (unsigned)(cfg->M / cfg->bs));
      check_stream_kernel<T, P, EXT, 128><<<grid, 128, 0, st>>>(a, bp);
    } else {
      dim3 grid((unsigned)((cfg->N + 255) / 256), (unsigned)(cfg->M / cfg->bs));
      check_stream_kernel<T, P, EXT, 256><<<grid, 256, 0, st>>>(a, bp);
    }
    next_launch();
  }
  return check_launch("aabft_check");
}

template <typename T, int P, bool EXT = false>
aabft_status run_correct(const aabft_config *cfg, const CheckArgs &a, BoundParams bp,
                         cudaStream_t st) {
  const int64_t nb = (cfg->M / cfg->bs) * (cfg->N / cfg->bs);
  const unsigned grid = (unsigned)std::min<int64_t>((nb + 255) / 256, 4096);
  if (nb > 0) {
    correct_kernel<T, P, EXT><<<grid, 256, 0, st>>>(a, bp, static_cast<T *>(const_cast<void *>(a.C)));
    next_launch();
  }
  return check_launch("aabft_correct");
}

#define AABFT_P_SWITCH(p, ...)          \
  switch (p) {                           \
    case 1: { constexpr int PP = 1; __VA_ARGS__; } \
    case 2: { constexpr int PP = 2; __VA_ARGS__; } \
    case 3: { constexpr int PP = 3; __VA_ARGS__; } \
    case 4: { constexpr int PP = 4; __VA_ARGS__; } \
    case 5: { constexpr int PP = 5; __VA_ARGS__; } \
    case 6: { constexpr int PP = 6; __VA_ARGS__; } \
    case 7: { constexpr int PP = 7; __VA_ARGS__; } \
    case 8: { constexpr int PP = 8; __VA_ARGS__; } \
  }

}  // namespace

// sum of per-part counters (SUM n[8], MAX max_ratio) -- used by the pipelined host entry point
__global__ void counts_sum_kernel(const aabft_counts *parts, int n, aabft_counts *out) {
  const int t = threadIdx.x;
  if (t < 8) {
    long long v = 0;
    for (int i = 0; i < n; ++i) v += parts[i].n[t];
    out->n[t] = v;
  } else if (t == 8) {
    double m = 0.0;
    for (int i = 0; i < n; ++i) m = fmax(m, parts[i].max_ratio);
    out->max_ratio = m;
  }
}

aabft_status launch_counts_sum(const aabft_counts *parts, int n, aabft_counts *out, cudaStream_t st) {
  counts_sum_kernel<<<1, 32, 0, st>>>(parts, n, out);
  next_launch();
  return check_launch("counts sum");
}

aabft_status launch_bound(const aabft_config *cfg, const aabft_encoded *enc, double *eps_col,
                          double *sig_col, double *eps_row, double *sig_row, cudaStream_t st) {
  const BoundParams bp = make_bound_params(cfg);
  const int64_t n = (cfg->M / cfg->bs) * cfg->N + cfg->M * (cfg->N / cfg->bs);
  const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((n + 255) / 256, 148 * 16));
  AABFT_P_SWITCH(cfg->p, {
    bound_kernel<PP><<<grid, 256, 0, st>>>(cfg->M, cfg->N, cfg->bs, bp, enc->topA_val,
                                           enc->topA_idx, enc->topB_val, enc->topB_idx, eps_col,
                                           sig_col, eps_row, sig_row);
    next_launch();
    return check_launch("aabft_bound");
  });
  set_error("p out of range");
  return AABFT_EINVAL;
}

aabft_status launch_bound_elements(const aabft_config *cfg, const aabft_encoded *enc,
                                   const int64_t *rows, const int64_t *cols, int64_t n,
                                   double *sig, double *eps, cudaStream_t st) {
  const BoundParams bp = make_bound_params(cfg);
  if (n <= 0) return AABFT_OK;
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, 148 * 16);
  AABFT_P_SWITCH(cfg->p, {
    bound_elements_kernel<PP><<<grid, 256, 0, st>>>(cfg->M, cfg->N, cfg->bs, bp, enc->topA_val,
                                                    enc->topA_idx, enc->topB_val, enc->topB_idx,
                                                    rows, cols, n, sig, eps);
    next_launch();
    return check_launch("aabft_bound_elements");
  });
  set_error("p out of range");
  return AABFT_EINVAL;
}

aabft_status launch_check(const aabft_config *cfg, const aabft_encoded *enc,
                          const aabft_product *prod, aabft_block_report *rep, aabft_counts *cnt,
                          void *gemm_ws, unsigned long long *acc, cudaStream_t st) {
  const BoundParams bp = make_bound_params(cfg);
  CheckArgs a = make_args(cfg, enc, prod, rep, cnt, gemm_ws);
  a.acc = acc;
  if (!acc && cudaMemsetAsync(cnt, 0, sizeof(aabft_counts), st) != cudaSuccess)
    return check_launch("aabft_check memset");
  if (cfg->dtype == AABFT_F64) {
    AABFT_P_SWITCH(cfg->p, return (run_check<double, PP>(cfg, a, bp, st)));
  } else {
    AABFT_P_SWITCH(cfg->p, return (run_check<float, PP>(cfg, a, bp, st)));
  }
  set_error("p out of range");
  return AABFT_EINVAL;
}

aabft_status launch_correct(const aabft_config *cfg, const aabft_encoded *enc,
                            const aabft_product *prod, aabft_block_report *rep,
                            aabft_counts *cnt, cudaStream_t st) {
  const BoundParams bp = make_bound_params(cfg);
  CheckArgs a = make_args(cfg, enc, prod, rep, cnt);
  set_refresh(cfg, prod, a);
  if (cfg->dtype == AABFT_F64) {
    AABFT_P_SWITCH(cfg->p, return (run_correct<double, PP>(cfg, a, bp, st)));
  } else {
    AABFT_P_SWITCH(cfg->p, return (run_correct<float, PP>(cfg, a, bp, st)));
  }
  set_error("p out of range");
  return AABFT_EINVAL;
}

// check / correct against an external eps (NEXT-3 comparators: SEA-ABFT bound, fixed-eps ABFT;
// reading R26).  The top-p tables are not used; P = 1 instantiations.
aabft_status launch_check_ext(const aabft_config *cfg, const aabft_product *prod,
                              const double *eps_col, const double *eps_row, double eps_fixed,
                              aabft_block_report *rep, aabft_counts *cnt, void *gemm_ws,
                              unsigned long long *acc, cudaStream_t st) {
  const BoundParams bp = make_bound_params(cfg);
  CheckArgs a = make_args(cfg, nullptr, prod, rep, cnt, gemm_ws);
  a.eps_col = eps_col;
  a.eps_row = eps_row;
  a.eps_fixed = eps_fixed;
  a.acc = acc;
  if (!acc && cudaMemsetAsync(cnt, 0, sizeof(aabft_counts), st) != cudaSuccess)
    return check_launch("aabft_check_ext memset");
  if (cfg->dtype == AABFT_F64) return run_check<double, 1, true>(cfg, a, bp, st);
  return run_check<float, 1, true>(cfg, a, bp, st);
}

aabft_status launch_correct_ext(const aabft_config *cfg, const aabft_product *prod,
                                const double *eps_row, double eps_fixed, aabft_block_report *rep,
                                aabft_counts *cnt, cudaStream_t st) {
  const BoundParams bp = make_bound_params(cfg);
  CheckArgs a = make_args(cfg, nullptr, prod, rep, cnt);
  set_refresh(cfg, prod, a);
  a.eps_row = eps_row;
  a.eps_fixed = eps_fixed;
  if (cfg->dtype == AABFT_F64) return run_correct<double, 1, true>(cfg, a, bp, st);
  return run_correct<float, 1, true>(cfg, a, bp, st);
}

}  // namespace aabft
