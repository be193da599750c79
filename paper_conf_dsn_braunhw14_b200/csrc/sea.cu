// sea.cu -- the SEA-ABFT comparator bound (NEXT-3, reporting only) on sm_100a.
//
// §III P:L109-115 (simplified error analysis of ref [28]) for the column checksum of an
// (m+1) x n column-checksum matrix A times a column b:
//   |c_{n+1} - c*_{n+1}| < ((n + 2m - 2) ||b||_2 sum_{i=1..m} ||a_i||_2 + n ||a_{m+1}||_2 ||b||_2) eps_M
// with partitioned encoding: m = bs rows of block-row I, a_{m+1} = Acs[I], b = column j
// of B, n = K; the row checksum (i, J) is the transposed statement and the corner (I, J) uses
// Acs[I] and Bcs[:, J] (reading R25).  ||x||_2 = sqrt of the sequential ascending sum of x_k^2
// in double (separately rounded products), so every norm and every eps is bit-identical to the
// definition -- the oracle's O11 -- with explicit round-to-nearest intrinsics (no contraction).
//
// Work: the norms read A, B (and the small Acs, Bcs) once: M*K + K*N elements, HBM-bound in
// principle but each norm is one sequential dependency chain of K double adds (the paper's
// "vector norms use only a small fraction of the available GPU threads").  Rows are
// one thread each with 16-byte vector loads (each thread's row stays in L1 across its
// iterations); columns are one thread each with coalesced row-segment loads.
#include <algorithm>

#include "common.cuh"

namespace aabft {
namespace {

// ||row r||_2 for R rows of an R x L row-major matrix (two matrices per launch: A then Acs)
template <typename T>
__global__ void __launch_bounds__(128) sea_norm_rows_kernel(const T *__restrict__ X0, int64_t ld0,
                                                            int64_t R0, const T *__restrict__ X1,
                                                            int64_t ld1, int64_t R1, int64_t L,
                                                            double *__restrict__ out) {
  const int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (r >= R0 + R1) return;
  const T *x = r < R0 ? X0 + r * ld0 : X1 + (r - R0) * ld1;
  double s = 0.0;
  constexpr int V = 16 / sizeof(T);  // elements per 16-byte load (rows are 16-B aligned)
  int64_t k = 0;
  for (; k + 4 * V <= L; k += 4 * V) {
    T v[4 * V];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      if constexpr (V == 2) {
        const double2 q = __ldg(reinterpret_cast<const double2 *>(x + k) + u);
        v[u * V] = (T)q.x; v[u * V + 1] = (T)q.y;
      } else {
        const float4 q = __ldg(reinterpret_cast<const float4 *>(x + k) + u);
        v[u * V] = (T)q.x; v[u * V + 1] = (T)q.y; v[u * V + 2] = (T)q.z; v[u * V + 3] = (T)q.w;
      }
    }
#pragma unroll
    for (int e = 0; e < 4 * V; ++e) {
      const double d = (double)v[e];
      s = __dadd_rn(s, __dmul_rn(d, d));  // ascending k
    }
  }
  for (; k < L; ++k) {
    const double d = (double)__ldg(x + k);
    s = __dadd_rn(s, __dmul_rn(d, d));
  }
  out[r] = __dsqrt_rn(s);
}

// ||column c||_2 for the C0 columns of X0 (L x C0) then the C1 columns of X1 (L x C1)
template <typename T>
__global__ void __launch_bounds__(128) sea_norm_cols_kernel(const T *__restrict__ X0, int64_t ld0,
                                                            int64_t C0, const T *__restrict__ X1,
                                                            int64_t ld1, int64_t C1, int64_t L,
                                                            double *__restrict__ out) {
  const int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (c >= C0 + C1) return;
  const T *x = c < C0 ? X0 + c : X1 + (c - C0);
  const int64_t ld = c < C0 ? ld0 : ld1;
  double s = 0.0;
  int64_t k = 0;
  for (; k + 8 <= L; k += 8) {
    T v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = __ldg(x + (k + u) * ld);
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const double d = (double)v[u];
      s = __dadd_rn(s, __dmul_rn(d, d));
    }
  }
  for (; k < L; ++k) {
    const double d = (double)__ldg(x + k * ld);
    s = __dadd_rn(s, __dmul_rn(d, d));
  }
  out[c] = __dsqrt_rn(s);
}

// SA[I] = sum of the bs row norms of block-row I, SB[J] likewise (sequential ascending)
__global__ void sea_block_sums_kernel(const double *__restrict__ nA, int64_t nI,
                                      const double *__restrict__ nB, int64_t nJ, int bs,
                                      double *__restrict__ SA, double *__restrict__ SB) {
  const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (t < nI) {
    double s = 0.0;
    for (int64_t i = t * bs; i < t * bs + bs; ++i) s = __dadd_rn(s, nA[i]);
    SA[t] = s;
  } else if (t < nI + nJ) {
    const int64_t J = t - nI;
    double s = 0.0;
    for (int64_t j = J * bs; j < J * bs + bs; ++j) s = __dadd_rn(s, nB[j]);
    SB[J] = s;
  }
}

// eps = ((c1 * ||b||) * S + (n * ||a_{m+1}||) * ||b||) * 2^-t, c1 = n + 2m - 2 (host-evaluated)
__device__ __forceinline__ double sea_eps(double c1, double n, double nb, double S, double ncs,
                                          int t) {
  return ldexp(__dadd_rn(__dmul_rn(__dmul_rn(c1, nb), S), __dmul_rn(__dmul_rn(n, ncs), nb)), -t);
}

__global__ void sea_eps_kernel(int64_t M, int64_t N, int bs, double c1, double n, int t,
                               const double *__restrict__ nA, const double *__restrict__ nAcs,
                               const double *__restrict__ nB, const double *__restrict__ nBcs,
                               const double *__restrict__ SA, const double *__restrict__ SB,
                               double *eps_col, double *eps_row, double *eps_corner) {
  const int64_t nI = M / bs, nJ = N / bs;
  const int64_t ncol = eps_col ? nI * N : 0, nrow = eps_row ? M * nJ : 0;
  const int64_t ncor = eps_corner ? nI * nJ : 0;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < ncol + nrow + ncor;
       e += (int64_t)gridDim.x * blockDim.x) {
    if (e < ncol) {  // column checksum (I, j): rows of block-row I, Acs[I], column j of B
      const int64_t I = e / N, j = e % N;
      eps_col[e] = sea_eps(c1, n, nB[j], SA[I], nAcs[I], t);
    } else if (e < ncol + nrow) {  // row checksum (i, J): columns of block J, Bcs[:, J], row i
      const int64_t f = e - ncol, i = f / nJ, J = f % nJ;
      eps_row[f] = sea_eps(c1, n, nA[i], SB[J], nBcs[J], t);
    } else {  // corner (I, J): Acs[I] and Bcs[:, J] (reading R25)
      const int64_t f = e - ncol - nrow, I = f / nJ, J = f % nJ;
      eps_corner[f] = sea_eps(c1, n, nBcs[J], SA[I], nAcs[I], t);
    }
  }
}

template <typename T>
aabft_status run_sea(const aabft_config *cfg, const T *A, int64_t lda, const T *B, int64_t ldb,
                     const aabft_encoded *enc, double *eps_col, double *eps_row,
                     double *eps_corner, void *ws, cudaStream_t st) {
  const int64_t M = cfg->M, N = cfg->N, K = cfg->K, bs = cfg->bs, nI = M / bs, nJ = N / bs;
  double *nA = static_cast<double *>(ws);  // M + nI: rows of A, then rows of Acs
  double *nB = nA + (M + nI);               // N + nJ: columns of B, then columns of Bcs
  double *SA = nB + (N + nJ);
  double *SB = SA + nI;
  sea_norm_rows_kernel<T><<<(unsigned)((M + nI + 127) / 128), 128, 0, st>>>(
      A, lda, M, static_cast<const T *>(enc->Acs), enc->ld_acs, nI, K, nA);
  sea_norm_cols_kernel<T><<<(unsigned)((N + nJ + 127) / 128), 128, 0, st>>>(
      B, ldb, N, static_cast<const T *>(enc->Bcs), enc->ld_bcs, nJ, K, nB);
  sea_block_sums_kernel<<<(unsigned)((nI + nJ + 127) / 128), 128, 0, st>>>(nA, nI, nB, nJ,
                                                                           (int)bs, SA, SB);
  const double n = (double)K;
  const double c1 = (double)K + 2.0 * (double)bs - 2.0;  // n + 2m - 2
  const int64_t tot = (eps_col ? nI * N : 0) + (eps_row ? M * nJ : 0) + (eps_corner ? nI * nJ : 0);
  const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((tot + 255) / 256, 148 * 16));
  sea_eps_kernel<<<grid, 256, 0, st>>>(M, N, (int)bs, c1, n, eff_t(cfg), nA, nA + M, nB, nB + N,
                                       SA, SB, eps_col, eps_row, eps_corner);
  next_launch(4);
  return check_launch("aabft_sea_bound");
}

}  // namespace

size_t sea_ws_bytes(const aabft_config *cfg) {
  const int64_t nI = cfg->M / cfg->bs, nJ = cfg->N / cfg->bs;
  return (size_t)(cfg->M + nI + cfg->N + nJ + nI + nJ) * sizeof(double);
}

aabft_status launch_sea_bound(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                              int64_t ldb, const aabft_encoded *enc, double *eps_col,
                              double *eps_row, double *eps_corner, void *ws, cudaStream_t st) {
  if (cfg->dtype == AABFT_F64)
    return run_sea<double>(cfg, static_cast<const double *>(A), lda,
                           static_cast<const double *>(B), ldb, enc, eps_col, eps_row,
                           eps_corner, ws, st);
  return run_sea<float>(cfg, static_cast<const float *>(A), lda, static_cast<const float *>(B),
                        ldb, enc, eps_col, eps_row, eps_corner, ws, st);
}

}  // namespace aabft
