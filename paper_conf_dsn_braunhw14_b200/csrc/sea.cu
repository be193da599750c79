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
// "vector norms use only a small fraction of the available GPU threads").  The chain
// stays one thread per vector; the loads feeding it are spread over 256-thread CTAs of 16
// vectors each (sea_norm_kernel), so the ~260 CTAs cover every SM with 32 KiB in flight.
#include <algorithm>

#include "common.cuh"

namespace aabft {
namespace {

// ||x||_2 of R0 + R1 vectors of length L, 16 vectors per 256-thread CTA.  ROWS: vector r is
// row r of a row-major matrix (X0 for r < R0, then X1); else vector c is column c.  The CTA
// stages a 16 x 128 tile of the vectors in shared memory with coalesced loads from all 8 warps
// (ROWS: a warp reads 32 consecutive k of one row; columns: a half-warp reads 16 consecutive
// columns of one k-row), the next tile's loads are in flight in registers while lanes 0..15 of
// warp 0 add their vector's 128 squares in ascending k -- the sequential chain of the
// definition, bit-identical to the oracle (zero padding past L adds +0 to a sum >= 0, exact).
constexpr int kSeaVec = 16, kSeaTile = 128, kSeaThreads = 256;
constexpr int kSeaPer = kSeaVec * kSeaTile / kSeaThreads;  // elements per thread per tile

template <typename T, bool ROWS>
__global__ void __launch_bounds__(kSeaThreads) sea_norm_kernel(const T *__restrict__ X0,
                                                               int64_t ld0, int64_t R0,
                                                               const T *__restrict__ X1,
                                                               int64_t ld1, int64_t R1, int64_t L,
                                                               double *__restrict__ out) {
  __shared__ double tile[2][kSeaVec][kSeaTile + 1];  // stride 129: conflict-free per-vector reads
  const int t = threadIdx.x;
  const int64_t v0 = (int64_t)blockIdx.x * kSeaVec;
  // this thread's kSeaPer (vector, k) slots of a tile and the base pointer of each
  const T *base[kSeaPer];
  int64_t step[kSeaPer];  // element stride along k
  int sv[kSeaPer], sk[kSeaPer];
  bool ok[kSeaPer];
#pragma unroll
  for (int e = 0; e < kSeaPer; ++e) {
    const int idx = t + kSeaThreads * e;
    sv[e] = ROWS ? idx / kSeaTile : idx % kSeaVec;
    sk[e] = ROWS ? idx % kSeaTile : idx / kSeaVec;
    const int64_t v = v0 + sv[e];
    ok[e] = v < R0 + R1;
    const bool first = v < R0;
    if (ROWS) {
      base[e] = ok[e] ? (first ? X0 + v * ld0 : X1 + (v - R0) * ld1) : X0;
      step[e] = 1;
    } else {
      base[e] = ok[e] ? (first ? X0 + v : X1 + (v - R0)) : X0;
      step[e] = first ? ld0 : ld1;
    }
  }
  double regs[kSeaPer];
  auto load = [&](int64_t k0) {
#pragma unroll
    for (int e = 0; e < kSeaPer; ++e) {
      const int64_t k = k0 + sk[e];
      regs[e] = (ok[e] && k < L) ? (double)__ldg(base[e] + k * step[e]) : 0.0;
    }
  };
  const int nt = (int)((L + kSeaTile - 1) / kSeaTile);
  double s = 0.0;
  load(0);
  for (int it = 0; it < nt; ++it) {
    double(*buf)[kSeaTile + 1] = tile[it & 1];
#pragma unroll
    for (int e = 0; e < kSeaPer; ++e) buf[sv[e]][sk[e]] = regs[e];
    __syncthreads();  // also orders warp 0's reads of tile[it & 1] two tiles ago before this store
    if (it + 1 < nt) load((int64_t)(it + 1) * kSeaTile);
    if (t < kSeaVec) {
#pragma unroll 16
      for (int k = 0; k < kSeaTile; ++k) {
        const double d = buf[t][k];
        s = __dadd_rn(s, __dmul_rn(d, d));  // ascending k
      }
    }
  }
  if (t < kSeaVec && v0 + t < R0 + R1) out[v0 + t] = __dsqrt_rn(s);
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
  sea_norm_kernel<T, true><<<(unsigned)((M + nI + kSeaVec - 1) / kSeaVec), kSeaThreads, 0, st>>>(
      A, lda, M, static_cast<const T *>(enc->Acs), enc->ld_acs, nI, K, nA);
  sea_norm_kernel<T, false><<<(unsigned)((N + nJ + kSeaVec - 1) / kSeaVec), kSeaThreads, 0, st>>>(
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
