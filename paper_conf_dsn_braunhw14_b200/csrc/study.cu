// study.cu -- NEXT-1: the exact rounding error of every carried checksum, for the
// paper's bound-quality experiment (§VI-B, Tables II/III: "the determined rounding
// error bounds are compared against exact rounding errors that have been computed using GMP").
//
// Instead of GMP on the host, the exact inner products of the checksum vectors are formed on
// the GPU in double-double: TwoProd via FMA (p = a*b, e = fma(a, b, -p) exactly) and a
// compensated (TwoSum) accumulation -- the Dot2 scheme of Ogita, Rump and Oishi, which is as
// accurate as an inner product in twice the working precision (relative error ~2^-104 * cond),
// far below the FP64 rounding errors being measured (~2^-52 * K).  One thread per checksum
// element; the per-element loads are coalesced along j (Ccol) or broadcast (Crow).
#include <algorithm>

#include "common.cuh"

namespace aabft {
namespace {

__device__ __forceinline__ void two_sum(double a, double b, double &s, double &e) {
  s = __dadd_rn(a, b);
  const double bb = __dsub_rn(s, a);
  e = __dadd_rn(__dsub_rn(a, __dsub_rn(s, bb)), __dsub_rn(b, bb));
}

// exact-ish dot product of x (stride sx) and y (stride sy), length K, in double-double
template <typename T>
__device__ __forceinline__ void dot2(const T *x, int64_t sx, const T *y, int64_t sy, int64_t K,
                                     double &hi, double &lo) {
  double s = 0.0, c = 0.0;
  for (int64_t k = 0; k < K; ++k) {
    const double a = (double)x[k * sx], b = (double)y[k * sy];
    const double p = __dmul_rn(a, b);
    const double pe = __fma_rn(a, b, -p);  // exact product error
    double t, te;
    two_sum(s, p, t, te);
    s = t;
    c = __dadd_rn(c, __dadd_rn(te, pe));
  }
  two_sum(s, c, hi, lo);
}

// err_col[I][j] = carried Ccol[I][j] - exact(Acs[I] . B[:, j]); err_row[i][J] likewise for Crow.
template <typename T>
__global__ void checksum_error_kernel(int64_t M, int64_t N, int64_t K, int bs, const T *A,
                                      int64_t lda, const T *B, int64_t ldb, const T *Acs,
                                      int64_t ld_acs, const T *Bcs, int64_t ld_bcs, const T *Ccol,
                                      int64_t ld_ccol, const T *Crow, int64_t ld_crow,
                                      double *err_col, double *err_row) {
  const int64_t ncol = (M / bs) * N, nrow = M * (N / bs);
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < ncol + nrow;
       e += (int64_t)gridDim.x * blockDim.x) {
    double hi, lo;
    if (e < ncol) {
      const int64_t I = e / N, j = e % N;
      dot2<T>(Acs + I * ld_acs, 1, B + j, ldb, K, hi, lo);
      const double carried = (double)Ccol[I * ld_ccol + j];
      err_col[e] = __dsub_rn(__dsub_rn(carried, hi), lo);
    } else {
      const int64_t f = e - ncol, nJ = N / bs, i = f / nJ, J = f % nJ;
      dot2<T>(A + i * lda, 1, Bcs + J, ld_bcs, K, hi, lo);
      const double carried = (double)Crow[i * ld_crow + J];
      err_row[f] = __dsub_rn(__dsub_rn(carried, hi), lo);
    }
  }
}

}  // namespace

aabft_status launch_checksum_errors(const aabft_config *cfg, const void *A, int64_t lda,
                                    const void *B, int64_t ldb, const aabft_encoded *enc,
                                    const aabft_product *prod, double *err_col, double *err_row,
                                    cudaStream_t st) {
  const int64_t n = (cfg->M / cfg->bs) * cfg->N + cfg->M * (cfg->N / cfg->bs);
  const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((n + 127) / 128, 148 * 32));
  if (cfg->dtype == AABFT_F64)
    checksum_error_kernel<double><<<grid, 128, 0, st>>>(
        cfg->M, cfg->N, cfg->K, cfg->bs, static_cast<const double *>(A), lda,
        static_cast<const double *>(B), ldb, static_cast<const double *>(enc->Acs), enc->ld_acs,
        static_cast<const double *>(enc->Bcs), enc->ld_bcs, static_cast<const double *>(prod->Ccol),
        prod->ld_ccol, static_cast<const double *>(prod->Crow), prod->ld_crow, err_col, err_row);
  else
    checksum_error_kernel<float><<<grid, 128, 0, st>>>(
        cfg->M, cfg->N, cfg->K, cfg->bs, static_cast<const float *>(A), lda,
        static_cast<const float *>(B), ldb, static_cast<const float *>(enc->Acs), enc->ld_acs,
        static_cast<const float *>(enc->Bcs), enc->ld_bcs, static_cast<const float *>(prod->Ccol),
        prod->ld_ccol, static_cast<const float *>(prod->Crow), prod->ld_crow, err_col, err_row);
  next_launch();
  return check_launch("aabft_checksum_errors");
}

}  // namespace aabft
