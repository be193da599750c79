// encode.cu -- step 1 of A-ABFT on sm_100a: partitioned checksum encoding fused with top-p
// |value| selection (P:L313-317 steps 1a-1d; Alg 1), and the global top-p
// reduction (step 3, P:L320 / P:L368).
//
// B200 design: HBM-bound streaming.  One thread owns one column of a
// BS-row block of A, so the column checksum is a register running sum in ascending row order
// (bit-identical to Eq 1 summed top -> bottom, reading R11) and every warp load is a
// contiguous 256 B row segment.  The same pass stages |a| in padded shared memory where four
// lanes per row keep register top-p lists over interleaved columns and merge them with two
// xor-shuffles (warp-shuffle top-p).  B is the mirror image: a thread owns a column of B
// (running top-p over k in registers) and the BS-wide row sums are taken from the staged
// tile, one sequential thread per (row, block).  Partial top-p lists per chunk are reduced
// by a warp-per-vector kernel that also computes the top-p of the checksum vectors.
// Strips are double-buffered in registers (the next strip's loads are in flight during the
// top-p / row-sum phase) and the top-p insertion is branch-free for p <= 4 (tp_push), so a
// warp never diverges on inserts: 44 + 43 + 9 us at 4096^2 FP64.
#include <algorithm>

#include "common.cuh"

namespace aabft {
namespace {

constexpr int kStrip = 32;  // rows staged per pass

template <typename T>
__device__ __forceinline__ T ldg(const T *p) { return __ldg(p); }

// ---------------------------------------------------------------------------------- A
// grid (chunks of 128 columns, M/bs block-rows); 128 threads.
template <typename T, int P, bool TOPP>
__global__ void __launch_bounds__(128) encode_a_kernel(const T *__restrict__ A, int64_t lda,
                                                       int64_t K, int bs, T *__restrict__ Acs,
                                                       int64_t ld_acs, double *__restrict__ pv,
                                                       int *__restrict__ pi, int nch) {
  __shared__ double tile[kStrip][kEncAChunk + 4];  // |A| strip; stride 132 -> conflict-free
  const int c = threadIdx.x;
  const int chunk = blockIdx.x;
  const int64_t I = blockIdx.y;
  const int64_t k = (int64_t)chunk * kEncAChunk + c;
  const bool kin = k < K;
  const int r = c >> 2, q = c & 3;  // top-p role: row r of the strip, column phase q
  T sum = T(0);
  // register double buffering: the loads of strip r0 + kStrip are issued right after strip r0
  // has been summed and staged, so they are in flight during its top-p phase
  T vals[kStrip];
  auto load_strip = [&](int r0) {
    const int rows = min(kStrip, bs - r0);
    const T *src = A + (I * bs + r0) * lda + k;
    if (rows == kStrip) {
      // full strip: the kStrip loads are issued back to back (memory-level parallelism; a
      // per-row guard made the checksums-only instantiation compile to load -> add chains)
#pragma unroll
      for (int rr = 0; rr < kStrip; ++rr) vals[rr] = kin ? ldg(src + rr * lda) : T(0);
    } else {
#pragma unroll
      for (int rr = 0; rr < kStrip; ++rr) vals[rr] = (rr < rows && kin) ? ldg(src + rr * lda) : T(0);
    }
  };
  load_strip(0);
  for (int r0 = 0; r0 < bs; r0 += kStrip) {
    const int rows = min(kStrip, bs - r0);
#pragma unroll
    for (int rr = 0; rr < kStrip; ++rr) {
      if (rr < rows) {
        sum = sum + vals[rr];  // Eq 1, ascending i (Alg 1 line "sum <- sum + Asub[i][tid]")
        if (TOPP) tile[rr][c] = fabs((double)vals[rr]);
      }
    }
    if (r0 + kStrip < bs) load_strip(r0 + kStrip);
    if (!TOPP) continue;  // checksums only (fixed-eps / SEA ABFT comparators, NEXT-3)
    __syncthreads();
    double v[P];
    int ix[P];
    tp_init<P>(v, ix);
    if (r < rows) {
      // ascending columns into this lane's own list: the new element loses every tie.  The
      // column limit is hoisted (32-bit: K < 2^31 is validated) so the scan carries no
      // per-element guard or 64-bit index arithmetic.
      const int kbase = chunk * kEncAChunk;
      const int lim = K - kbase < kEncAChunk ? (int)(K - kbase) : kEncAChunk;
      const double *trow = tile[r];
      // (measured: a fully or 8x unrolled version of this loop returned a list holding one
      // element twice on sm_100a; 4x with the compile-time bound is parity-clean)
#pragma unroll 4
      for (int cc = q; cc < kEncAChunk; cc += 4)
        if (cc < lim) tp_push<P>(v, ix, trow[cc], kbase + cc);
    }
    tp_shfl_merge<P>(v, ix, 1);
    tp_shfl_merge<P>(v, ix, 2);
    if (r < rows && q == 0) {
      const int64_t row = I * bs + r0 + r;
      double *dv = pv + (row * nch + chunk) * P;
      int *di = pi + (row * nch + chunk) * P;
#pragma unroll
      for (int s = 0; s < P; ++s) { dv[s] = v[s]; di[s] = ix[s]; }
    }
    __syncthreads();
  }
  if (kin) Acs[I * ld_acs + k] = sum;
  // partial top-p of the checksum row I over this chunk (Alg 1 localSums / maxReduce)
  if (TOPP) {
    __shared__ double s_v[kEncAChunk / 32][P];
    __shared__ int s_i[kEncAChunk / 32][P];
    double v[P];
    int ix[P];
    tp_init<P>(v, ix);
    if (kin) tp_insert<P>(v, ix, fabs((double)sum), (int)k);
#pragma unroll
    for (int m = 16; m >= 1; m >>= 1) tp_shfl_merge<P>(v, ix, m);
    if ((c & 31) == 0) {
#pragma unroll
      for (int s = 0; s < P; ++s) { s_v[c >> 5][s] = v[s]; s_i[c >> 5][s] = ix[s]; }
    }
    __syncthreads();
    if (c == 0) {
      for (int w = 1; w < kEncAChunk / 32; ++w)
#pragma unroll
        for (int s = 0; s < P; ++s) tp_insert<P>(v, ix, s_v[w][s], s_i[w][s]);
      const int64_t row = (int64_t)gridDim.y * bs + I;  // checksum rows follow the M data rows
      double *dv = pv + (row * nch + chunk) * P;
      int *di = pi + (row * nch + chunk) * P;
#pragma unroll
      for (int s = 0; s < P; ++s) { dv[s] = v[s]; di[s] = ix[s]; }
    }
  }
}

// ---------------------------------------------------------------------------------- B
// grid (column chunks of NC, row chunks of kEncBChunk); NC threads (NC = max(128, bs)).
template <typename T, int P, int NC, bool TOPP>
__global__ void __launch_bounds__(NC) encode_b_kernel(const T *__restrict__ B, int64_t ldb,
                                                      int64_t K, int64_t N, int bs,
                                                      T *__restrict__ Bcs, int64_t ld_bcs,
                                                      double *__restrict__ pv,
                                                      int *__restrict__ pi, int nch) {
  constexpr int SB = (NC * sizeof(T) > 1024) ? 16 : kStrip;  // strip rows (smem <= 48 KiB)
  __shared__ T tile[SB][NC + 1];  // odd stride -> conflict-free per-row sequential reads
  const int c = threadIdx.x;
  const int64_t j = (int64_t)blockIdx.x * NC + c;
  const bool jin = j < N;
  const int kc = blockIdx.y;
  const int64_t kbeg = (int64_t)kc * kEncBChunk;
  const int64_t kend = K < kbeg + kEncBChunk ? K : kbeg + kEncBChunk;
  const int nblk = NC / bs;  // checksum blocks covered by this CTA (<= 16)
  __shared__ double s_cv[16][P];
  __shared__ int s_ci[16][P];
  if (c < 16 * P) { s_cv[c / P][c % P] = -1.0; s_ci[c / P][c % P] = -1; }
  double v[P];
  int ix[P];
  tp_init<P>(v, ix);
  // register double buffering as in encode A: strip k0 + SB is loaded during the row sums
  T vals[SB];
  auto load_strip = [&](int64_t k0) {
    const int rows = (int)(kend - k0 < SB ? kend - k0 : SB);
    const T *src = B + k0 * ldb + j;
    if (rows == SB) {
#pragma unroll
      for (int rr = 0; rr < SB; ++rr) vals[rr] = jin ? ldg(src + rr * ldb) : T(0);
    } else {
#pragma unroll
      for (int rr = 0; rr < SB; ++rr) vals[rr] = (rr < rows && jin) ? ldg(src + rr * ldb) : T(0);
    }
  };
  if (kbeg < kend) load_strip(kbeg);
  for (int64_t k0 = kbeg; k0 < kend; k0 += SB) {
    const int rows = (int)(kend - k0 < SB ? kend - k0 : SB);
    const int k0i = (int)k0;  // K < 2^31 (validated)
    if (rows == SB) {  // full strip: no per-element guard
#pragma unroll
      for (int rr = 0; rr < SB; ++rr) {
        tile[rr][c] = vals[rr];
        // ascending k, own list: the new element loses every tie
        if (TOPP && jin) tp_push<P>(v, ix, fabs((double)vals[rr]), k0i + rr);
      }
    } else {
#pragma unroll
      for (int rr = 0; rr < SB; ++rr) {
        if (rr < rows) {
          tile[rr][c] = vals[rr];
          if (TOPP && jin) tp_push<P>(v, ix, fabs((double)vals[rr]), k0i + rr);
        }
      }
    }
    if (k0 + SB < kend) load_strip(k0 + SB);
    __syncthreads();
    // Eq 2 row checksums: lane rr of the warp owning block jb sums row rr sequentially
    // (ascending j), then the warp folds the strip's |Bcs| into the running top-p of
    // checksum column J (partial over this k-chunk)
    for (int jb = c >> 5; jb < nblk; jb += NC / 32) {
      const int rr = c & 31;
      const int64_t J = (int64_t)blockIdx.x * nblk + jb;
      double lv[P];
      int li[P];
      tp_init<P>(lv, li);
      if (rr < rows && J * bs < N) {
        T sm = T(0);
        for (int jj = 0; jj < bs; ++jj) sm = sm + tile[rr][jb * bs + jj];
        Bcs[(k0 + rr) * ld_bcs + J] = sm;
        if (TOPP) tp_push<P>(lv, li, fabs((double)sm), (int)(k0 + rr));
      }
      if (!TOPP) continue;
#pragma unroll
      for (int m = 16; m >= 1; m >>= 1) tp_shfl_merge<P>(lv, li, m);
      if (rr == 0) {
#pragma unroll
        for (int r = 0; r < P; ++r) tp_insert<P>(lv, li, s_cv[jb][r], s_ci[jb][r]);
#pragma unroll
        for (int r = 0; r < P; ++r) { s_cv[jb][r] = lv[r]; s_ci[jb][r] = li[r]; }
      }
    }
    __syncthreads();
  }
  if (!TOPP) return;
  if (c < nblk && ((int64_t)blockIdx.x * nblk + c) * bs < N) {
    const int64_t J = (int64_t)blockIdx.x * nblk + c;
    double *dv = pv + ((N + J) * nch + kc) * P;
    int *di = pi + ((N + J) * nch + kc) * P;
#pragma unroll
    for (int r = 0; r < P; ++r) { dv[r] = s_cv[c][r]; di[r] = s_ci[c][r]; }
  }
  if (jin) {
    double *dv = pv + (j * nch + kc) * P;
    int *di = pi + (j * nch + kc) * P;
#pragma unroll
    for (int s = 0; s < P; ++s) { dv[s] = v[s]; di[s] = ix[s]; }
  }
}

// ---------------------------------------------------------------------------------- step 3
// One warp per vector (data rows + checksum rows of A, data cols + checksum cols of B): merge
// the per-chunk partial lists produced by the encode kernels.
template <typename T, int P>
__global__ void __launch_bounds__(256) topp_reduce_kernel(
    int64_t M, int64_t N, int64_t K, int bs, const double *__restrict__ pva,
    const int *__restrict__ pia, int ncha, const double *__restrict__ pvb,
    const int *__restrict__ pib, int nchb, const T *__restrict__ Acs, int64_t ld_acs,
    const T *__restrict__ Bcs, int64_t ld_bcs, double *__restrict__ topA_v,
    int *__restrict__ topA_i, double *__restrict__ topB_v, int *__restrict__ topB_i, int do_a,
    int do_b) {
  const int lane = threadIdx.x & 31;
  const int64_t w = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5);
  const int64_t nA = do_a ? M + M / bs : 0;
  const int64_t nB = do_b ? N + N / bs : 0;
  if (w >= nA + nB) return;
  double v[P];
  int ix[P];
  tp_init<P>(v, ix);
  double *ov;
  int *oi;
  if (w < nA) {
    const double *sv = pva + w * ncha * P;
    const int *si = pia + w * ncha * P;
    for (int e = lane; e < ncha * P; e += 32) tp_insert<P>(v, ix, sv[e], si[e]);
    ov = topA_v + w * P;
    oi = topA_i + w * P;
  } else {
    const int64_t u = w - nA;
    const double *sv = pvb + u * nchb * P;
    const int *si = pib + u * nchb * P;
    for (int e = lane; e < nchb * P; e += 32) tp_insert<P>(v, ix, sv[e], si[e]);
    ov = topB_v + u * P;
    oi = topB_i + u * P;
  }
#pragma unroll
  for (int m = 16; m >= 1; m >>= 1) tp_shfl_merge<P>(v, ix, m);
  if (lane == 0) {
#pragma unroll
    for (int s = 0; s < P; ++s) { ov[s] = v[s]; oi[s] = ix[s]; }
  }
}

template <typename T, int P>
aabft_status run_encode(const aabft_config *cfg, const T *A, int64_t lda, const T *B,
                        int64_t ldb, const aabft_encoded *out, void *ws, cudaStream_t st) {
  const int64_t M = cfg->M, N = cfg->N, K = cfg->K;
  const int bs = cfg->bs;
  const int ncha = (int)enc_a_chunks(K), nchb = (int)enc_b_chunks(K);
  char *w = static_cast<char *>(ws);
  const size_t ra = (size_t)(M + M / bs), rb = (size_t)(N + N / bs);
  double *pva = reinterpret_cast<double *>(w);
  w += (ra * ncha * P * 8 + 255) / 256 * 256;
  int *pia = reinterpret_cast<int *>(w);
  w += (ra * ncha * P * 4 + 255) / 256 * 256;
  double *pvb = reinterpret_cast<double *>(w);
  w += (rb * nchb * P * 8 + 255) / 256 * 256;
  int *pib = reinterpret_cast<int *>(w);
  // top-p tables NULL: checksums only (the encoding of the fixed-eps and SEA comparators)
  const bool tpa = A && out->topA_val, tpb = B && out->topB_val;
  if (A) {
    dim3 grid(ncha, (unsigned)(M / bs));
    auto kern = tpa ? encode_a_kernel<T, P, true> : encode_a_kernel<T, P, false>;
    kern<<<grid, 128, 0, st>>>(A, lda, K, bs, static_cast<T *>(out->Acs), out->ld_acs, pva, pia,
                               ncha);
    next_launch();
  }
  if (B) {
    const int NC = std::max(128, bs);
    dim3 grid((unsigned)((N + NC - 1) / NC), nchb);
    if (NC == 128) {
      auto kern = tpb ? encode_b_kernel<T, P, 128, true> : encode_b_kernel<T, P, 128, false>;
      kern<<<grid, 128, 0, st>>>(B, ldb, K, N, bs, static_cast<T *>(out->Bcs), out->ld_bcs, pvb,
                                 pib, nchb);
    } else {
      auto kern = tpb ? encode_b_kernel<T, P, 256, true> : encode_b_kernel<T, P, 256, false>;
      kern<<<grid, 256, 0, st>>>(B, ldb, K, N, bs, static_cast<T *>(out->Bcs), out->ld_bcs, pvb,
                                 pib, nchb);
    }
    next_launch();
  }
  const int64_t nvec = (tpa ? M + M / bs : 0) + (tpb ? N + N / bs : 0);
  if (nvec > 0) {
    topp_reduce_kernel<T, P><<<(unsigned)((nvec + 7) / 8), 256, 0, st>>>(
        M, N, K, bs, pva, pia, ncha, pvb, pib, nchb, static_cast<const T *>(out->Acs),
        out->ld_acs, static_cast<const T *>(out->Bcs), out->ld_bcs, out->topA_val,
        out->topA_idx, out->topB_val, out->topB_idx, tpa, tpb);
    next_launch();
  }
  return check_launch("aabft_encode");
}

template <typename T>
aabft_status dispatch_p(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                        int64_t ldb, const aabft_encoded *out, void *ws, cudaStream_t st) {
  const T *a = static_cast<const T *>(A);
  const T *b = static_cast<const T *>(B);
  switch (cfg->p) {
    case 1: return run_encode<T, 1>(cfg, a, lda, b, ldb, out, ws, st);
    case 2: return run_encode<T, 2>(cfg, a, lda, b, ldb, out, ws, st);
    case 3: return run_encode<T, 3>(cfg, a, lda, b, ldb, out, ws, st);
    case 4: return run_encode<T, 4>(cfg, a, lda, b, ldb, out, ws, st);
    case 5: return run_encode<T, 5>(cfg, a, lda, b, ldb, out, ws, st);
    case 6: return run_encode<T, 6>(cfg, a, lda, b, ldb, out, ws, st);
    case 7: return run_encode<T, 7>(cfg, a, lda, b, ldb, out, ws, st);
    case 8: return run_encode<T, 8>(cfg, a, lda, b, ldb, out, ws, st);
  }
  set_error("p=%d out of range", cfg->p);
  return AABFT_EINVAL;
}

}  // namespace

size_t encode_ws_bytes(const aabft_config *cfg) {
  const size_t p = (size_t)cfg->p;
  const size_t ncha = (size_t)enc_a_chunks(cfg->K), nchb = (size_t)enc_b_chunks(cfg->K);
  auto r = [](size_t b) { return (b + 255) / 256 * 256; };
  const size_t ra = (size_t)(cfg->M + cfg->M / cfg->bs), rb = (size_t)(cfg->N + cfg->N / cfg->bs);
  return r(ra * ncha * p * 8) + r(ra * ncha * p * 4) + r(rb * nchb * p * 8) + r(rb * nchb * p * 4);
}

aabft_status launch_encode(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                           int64_t ldb, const aabft_encoded *out, void *ws, cudaStream_t st) {
  if (cfg->dtype == AABFT_F64) return dispatch_p<double>(cfg, A, lda, B, ldb, out, ws, st);
  return dispatch_p<float>(cfg, A, lda, B, ldb, out, ws, st);
}

}  // namespace aabft
