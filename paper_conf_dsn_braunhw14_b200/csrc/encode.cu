// encode.cu -- step 1 of A-ABFT on sm_100a: partitioned checksum encoding fused with top-p
// |value| selection (P:L313-317 steps 1a-1d; Alg 1), and the global top-p
// reduction (step 3, P:L320 / P:L368).
//
// B200 design: HBM-bound streaming.  One thread owns one column of a
// BS-row block of A, so the column checksum is a register running sum in ascending row order
// (bit-identical to Eq 1 summed top -> bottom, reading R11) and every warp load is a
// contiguous 256 B row segment.  The same pass stages the selection KEYS of |a| in padded
// shared memory, where four lanes per row keep register top-p lists over interleaved columns
// and merge them with two xor-shuffles (warp-shuffle top-p).  B is the mirror image: a thread
// owns a column of B (running top-p over k in registers) and the BS-wide row sums are taken
// from the staged tile, one sequential thread per (row, block).
//  * Selection keys: the bit pattern of |x| (+1) as an unsigned integer orders like |x|, so
//    the top-p compares and selects run on the integer ALU (ISETP/SEL) rather than the FP64
//    pipe (FP32 data: 32-bit keys); the insertion is branch-free (kp_push), so a warp never
//    diverges on inserts.
//  * Each CTA parks its chunk's partial lists; step 3 merges them with a warp per vector
//    across the whole GPU (topp_reduce_kernel).  A last-CTA-per-group merge inside the encode
//    launches was measured slower: the merges serialise on L2 latency in a few CTAs
//    (DESIGN.md 8.7).
//  * Strips are double-buffered in registers (the next strip's loads are in flight during the
//    top-p / row-sum phase).
#include <algorithm>
#include <atomic>

#include "common.cuh"

namespace aabft {
namespace {

#ifndef AABFT_ENC_STRIP
#define AABFT_ENC_STRIP 32
#endif
constexpr int kStrip = AABFT_ENC_STRIP;  // rows staged per pass

template <typename T>
__device__ __forceinline__ T ldg(const T *p) { return __ldg(p); }

// ------------------------------------------------------------------------- selection keys
template <typename T> struct Key;
template <> struct Key<double> {
  using type = unsigned long long;
  static __device__ __forceinline__ type of(double x) {
    return ((unsigned long long)__double_as_longlong(x) & 0x7FFFFFFFFFFFFFFFull) + 1ull;
  }
  static __device__ __forceinline__ double val(type k) { return __longlong_as_double((long long)(k - 1ull)); }
};
template <> struct Key<float> {
  using type = unsigned int;
  static __device__ __forceinline__ type of(float x) { return (__float_as_uint(x) & 0x7FFFFFFFu) + 1u; }
  static __device__ __forceinline__ double val(type k) { return (double)__uint_as_float(k - 1u); }
};

// key 0 with index -1 is below every element (keys are >= 1)
template <int P, typename KT>
__device__ __forceinline__ void kp_init(KT (&v)[P], int (&ix)[P]) {
#pragma unroll
  for (int r = 0; r < P; ++r) { v[r] = 0; ix[r] = -1; }
}

// push an element that loses every tie (larger index than everything in the list: a lane
// scanning its own elements in ascending index order); branch-free for every P
template <int P, typename KT>
__device__ __forceinline__ void kp_push(KT (&v)[P], int (&ix)[P], KT a, int idx) {
  bool g[P];
#pragma unroll
  for (int r = 0; r < P; ++r) g[r] = a > v[r];
#pragma unroll
  for (int r = P - 1; r >= 1; --r) {
    const KT vr = g[r - 1] ? v[r - 1] : (g[r] ? a : v[r]);
    const int ir = g[r - 1] ? ix[r - 1] : (g[r] ? idx : ix[r]);
    v[r] = vr;
    ix[r] = ir;
  }
  v[0] = g[0] ? a : v[0];
  ix[0] = g[0] ? idx : ix[0];
}

// insertion with the full order (key desc, index asc; empty slots: key 0, index -1, which as
// an unsigned index is larger than every real one).  Branch-free: g[r] = "a precedes slot r"
// is monotone in r for a sorted list, so the same shift as kp_push applies; an empty candidate
// (key 0, index -1) precedes nothing.
template <int P, typename KT>
__device__ __forceinline__ void kp_insert(KT (&v)[P], int (&ix)[P], KT a, int idx) {
  bool g[P];
#pragma unroll
  for (int r = 0; r < P; ++r) g[r] = a > v[r] || (a == v[r] && (unsigned)idx < (unsigned)ix[r]);
#pragma unroll
  for (int r = P - 1; r >= 1; --r) {
    const KT vr = g[r - 1] ? v[r - 1] : (g[r] ? a : v[r]);
    const int ir = g[r - 1] ? ix[r - 1] : (g[r] ? idx : ix[r]);
    v[r] = vr;
    ix[r] = ir;
  }
  v[0] = g[0] ? a : v[0];
  ix[0] = g[0] ? idx : ix[0];
}

template <int P, typename KT>
__device__ __forceinline__ void kp_shfl_merge(KT (&v)[P], int (&ix)[P], int lane_mask) {
  KT ov[P];
  int oi[P];
#pragma unroll
  for (int r = 0; r < P; ++r) {
    ov[r] = __shfl_xor_sync(0xffffffffu, v[r], lane_mask);
    oi[r] = __shfl_xor_sync(0xffffffffu, ix[r], lane_mask);
  }
#pragma unroll
  for (int r = 0; r < P; ++r) kp_insert<P, KT>(v, ix, ov[r], oi[r]);
}

template <typename T, int P>
__device__ __forceinline__ void kp_store(double *dv, int *di, const typename Key<T>::type (&v)[P],
                                         const int (&ix)[P]) {
#pragma unroll
  for (int s = 0; s < P; ++s) {
    dv[s] = ix[s] < 0 ? -1.0 : Key<T>::val(v[s]);
    di[s] = ix[s];
  }
}

// Step 3 for one vector: merge its `nch` partial lists (value desc, index asc) with a warp and
// write the final p entries.  Partial lists come from other CTAs: read them through L2.
template <int P>
__device__ __forceinline__ void merge_vector(const double *__restrict__ pv, const int *__restrict__ pi,
                                             int nch, double *ov, int *oi, int lane) {
  double v[P];
  int ix[P];
  tp_init<P>(v, ix);
  for (int e = lane; e < nch * P; e += 32) tp_insert<P>(v, ix, __ldcg(pv + e), __ldcg(pi + e));
#pragma unroll
  for (int m = 16; m >= 1; m >>= 1) tp_shfl_merge<P>(v, ix, m);
  if (lane == 0) {
#pragma unroll
    for (int s = 0; s < P; ++s) { ov[s] = v[s]; oi[s] = ix[s]; }
  }
}

// ---------------------------------------------------------------------------------- A
// 1-D grid: unit u -> block-row I = u / nch, column chunk = u % nch (128 columns); 128 threads.
template <typename T>
__host__ __device__ constexpr int enc_a_smem() { return kStrip * (kEncAChunk + 4) * (int)sizeof(typename Key<T>::type); }
template <typename T, int NC>
__host__ __device__ constexpr int enc_b_smem() { return ((NC * sizeof(T) > 1024) ? 16 : kStrip) * (NC + 1) * (int)sizeof(T); }

template <typename T, int P, bool TOPP>
__device__ __forceinline__ void encode_a_body(const T *__restrict__ A, int64_t lda, int64_t M,
                                              int64_t K, int bs, T *__restrict__ Acs,
                                              int64_t ld_acs, double *__restrict__ pv,
                                              int *__restrict__ pi, int nch, unsigned unit,
                                              unsigned char *sbuf) {
  using KT = typename Key<T>::type;
  // keys of the |A| strip, stride kEncAChunk + 4: conflict-free lane reads
  KT (*tile)[kEncAChunk + 4] = reinterpret_cast<KT (*)[kEncAChunk + 4]>(sbuf);
  const int c = threadIdx.x;
  const int chunk = (int)(unit % (unsigned)nch);
  const int64_t I = unit / (unsigned)nch;
  const int64_t k = (int64_t)chunk * kEncAChunk + c;
  const bool kin = k < K;
  const int r = c >> 2, q = c & 3;  // top-p role: row r of the strip, column phase q
  T sum = T(0);
  T vals[kStrip];
  auto load_strip = [&](int r0) {
    const int rows = min(kStrip, bs - r0);
    const T *src = A + (I * bs + r0) * lda + k;
    if (rows == kStrip) {
      // full strip: the kStrip loads are issued back to back (memory-level parallelism)
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
        if (TOPP) tile[rr][c] = Key<T>::of(vals[rr]);
      }
    }
    if (r0 + kStrip < bs) load_strip(r0 + kStrip);
    if (!TOPP) continue;  // checksums only (fixed-eps / SEA ABFT comparators, NEXT-3)
    __syncthreads();
    KT v[P], v2[P];
    int ix[P], ix2[P];
    kp_init<P>(v, ix);
    kp_init<P>(v2, ix2);
    if (r < rows) {
      // ascending columns into this lane's own two lists (columns q + 8t and q + 4 + 8t: two
      // independent dependency chains): the new element loses every tie within its list
      const int kbase = chunk * kEncAChunk;
      const int lim = K - kbase < kEncAChunk ? (int)(K - kbase) : kEncAChunk;
      const KT *trow = tile[r];
#pragma unroll 4
      for (int cc = q; cc < kEncAChunk; cc += 8) {
        const KT k1 = cc < lim ? trow[cc] : KT(0);  // key 0 never enters a list
        const KT k2 = cc + 4 < lim ? trow[cc + 4] : KT(0);
        kp_push<P, KT>(v, ix, k1, kbase + cc);
        kp_push<P, KT>(v2, ix2, k2, kbase + cc + 4);
      }
#pragma unroll
      for (int t = 0; t < P; ++t) kp_insert<P, KT>(v, ix, v2[t], ix2[t]);
    }
    kp_shfl_merge<P, KT>(v, ix, 1);
    kp_shfl_merge<P, KT>(v, ix, 2);
    if (r < rows && q == 0) {
      const int64_t row = I * bs + r0 + r;
      kp_store<T, P>(pv + (row * nch + chunk) * P, pi + (row * nch + chunk) * P, v, ix);
    }
    __syncthreads();
  }
  if (kin) Acs[I * ld_acs + k] = sum;
  if (!TOPP) return;
  // partial top-p of the checksum row I over this chunk (Alg 1 localSums / maxReduce)
  {
    __shared__ KT s_v[kEncAChunk / 32][P];
    __shared__ int s_i[kEncAChunk / 32][P];
    KT v[P];
    int ix[P];
    kp_init<P>(v, ix);
    if (kin) kp_push<P, KT>(v, ix, Key<T>::of(sum), (int)k);
#pragma unroll
    for (int m = 16; m >= 1; m >>= 1) kp_shfl_merge<P, KT>(v, ix, m);
    if ((c & 31) == 0) {
#pragma unroll
      for (int s = 0; s < P; ++s) { s_v[c >> 5][s] = v[s]; s_i[c >> 5][s] = ix[s]; }
    }
    __syncthreads();
    if (c == 0) {
      for (int w = 1; w < kEncAChunk / 32; ++w)
#pragma unroll
        for (int s = 0; s < P; ++s) kp_insert<P, KT>(v, ix, s_v[w][s], s_i[w][s]);
      const int64_t row = M + I;  // checksum rows follow the M data rows
      kp_store<T, P>(pv + (row * nch + chunk) * P, pi + (row * nch + chunk) * P, v, ix);
    }
  }
}

template <typename T, int P, bool TOPP>
__global__ void __launch_bounds__(128) encode_a_kernel(const T *__restrict__ A, int64_t lda,
                                                       int64_t M, int64_t K, int bs,
                                                       T *__restrict__ Acs, int64_t ld_acs,
                                                       double *__restrict__ pv,
                                                       int *__restrict__ pi, int nch) {
  __shared__ __align__(16) unsigned char sbuf[enc_a_smem<T>()];
  encode_a_body<T, P, TOPP>(A, lda, M, K, bs, Acs, ld_acs, pv, pi, nch, blockIdx.x, sbuf);
}

// ---------------------------------------------------------------------------------- B
// 1-D grid: unit u -> column chunk jc = u / nch (NC columns), row chunk kc = u % nch
// (kEncBChunk rows of B); NC threads (NC = max(128, bs)).
template <typename T, int P, int NC, bool TOPP>
__device__ __forceinline__ void encode_b_body(const T *__restrict__ B, int64_t ldb, int64_t K,
                                              int64_t N, int bs, T *__restrict__ Bcs,
                                              int64_t ld_bcs, double *__restrict__ pv,
                                              int *__restrict__ pi, int nch, unsigned unit,
                                              unsigned char *sbuf) {
  using KT = typename Key<T>::type;
  constexpr int SB = (NC * sizeof(T) > 1024) ? 16 : kStrip;  // strip rows (smem <= 48 KiB)
  // odd stride NC + 1: conflict-free per-row sequential reads
  T (*tile)[NC + 1] = reinterpret_cast<T (*)[NC + 1]>(sbuf);
  const int c = threadIdx.x;
  const int64_t jc = unit / (unsigned)nch;
  const int kc = (int)(unit % (unsigned)nch);
  const int64_t j = jc * NC + c;
  const bool jin = j < N;
  const int64_t kbeg = (int64_t)kc * kEncBChunk;
  const int64_t kend = K < kbeg + kEncBChunk ? K : kbeg + kEncBChunk;
  const int nblk = NC / bs;  // checksum blocks covered by this CTA (<= 16)
  // checksum-column top-p.  bs >= 32 (at most one block per warp): a running list per lane --
  // lane rr of the warp owning block jb sees rows k0 + rr in ascending k across strips --
  // merged across the warp once at the end.  Smaller blocks (several per warp): the strip's
  // 32 row sums are folded into a shared-memory list per block after every strip.
  const bool lane_lists = nblk <= NC / 32;
  KT cvl[P];
  int cil[P];
  kp_init<P>(cvl, cil);
  __shared__ KT s_cv[16][P];
  __shared__ int s_ci[16][P];
  if (c < 16 * P) { s_cv[c / P][c % P] = 0; s_ci[c / P][c % P] = -1; }
  KT v[P], v2[P];  // running top-p of column j over even / odd rows (two dependency chains)
  int ix[P], ix2[P];
  kp_init<P>(v, ix);
  kp_init<P>(v2, ix2);
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
        if (TOPP) {
          if (rr & 1) kp_push<P, KT>(v2, ix2, Key<T>::of(vals[rr]), k0i + rr);
          else kp_push<P, KT>(v, ix, Key<T>::of(vals[rr]), k0i + rr);
        }
      }
    } else {
#pragma unroll
      for (int rr = 0; rr < SB; ++rr) {
        if (rr < rows) {
          tile[rr][c] = vals[rr];
          if (TOPP) {
            if (rr & 1) kp_push<P, KT>(v2, ix2, Key<T>::of(vals[rr]), k0i + rr);
            else kp_push<P, KT>(v, ix, Key<T>::of(vals[rr]), k0i + rr);
          }
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
      const int64_t J = jc * nblk + jb;
      KT lv[P];
      int li[P];
      kp_init<P>(lv, li);
      if (rr < rows && J * bs < N) {
        T sm = T(0);
        for (int jj = 0; jj < bs; ++jj) sm = sm + tile[rr][jb * bs + jj];
        Bcs[(k0 + rr) * ld_bcs + J] = sm;
        if (TOPP) {
          if (lane_lists) kp_push<P, KT>(cvl, cil, Key<T>::of(sm), (int)(k0 + rr));
          else kp_push<P, KT>(lv, li, Key<T>::of(sm), (int)(k0 + rr));
        }
      }
      if (!TOPP || lane_lists) continue;
#pragma unroll
      for (int m = 16; m >= 1; m >>= 1) kp_shfl_merge<P, KT>(lv, li, m);
      if (rr == 0) {
#pragma unroll
        for (int r = 0; r < P; ++r) kp_insert<P, KT>(lv, li, s_cv[jb][r], s_ci[jb][r]);
#pragma unroll
        for (int r = 0; r < P; ++r) { s_cv[jb][r] = lv[r]; s_ci[jb][r] = li[r]; }
      }
    }
    __syncthreads();
  }
  if (!TOPP) return;
#pragma unroll
  for (int t = 0; t < P; ++t) kp_insert<P, KT>(v, ix, v2[t], ix2[t]);
  if (lane_lists) {
    // checksum columns: merge the 32 lanes' lists of the warp's block once
    const int jb = c >> 5;
    if (jb < nblk) {  // warp-uniform
#pragma unroll
      for (int m = 16; m >= 1; m >>= 1) kp_shfl_merge<P, KT>(cvl, cil, m);
      const int64_t J = jc * nblk + jb;
      if ((c & 31) == 0 && J * bs < N)
        kp_store<T, P>(pv + ((N + J) * nch + kc) * P, pi + ((N + J) * nch + kc) * P, cvl, cil);
    }
  } else if (c < nblk && (jc * nblk + c) * bs < N) {
    const int64_t J = jc * nblk + c;
    KT cv[P];
    int ci[P];
#pragma unroll
    for (int r = 0; r < P; ++r) { cv[r] = s_cv[c][r]; ci[r] = s_ci[c][r]; }
    kp_store<T, P>(pv + ((N + J) * nch + kc) * P, pi + ((N + J) * nch + kc) * P, cv, ci);
  }
  if (jin) kp_store<T, P>(pv + (j * nch + kc) * P, pi + (j * nch + kc) * P, v, ix);
}

template <typename T, int P, int NC, bool TOPP>
__global__ void __launch_bounds__(NC) encode_b_kernel(const T *__restrict__ B, int64_t ldb,
                                                      int64_t K, int64_t N, int bs,
                                                      T *__restrict__ Bcs, int64_t ld_bcs,
                                                      double *__restrict__ pv,
                                                      int *__restrict__ pi, int nch) {
  __shared__ __align__(16) unsigned char sbuf[enc_b_smem<T, NC>()];
  encode_b_body<T, P, NC, TOPP>(B, ldb, K, N, bs, Bcs, ld_bcs, pv, pi, nch, blockIdx.x, sbuf);
}

// A and B in ONE launch (bs <= 128): the B units (longer: kEncBChunk rows each) come first,
// then the A units; one shared buffer serves whichever body the CTA runs.  Saves a launch
// boundary and lets the A units fill the machine while B's last units finish.
template <typename T, int P, bool TOPP>
#ifndef AABFT_ENC_MINB
#define AABFT_ENC_MINB 1
#endif
__global__ void __launch_bounds__(128, AABFT_ENC_MINB) encode_ab_kernel(
    const T *__restrict__ A, int64_t lda, int64_t M, int64_t K, int bs, T *__restrict__ Acs,
    int64_t ld_acs, double *__restrict__ pva, int *__restrict__ pia, int ncha,
    const T *__restrict__ B, int64_t ldb, int64_t N, T *__restrict__ Bcs, int64_t ld_bcs,
    double *__restrict__ pvb, int *__restrict__ pib, int nchb, unsigned nB) {
  constexpr int SA = enc_a_smem<T>(), SBb = enc_b_smem<T, 128>();
  __shared__ __align__(16) unsigned char sbuf[SA > SBb ? SA : SBb];
  if (blockIdx.x < nB)
    encode_b_body<T, P, 128, TOPP>(B, ldb, K, N, bs, Bcs, ld_bcs, pvb, pib, nchb, blockIdx.x, sbuf);
  else
    encode_a_body<T, P, TOPP>(A, lda, M, K, bs, Acs, ld_acs, pva, pia, ncha, blockIdx.x - nB, sbuf);
}

// ---------------------------------------------------------------------------------- step 3
// One warp per vector (data rows + checksum rows of A, data cols + checksum cols of B): merge
// the per-chunk partial lists produced by the encode kernels.
template <int P>
__global__ void __launch_bounds__(256) topp_reduce_kernel(
    int64_t M, int64_t N, int bs, const double *__restrict__ pva, const int *__restrict__ pia,
    int ncha, const double *__restrict__ pvb, const int *__restrict__ pib, int nchb,
    double *__restrict__ topA_v, int *__restrict__ topA_i, double *__restrict__ topB_v,
    int *__restrict__ topB_i, int do_a, int do_b) {
  const int lane = threadIdx.x & 31;
  const int64_t w = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5);
  const int64_t nA = do_a ? M + M / bs : 0;
  const int64_t nB = do_b ? N + N / bs : 0;
  if (w >= nA + nB) return;
  if (w < nA) {
    merge_vector<P>(pva + w * ncha * P, pia + w * ncha * P, ncha, topA_v + w * P, topA_i + w * P, lane);
  } else {
    const int64_t u = w - nA;
    merge_vector<P>(pvb + u * nchb * P, pib + u * nchb * P, nchb, topB_v + u * P, topB_i + u * P, lane);
  }
}

// ------------------------------------------------------------ encode overlapped with the GEMM
// AABFT_FLAG_OVERLAP_ENCODE (FP64, bs in {16, 32, 64}, p <= 4).  The encode is HBM-bound and
// the FP64 GEMM is DMMA-bound, and only the GEMM's checksum tiles (Ccol = Acs.B,
// Crow = A.Bcs; the last tiles of its schedule) read the encoding, so the two run AT THE SAME
// TIME: this kernel is a small persistent grid (one 64-thread CTA per SM, <= 64 registers,
// ~20 KB of shared memory: it fits next to the GEMM's three CTAs per SM) that triggers its
// dependents as soon as it starts (programmatic dependent launch); the GEMM launched after it
// streams its data tiles at once and waits for this grid (griddepcontrol.wait) only before
// its first checksum tile.  The paper runs its global top-p reduction "in parallel to the
// matrix multiplication kernel"; here the whole of step 1 does.
//
// A unit = one block-row I of A over all K, a B unit = 64 columns of B over all K, so every
// vector's top-p list is complete inside one CTA (no partial lists, no reduction kernel).
// Tiles of 16 rows x 64 columns arrive by cp.async (every thread copies 16-byte chunks; rows
// padded in shared memory) through a 2-stage ring.  The arithmetic is the sequential definition, as in the kernels above:
// Acs -- a thread per column adds the block's rows in ascending i; Bcs -- a thread per
// (row, block) adds the block's columns in ascending j; top-p -- branch-free pushes in
// ascending index order, merged with the full order (key desc, index asc), so the results are
// bit-identical to encode_ab_kernel + topp_reduce_kernel.
constexpr int kOvR = 16, kOvC = 64;             // tile: 16 rows x 64 columns of doubles
// padded row pitches (doubles; 16-byte multiples for cp.async): A 68 -- a half-warp of the
// 4-lanes-per-row top-p scan touches 16 distinct bank pairs; B 66 -- the 16 row-sum threads
// read one column with a 2-way conflict at most; every column pass is conflict-free
constexpr int kOvPitchA = 68, kOvPitchB = 66;
constexpr int kOvTileBytes = kOvR * kOvPitchA * 8;  // 8.5 KiB per stage
constexpr int kOvStages = 2;
constexpr int kOvThreads = 64;
constexpr int kOvMaxP = 4;
constexpr int kOvSmem = kOvStages * kOvTileBytes + 64 * kOvMaxP * 12 /*row lists*/ +
                        2 * kOvMaxP * 12 /*warp lists*/;

struct OvArgs {
  const double *A;
  int64_t lda;
  const double *B;
  int64_t ldb;
  int64_t M, N, K;
  int bs;
  int nA, nB;       // units: B units (64-column groups) first, then A units (block-rows)
  int nkt;          // B unit: 16-row tiles over K
  int nkc, nrt;     // A unit: 64-column chunks over K x 16-row tiles per block
  double *Acs;
  int64_t ld_acs;
  double *Bcs;
  int64_t ld_bcs;
  double *topA_v;
  int *topA_i;
  double *topB_v;
  int *topB_i;
};

template <int PITCH>
__device__ __forceinline__ double ov_at(const uint8_t *t, int r, int c) {
  return *reinterpret_cast<const double *>(t + (r * PITCH + c) * 8);
}

__device__ __forceinline__ int ov_unit_tiles(const OvArgs &a, int u) {
  return u < a.nB ? a.nkt : a.nkc * a.nrt;
}

// 16-byte cp.async global -> shared with zero fill beyond `bytes` (L2 only: .cg).  The loads
// go through the SM's load/store path, not its TMA unit, which the concurrently running GEMM
// keeps busy with its operand tiles (measured: sharing the TMA unit slowed both kernels)
__device__ __forceinline__ void ov_cp16(void *dst, const void *src, int bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(dst)), "l"(src),
               "r"(bytes)
               : "memory");
}

// all 64 threads: tile `t` of unit `u` into `dst` (one 16-byte chunk per thread and row pair:
// each warp instruction copies one contiguous 512-byte row segment)
__device__ __forceinline__ void ov_issue(const OvArgs &a, uint8_t *dst, int u, int t) {
  const int tid = threadIdx.x, c2 = tid & 31;
  if (u < a.nB) {
    const int64_t j = (int64_t)u * kOvC + 2 * c2;
    const int cb = (int)(a.N - j < 2 ? (a.N - j > 0 ? a.N - j : 0) : 2) * 8;
#pragma unroll
    for (int i = 0; i < kOvR / 2; ++i) {
      const int r = (tid >> 5) + 2 * i;
      const int64_t k = (int64_t)t * kOvR + r;
      const int bytes = k < a.K ? cb : 0;
      ov_cp16(dst + (r * kOvPitchB + 2 * c2) * 8, bytes ? a.B + k * a.ldb + j : a.B, bytes);
    }
  } else {
    const int I = u - a.nB, kc = t / a.nrt, rt = t % a.nrt;
    const int64_t k = (int64_t)kc * kOvC + 2 * c2;
    const int bytes = (int)(a.K - k < 2 ? (a.K - k > 0 ? a.K - k : 0) : 2) * 8;
#pragma unroll
    for (int i = 0; i < kOvR / 2; ++i) {
      const int r = (tid >> 5) + 2 * i;
      const int64_t row = (int64_t)I * a.bs + rt * kOvR + r;
      ov_cp16(dst + (r * kOvPitchA + 2 * c2) * 8, bytes ? a.A + row * a.lda + k : a.A, bytes);
    }
  }
  asm volatile("cp.async.commit_group;" ::: "memory");
}

#ifdef AABFT_OV_PROBE
// timing diagnosis: [0] first encode CTA start, [1] last encode CTA end (globaltimer, ns)
__device__ unsigned long long g_ov_probe[2] = {~0ull, 0ull};
__device__ __forceinline__ unsigned long long ov_gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#endif

template <int P, int BS>
__global__ void __launch_bounds__(kOvThreads, 16) encode_overlap_kernel(const OvArgs a) {
  // the dependent GEMM may start now: it reads the encoding only after griddepcontrol.wait
  griddep_launch_dependents();
#ifdef AABFT_OV_NOOP
  return;  // timing diagnosis only (no encoding is produced)
#endif
#ifdef AABFT_OV_PROBE
  if (threadIdx.x == 0) atomicMin(&g_ov_probe[0], ov_gtime());
#endif
  using KT = unsigned long long;
  extern __shared__ __align__(16) uint8_t ring[];
  KT *s_rv = reinterpret_cast<KT *>(ring + kOvStages * kOvTileBytes);  // [64 rows][P] (A)
  int *s_ri = reinterpret_cast<int *>(s_rv + 64 * P);
  KT *s_wv = reinterpret_cast<KT *>(s_ri + 64 * P);   // [2 warps][P] cross-warp merge
  int *s_wi = reinterpret_cast<int *>(s_wv + 2 * P);
  const int tid = threadIdx.x, lane = tid & 31;
  const int nunits = a.nA + a.nB;
  // issue cursor (uniform over the CTA): unit iu, tile it; one commit group per stage
  int iu = blockIdx.x, it = 0;
  for (int s = 0; s < kOvStages; ++s) {
    if (iu < nunits) {
      ov_issue(a, ring + s * kOvTileBytes, iu, it);
      if (++it == ov_unit_tiles(a, iu)) { it = 0; iu += gridDim.x; }
    } else {
      asm volatile("cp.async.commit_group;" ::: "memory");
    }
  }
  int job = 0;
  for (int u = blockIdx.x; u < nunits; u += gridDim.x) {
    const int ntile = ov_unit_tiles(a, u);
    KT cv[P];  // B: column list of column j0 + tid; A: checksum-row list over columns k0 + tid
    int ci[P];
    KT sv[P];  // B: list of checksum column J over this thread's rows
    int si[P];
    kp_init<P, KT>(cv, ci);
    kp_init<P, KT>(sv, si);
    double colsum = 0.0;
    const bool isB = u < a.nB;
    if (!isB) {
      for (int e = tid; e < a.bs * P; e += kOvThreads) { s_rv[e] = 0; s_ri[e] = -1; }
    }
    for (int t = 0; t < ntile; ++t, ++job) {
      const int s = job % kOvStages;
      asm volatile("cp.async.wait_group %0;" ::"n"(kOvStages - 1) : "memory");
      __syncthreads();  // every thread's chunks of stage s have landed
      const uint8_t *tile = ring + s * kOvTileBytes;
      if (isB) {
        const int64_t j0 = (int64_t)u * kOvC;
        const int k0 = t * kOvR;
        // column top-p: thread tid owns column j0 + tid, rows in ascending k
#pragma unroll
        for (int r = 0; r < kOvR; ++r)
          if (k0 + r < a.K) kp_push<P, KT>(cv, ci, Key<double>::of(ov_at<kOvPitchB>(tile, r, tid)), k0 + r);
        // Eq 2 row checksums: thread (r, b) adds block b's bs columns of row r, ascending j
        const int r = tid & 15, b = tid >> 4;
        const int64_t J = j0 / BS + b;
        if (b < kOvC / BS && k0 + r < a.K && J * BS < a.N) {
          double sm = 0.0;
#pragma unroll
          for (int j8 = 0; j8 < BS; j8 += 8) {  // loads of a batch issued together
            double x[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) x[e] = ov_at<kOvPitchB>(tile, r, b * BS + j8 + e);
#pragma unroll
            for (int e = 0; e < 8; ++e) {
#ifdef AABFT_OV_NODADD  // timing diagnosis only: integer adds instead of FP64 adds
              sm = __longlong_as_double(__double_as_longlong(sm) + __double_as_longlong(x[e]));
#else
              sm = sm + x[e];
#endif
            }
          }
          a.Bcs[(int64_t)(k0 + r) * a.ld_bcs + J] = sm;
          kp_push<P, KT>(sv, si, Key<double>::of(sm), k0 + r);
        }
      } else {
        const int I = u - a.nB, kc = t / a.nrt, rt = t % a.nrt;
        const int k0 = kc * kOvC;
        // Eq 1 column checksums: ascending i across the block's row tiles
        if (rt == 0) colsum = 0.0;
#pragma unroll
        for (int r = 0; r < kOvR; ++r) {
#ifdef AABFT_OV_NODADD
          colsum = __longlong_as_double(__double_as_longlong(colsum) +
                                        __double_as_longlong(ov_at<kOvPitchA>(tile, r, tid)));
#else
          colsum = colsum + ov_at<kOvPitchA>(tile, r, tid);
#endif
        }
        // row top-p: 4 lanes per row, lane q scans columns q, q + 4, ... (ascending)
        {
          const int r = tid >> 2, q = tid & 3;
          KT lv[P];
          int li[P];
          kp_init<P, KT>(lv, li);
#pragma unroll
          for (int m = 0; m < kOvC / 4; ++m) {
            const int c = q + 4 * m;
            const KT key = k0 + c < a.K ? Key<double>::of(ov_at<kOvPitchA>(tile, r, c)) : KT(0);
            kp_push<P, KT>(lv, li, key, k0 + c);
          }
          kp_shfl_merge<P, KT>(lv, li, 1);
          kp_shfl_merge<P, KT>(lv, li, 2);
          if (q == 0) {  // fold into the row's running list (earlier chunks: smaller indices)
            const int row = rt * kOvR + r;
#pragma unroll
            for (int e = 0; e < P; ++e) kp_insert<P, KT>(lv, li, s_rv[row * P + e], s_ri[row * P + e]);
#pragma unroll
            for (int e = 0; e < P; ++e) { s_rv[row * P + e] = lv[e]; s_ri[row * P + e] = li[e]; }
          }
        }
        if (rt == a.nrt - 1 && k0 + tid < a.K) {
          a.Acs[(int64_t)I * a.ld_acs + k0 + tid] = colsum;
          kp_push<P, KT>(cv, ci, Key<double>::of(colsum), k0 + tid);
        }
      }
      __syncthreads();  // stage s fully read
      if (iu < nunits) {
        ov_issue(a, ring + s * kOvTileBytes, iu, it);
        if (++it == ov_unit_tiles(a, iu)) { it = 0; iu += gridDim.x; }
      } else {
        asm volatile("cp.async.commit_group;" ::: "memory");
      }
    }
    // ---- unit epilogue: complete lists
    if (isB) {
      const int64_t j = (int64_t)u * kOvC + tid;
      if (j < a.N) kp_store<double, P>(a.topB_v + j * P, a.topB_i + j * P, cv, ci);
      // checksum column J: merge the 16 lanes (r = 0..15) of block b
#pragma unroll
      for (int m = 1; m < 16; m <<= 1) kp_shfl_merge<P, KT>(sv, si, m);
      const int r = tid & 15, b = tid >> 4;
      const int64_t J = (int64_t)u * kOvC / BS + b;
      if (r == 0 && b < kOvC / BS && J * BS < a.N)
        kp_store<double, P>(a.topB_v + (a.N + J) * P, a.topB_i + (a.N + J) * P, sv, si);
    } else {
      const int64_t I = u - a.nB;
      for (int row = tid; row < a.bs; row += kOvThreads) {
        KT v[P];
        int ix[P];
#pragma unroll
        for (int e = 0; e < P; ++e) { v[e] = s_rv[row * P + e]; ix[e] = s_ri[row * P + e]; }
        const int64_t gr = I * a.bs + row;
        kp_store<double, P>(a.topA_v + gr * P, a.topA_i + gr * P, v, ix);
      }
      // checksum row I: merge the 64 column-owners' lists
#pragma unroll
      for (int m = 16; m >= 1; m >>= 1) kp_shfl_merge<P, KT>(cv, ci, m);
      if (lane == 0) {
#pragma unroll
        for (int e = 0; e < P; ++e) { s_wv[(tid >> 5) * P + e] = cv[e]; s_wi[(tid >> 5) * P + e] = ci[e]; }
      }
      __syncthreads();
      if (tid == 0) {
#pragma unroll
        for (int e = 0; e < P; ++e) kp_insert<P, KT>(cv, ci, s_wv[P + e], s_wi[P + e]);
        kp_store<double, P>(a.topA_v + (a.M + I) * P, a.topA_i + (a.M + I) * P, cv, ci);
      }
      __syncthreads();  // s_rv / s_wv free for the next unit
    }
  }
  asm volatile("cp.async.wait_all;" ::: "memory");
#ifdef AABFT_OV_PROBE
  if (threadIdx.x == 0) atomicMax(&g_ov_probe[1], ov_gtime());
#endif
}

template <int P, int BS>
aabft_status run_encode_overlap(const aabft_config *cfg, const double *A, int64_t lda,
                                const double *B, int64_t ldb, const aabft_encoded *out,
                                cudaStream_t st) {
  const int64_t M = cfg->M, N = cfg->N, K = cfg->K;
  OvArgs a{};
  a.A = A; a.lda = lda; a.B = B; a.ldb = ldb;
  a.M = M; a.N = N; a.K = K; a.bs = cfg->bs;
  a.nB = (int)((N + kOvC - 1) / kOvC);
  a.nA = (int)(M / cfg->bs);
  a.nkt = (int)((K + kOvR - 1) / kOvR);
  a.nkc = (int)((K + kOvC - 1) / kOvC);
  a.nrt = cfg->bs / kOvR;
  a.Acs = static_cast<double *>(out->Acs); a.ld_acs = out->ld_acs;
  a.Bcs = static_cast<double *>(out->Bcs); a.ld_bcs = out->ld_bcs;
  a.topA_v = out->topA_val; a.topA_i = out->topA_idx;
  a.topB_v = out->topB_val; a.topB_i = out->topB_idx;
  static std::atomic<int> sms_dev[64];  // per instantiation and device
  int dev = 0;
  cudaGetDevice(&dev);
  int sms = sms_dev[dev & 63].load(std::memory_order_relaxed);
  if (!sms) {
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess)
      return check_launch("encode_overlap SM count");
    for (const void *fn : {(const void *)encode_overlap_kernel<P, BS>}) {
      if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, kOvSmem) != cudaSuccess ||
          cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout,
                               cudaSharedmemCarveoutMaxShared) != cudaSuccess)
        return check_launch("encode_overlap attributes");
    }
    sms_dev[dev & 63].store(sms, std::memory_order_relaxed);
  }
  const int units = a.nA + a.nB;
  const int grid = std::min(units, sms);  // one CTA per SM, next to the GEMM's CTAs
  encode_overlap_kernel<P, BS><<<grid, kOvThreads, kOvSmem, st>>>(a);
  next_launch();
  return check_launch("aabft_encode (overlapped)");
}

// workspace: [A partial values][A partial indices][B values][B indices]
struct EncWs {
  double *pva, *pvb;
  int *pia, *pib;
};

size_t r256e(size_t b) { return (b + 255) / 256 * 256; }

EncWs enc_ws(const aabft_config *cfg, void *ws) {
  const size_t p = (size_t)cfg->p;
  const size_t ncha = (size_t)enc_a_chunks(cfg->K), nchb = (size_t)enc_b_chunks(cfg->K);
  const size_t ra = (size_t)(cfg->M + cfg->M / cfg->bs), rb = (size_t)(cfg->N + cfg->N / cfg->bs);
  char *w = static_cast<char *>(ws);
  EncWs e;
  e.pva = reinterpret_cast<double *>(w); w += r256e(ra * ncha * p * 8);
  e.pia = reinterpret_cast<int *>(w); w += r256e(ra * ncha * p * 4);
  e.pvb = reinterpret_cast<double *>(w); w += r256e(rb * nchb * p * 8);
  e.pib = reinterpret_cast<int *>(w);
  return e;
}

template <typename T, int P>
aabft_status run_encode(const aabft_config *cfg, const T *A, int64_t lda, const T *B,
                        int64_t ldb, const aabft_encoded *out, void *ws, cudaStream_t st) {
  const int64_t M = cfg->M, N = cfg->N, K = cfg->K;
  const int bs = cfg->bs;
  const int ncha = (int)enc_a_chunks(K), nchb = (int)enc_b_chunks(K);
  const EncWs e = enc_ws(cfg, ws);
  // top-p tables NULL: checksums only (the encoding of the fixed-eps and SEA comparators);
  // AABFT_FLAG_TOPP_IN_GEMM: the FP64 GEMM selects the top-p from its operand tiles instead
  const bool defer = (cfg->flags & AABFT_FLAG_TOPP_IN_GEMM) && gemm_f64_topp_ok(cfg);
  const bool tpa = A && out->topA_val && !defer, tpb = B && out->topB_val && !defer;
  const int NCb = std::max(128, bs);
  if (A && B && NCb == 128 && tpa == tpb) {
    const unsigned nA = (unsigned)((M / bs) * ncha), nB = (unsigned)(((N + 127) / 128) * nchb);
    auto kern = tpa ? encode_ab_kernel<T, P, true> : encode_ab_kernel<T, P, false>;
    kern<<<nA + nB, 128, 0, st>>>(A, lda, M, K, bs, static_cast<T *>(out->Acs), out->ld_acs, e.pva,
                                  e.pia, ncha, B, ldb, N, static_cast<T *>(out->Bcs), out->ld_bcs,
                                  e.pvb, e.pib, nchb, nB);
    next_launch();
    A = nullptr;  // both done
    B = nullptr;
  }
  if (A) {
    const unsigned grid = (unsigned)((M / bs) * ncha);
    auto kern = tpa ? encode_a_kernel<T, P, true> : encode_a_kernel<T, P, false>;
    kern<<<grid, 128, 0, st>>>(A, lda, M, K, bs, static_cast<T *>(out->Acs), out->ld_acs, e.pva,
                               e.pia, ncha);
    next_launch();
  }
  if (B) {
    const int NC = std::max(128, bs);
    const unsigned grid = (unsigned)(((N + NC - 1) / NC) * nchb);
    if (NC == 128) {
      auto kern = tpb ? encode_b_kernel<T, P, 128, true> : encode_b_kernel<T, P, 128, false>;
      kern<<<grid, 128, 0, st>>>(B, ldb, K, N, bs, static_cast<T *>(out->Bcs), out->ld_bcs, e.pvb,
                                 e.pib, nchb);
    } else {
      auto kern = tpb ? encode_b_kernel<T, P, 256, true> : encode_b_kernel<T, P, 256, false>;
      kern<<<grid, 256, 0, st>>>(B, ldb, K, N, bs, static_cast<T *>(out->Bcs), out->ld_bcs, e.pvb,
                                 e.pib, nchb);
    }
    next_launch();
  }
  const int64_t nvec = (tpa ? M + M / bs : 0) + (tpb ? N + N / bs : 0);
  if (nvec > 0) {
    topp_reduce_kernel<P><<<(unsigned)((nvec + 7) / 8), 256, 0, st>>>(
        M, N, bs, e.pva, e.pia, ncha, e.pvb, e.pib, nchb, out->topA_val, out->topA_idx,
        out->topB_val, out->topB_idx, tpa, tpb);
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

#ifdef AABFT_OV_PROBE
extern "C" int aabft_debug_ov_probe(unsigned long long *out2) {
  cudaMemcpyFromSymbol(out2, g_ov_probe, 16);
  const unsigned long long init[2] = {~0ull, 0ull};
  cudaMemcpyToSymbol(g_ov_probe, init, 16);
  return 0;
}
#endif

size_t encode_ws_bytes(const aabft_config *cfg) {
  const size_t p = (size_t)cfg->p;
  const size_t ncha = (size_t)enc_a_chunks(cfg->K), nchb = (size_t)enc_b_chunks(cfg->K);
  const size_t ra = (size_t)(cfg->M + cfg->M / cfg->bs), rb = (size_t)(cfg->N + cfg->N / cfg->bs);
  return r256e(ra * ncha * p * 8) + r256e(ra * ncha * p * 4) + r256e(rb * nchb * p * 8) +
         r256e(rb * nchb * p * 4);
}

bool encode_overlap_ok(const aabft_config *cfg) {
  return (cfg->flags & AABFT_FLAG_OVERLAP_ENCODE) && cfg->dtype == AABFT_F64 &&
         cfg->bs >= 16 && cfg->bs <= 64 && cfg->p <= kOvMaxP &&
         !((cfg->flags & AABFT_FLAG_TOPP_IN_GEMM) && gemm_f64_topp_ok(cfg));
}

aabft_status launch_encode(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                           int64_t ldb, const aabft_encoded *out, void *ws, cudaStream_t st) {
  if (encode_overlap_ok(cfg) && A && B && out->topA_val && out->topB_val) {
    const double *a = static_cast<const double *>(A), *b = static_cast<const double *>(B);
#define AABFT_OV_CASE(PP, BB) \
  if (cfg->p == PP && cfg->bs == BB) return run_encode_overlap<PP, BB>(cfg, a, lda, b, ldb, out, st);
#define AABFT_OV_BS(PP) AABFT_OV_CASE(PP, 16) AABFT_OV_CASE(PP, 32) AABFT_OV_CASE(PP, 64)
    AABFT_OV_BS(1) AABFT_OV_BS(2) AABFT_OV_BS(3) AABFT_OV_BS(4)
#undef AABFT_OV_BS
#undef AABFT_OV_CASE
  }
  if (cfg->dtype == AABFT_F64) return dispatch_p<double>(cfg, A, lda, B, ldb, out, ws, st);
  return dispatch_p<float>(cfg, A, lda, B, ldb, out, ws, st);
}

}  // namespace aabft
