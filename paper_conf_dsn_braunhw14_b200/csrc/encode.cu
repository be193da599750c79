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
__global__ void __launch_bounds__(128) encode_ab_kernel(
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

size_t encode_ws_bytes(const aabft_config *cfg) {
  const size_t p = (size_t)cfg->p;
  const size_t ncha = (size_t)enc_a_chunks(cfg->K), nchb = (size_t)enc_b_chunks(cfg->K);
  const size_t ra = (size_t)(cfg->M + cfg->M / cfg->bs), rb = (size_t)(cfg->N + cfg->N / cfg->bs);
  return r256e(ra * ncha * p * 8) + r256e(ra * ncha * p * 4) + r256e(rb * nchb * p * 8) +
         r256e(rb * nchb * p * 4);
}

aabft_status launch_encode(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                           int64_t ldb, const aabft_encoded *out, void *ws, cudaStream_t st) {
  if (cfg->dtype == AABFT_F64) return dispatch_p<double>(cfg, A, lda, B, ldb, out, ws, st);
  return dispatch_p<float>(cfg, A, lda, B, ldb, out, ws, st);
}

}  // namespace aabft
