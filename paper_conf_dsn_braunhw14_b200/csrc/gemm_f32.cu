// gemm_f32.cu -- step 2 of A-ABFT (Eq 3) for FP32 on the FFMA pipe (no TF32: a
// tensor-core TF32 product would change the rounding model the bound assumes, north_star).
//
// B200 design: 128 x 128 x 8 CTA tiles, 256 threads, 8 x 8 register
// micro-tiles split 2 x 2 (rows ty*4 / 64+ty*4, cols tx*4 / 64+tx*4) so every shared-memory
// read is an LDS.128 broadcast or a contiguous row.  Global -> register prefetch of the next
// k-tile overlaps the 512 FFMAs of the current one (register double buffering, one barrier per
// k-tile).  Every element accumulates c = fma(a_k, b_k, c) in ascending k, which is exactly
// the fused sequential inner product of Eq 15 / §IV-D -- the FP32 product is bit-identical
// to the definition.  Same three tile types as the FP64 kernel (C, Ccol, Crow) and the same
// fault hooks (site 1 at k-tile granularity, BK = 8).
#include "common.cuh"

namespace aabft {
namespace {

constexpr int BM = 128, BN = 128, BK = 8, THREADS = 256, AST = BM + 4;
constexpr int MAXF = 256;  // faults per 128x128 tile kept in smem (one per 8x8 block)
constexpr int GROUP_M = 8;

struct SgemmArgs {
  const float *A;
  int64_t lda;
  const float *Acs;
  int64_t ld_acs;
  const float *B;
  int64_t ldb;
  const float *Bcs;
  int64_t ld_bcs;
  int64_t M, N, K, Mcs, Ncs;
  float *C;
  int64_t ldc;
  float *Ccol;
  int64_t ld_ccol;
  float *Crow;
  int64_t ld_crow;
  int64_t n0, n1, n2;
  int tm0, tn0, tm1, tn2;
  const aabft_fault *faults;
  int nfaults;
};

__device__ __forceinline__ float4 load4(const float *base, int64_t ld, int64_t r, int64_t rows,
                                        int64_t c, int64_t cols) {
  if (r < rows && c + 3 < cols) return __ldg(reinterpret_cast<const float4 *>(base + r * ld + c));
  float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
  if (r < rows) {
    const float *p = base + r * ld;
    if (c < cols) v.x = __ldg(p + c);
    if (c + 1 < cols) v.y = __ldg(p + c + 1);
    if (c + 2 < cols) v.z = __ldg(p + c + 2);
    if (c + 3 < cols) v.w = __ldg(p + c + 3);
  }
  return v;
}

__device__ __forceinline__ float xor_bits(float v, uint64_t m) {
  return __int_as_float(__float_as_int(v) ^ (int)(uint32_t)m);
}

__global__ void __launch_bounds__(THREADS, 2) gemm_f32_kernel(const SgemmArgs args) {
  __shared__ __align__(16) float As[2][BK][AST];
  __shared__ __align__(16) float Bs[2][BK][BN];
  __shared__ aabft_fault s_f[MAXF];
  __shared__ int s_nf;

  int64_t bid = blockIdx.x;
  int type, tm, tn;
  if (bid < args.n0) {
    type = 0;
    const int64_t group = (int64_t)GROUP_M * args.tn0;
    const int64_t g = bid / group;
    const int first_m = (int)(g * GROUP_M);
    const int gm = min(args.tm0 - first_m, GROUP_M);
    const int64_t in = bid % group;
    tm = first_m + (int)(in % gm);
    tn = (int)(in / gm);
  } else if (bid < args.n0 + args.n1) {
    type = 1;
    bid -= args.n0;
    tm = (int)(bid / args.tn0);
    tn = (int)(bid % args.tn0);
  } else {
    type = 2;
    bid -= args.n0 + args.n1;
    tm = (int)(bid / args.tn2);
    tn = (int)(bid % args.tn2);
  }
  const int64_t m0 = (int64_t)tm * BM, n0 = (int64_t)tn * BN;
  const float *Ap = type == 1 ? args.Acs : args.A;
  const int64_t lda = type == 1 ? args.ld_acs : args.lda;
  const float *Bp = type == 2 ? args.Bcs : args.B;
  const int64_t ldb = type == 2 ? args.ld_bcs : args.ldb;
  const int64_t rows_valid = type == 1 ? args.Mcs : args.M;
  const int64_t cols_valid = type == 2 ? args.Ncs : args.N;
  const int64_t K = args.K;

  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  const int a_row = tid >> 1, a_k = (tid & 1) * 4;
  const int b_k = tid >> 5, b_n = (tid & 31) * 4;

  int nf = 0;
  if (args.nfaults > 0) {
    if (tid == 0) s_nf = 0;
    __syncthreads();
    for (int f = tid; f < args.nfaults; f += THREADS) {
      const aabft_fault ft = args.faults[f];
      int64_t r = ft.row, c = ft.col;
      bool hit;
      if (type == 0) hit = r < args.M && c < args.N;
      else if (type == 1) { hit = r >= args.M && c < args.N; r -= args.M; }
      else { hit = c >= args.N && r < args.M; c -= args.N; }
      if (hit && r >= m0 && r < m0 + BM && c >= n0 && c < n0 + BN) {
        const int slot = atomicAdd(&s_nf, 1);
        if (slot < MAXF) {
          aabft_fault loc = ft;
          loc.row = r - m0;
          loc.col = c - n0;
          s_f[slot] = loc;
        }
      }
    }
    __syncthreads();
    nf = min(s_nf, MAXF);
  }

  float acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;

  const int nk = (int)((K + BK - 1) / BK);
  float4 ra = load4(Ap, lda, m0 + a_row, rows_valid, a_k, K);
  float4 rb = load4(Bp, ldb, b_k, K, n0 + b_n, cols_valid);
  As[0][a_k + 0][a_row] = ra.x;
  As[0][a_k + 1][a_row] = ra.y;
  As[0][a_k + 2][a_row] = ra.z;
  As[0][a_k + 3][a_row] = ra.w;
  *reinterpret_cast<float4 *>(&Bs[0][b_k][b_n]) = rb;
  __syncthreads();

  for (int kt = 0; kt < nk; ++kt) {
    const int cur = kt & 1;
    if (kt + 1 < nk) {
      const int64_t k0 = (int64_t)(kt + 1) * BK;
      ra = load4(Ap, lda, m0 + a_row, rows_valid, k0 + a_k, K);
      rb = load4(Bp, ldb, k0 + b_k, K, n0 + b_n, cols_valid);
    }
#pragma unroll
    for (int k = 0; k < BK; ++k) {
      const float4 a0 = *reinterpret_cast<const float4 *>(&As[cur][k][ty * 4]);
      const float4 a1 = *reinterpret_cast<const float4 *>(&As[cur][k][64 + ty * 4]);
      const float4 b0 = *reinterpret_cast<const float4 *>(&Bs[cur][k][tx * 4]);
      const float4 b1 = *reinterpret_cast<const float4 *>(&Bs[cur][k][64 + tx * 4]);
      const float av[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
      const float bv[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
    }
    if (nf > 0) {
      for (int f = 0; f < nf; ++f) {
        const aabft_fault ft = s_f[f];
        if (ft.site != 1 || ft.k_step / BK != kt) continue;
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int j = 0; j < 8; ++j) {
            const int r = (i < 4 ? ty * 4 + i : 64 + ty * 4 + i - 4);
            const int c = (j < 4 ? tx * 4 + j : 64 + tx * 4 + j - 4);
            if (r == ft.row && c == ft.col) acc[i][j] = xor_bits(acc[i][j], ft.xor_mask);
          }
      }
    }
    if (kt + 1 < nk) {
      const int nxt = cur ^ 1;
      As[nxt][a_k + 0][a_row] = ra.x;
      As[nxt][a_k + 1][a_row] = ra.y;
      As[nxt][a_k + 2][a_row] = ra.z;
      As[nxt][a_k + 3][a_row] = ra.w;
      *reinterpret_cast<float4 *>(&Bs[nxt][b_k][b_n]) = rb;
    }
    __syncthreads();
  }

  if (nf > 0) {
    for (int f = 0; f < nf; ++f) {
      const aabft_fault ft = s_f[f];
      if (ft.site == 1) continue;
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int r = (i < 4 ? ty * 4 + i : 64 + ty * 4 + i - 4);
          const int c = (j < 4 ? tx * 4 + j : 64 + tx * 4 + j - 4);
          if (r == ft.row && c == ft.col)
            acc[i][j] = ft.site == 0 ? xor_bits(acc[i][j], ft.xor_mask)
                                     : (float)((double)acc[i][j] + ft.add);
        }
    }
  }
  float *out;
  int64_t ld;
  if (type == 0) { out = args.C; ld = args.ldc; }
  else if (type == 1) { out = args.Ccol; ld = args.ld_ccol; }
  else { out = args.Crow; ld = args.ld_crow; }
  const bool vec_ok = (ld % 4 == 0) && ((reinterpret_cast<uintptr_t>(out) & 15) == 0);
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int64_t r = m0 + (i < 4 ? ty * 4 + i : 64 + ty * 4 + i - 4);
    if (r >= rows_valid) continue;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int64_t c = n0 + h * 64 + tx * 4;
      float *p = out + r * ld + c;
      if (c + 3 < cols_valid && vec_ok) {
        *reinterpret_cast<float4 *>(p) =
            make_float4(acc[i][h * 4], acc[i][h * 4 + 1], acc[i][h * 4 + 2], acc[i][h * 4 + 3]);
      } else {
#pragma unroll
        for (int j = 0; j < 4; ++j)
          if (c + j < cols_valid) p[j] = acc[i][h * 4 + j];
      }
    }
  }
}

}  // namespace

aabft_status launch_gemm_f32(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                             int64_t ldb, const aabft_encoded *enc, const aabft_product *out,
                             const aabft_fault *faults, int32_t nfaults, bool plain,
                             cudaStream_t st) {
  const int64_t M = cfg->M, N = cfg->N, K = cfg->K, bs = cfg->bs;
  SgemmArgs a{};
  a.A = static_cast<const float *>(A); a.lda = lda;
  a.B = static_cast<const float *>(B); a.ldb = ldb;
  a.Acs = plain ? nullptr : static_cast<const float *>(enc->Acs);
  a.ld_acs = plain ? 0 : enc->ld_acs;
  a.Bcs = plain ? nullptr : static_cast<const float *>(enc->Bcs);
  a.ld_bcs = plain ? 0 : enc->ld_bcs;
  a.M = M; a.N = N; a.K = K;
  a.Mcs = plain ? 0 : M / bs;
  a.Ncs = plain ? 0 : N / bs;
  a.C = static_cast<float *>(out->C); a.ldc = out->ldc;
  a.Ccol = plain ? nullptr : static_cast<float *>(out->Ccol);
  a.ld_ccol = plain ? 0 : out->ld_ccol;
  a.Crow = plain ? nullptr : static_cast<float *>(out->Crow);
  a.ld_crow = plain ? 0 : out->ld_crow;
  a.tm0 = (int)((M + BM - 1) / BM);
  a.tn0 = (int)((N + BN - 1) / BN);
  a.tm1 = plain ? 0 : (int)((a.Mcs + BM - 1) / BM);
  a.tn2 = plain ? 0 : (int)((a.Ncs + BN - 1) / BN);
  a.n0 = (int64_t)a.tm0 * a.tn0;
  a.n1 = (int64_t)a.tm1 * a.tn0;
  a.n2 = (int64_t)a.tm0 * a.tn2;
  a.faults = faults;
  a.nfaults = faults ? nfaults : 0;
  const int64_t tiles = a.n0 + a.n1 + a.n2;
  if (tiles > 0) {
    gemm_f32_kernel<<<(unsigned)tiles, THREADS, 0, st>>>(a);
    next_launch();
  }
  return check_launch("aabft_gemm(f32)");
}

}  // namespace aabft
