// gemm_f32.cu -- step 2 of A-ABFT (Eq 3) for FP32 on the FFMA pipe (no TF32: a
// tensor-core TF32 product would change the rounding model the bound assumes, north_star).
//
// B200 design: 128 x 128 x 32 CTA tiles, 256 threads, 8 x 8 register
// micro-tiles split 2 x 2 (rows ty*4 / 64+ty*4, cols tx*4 / 64+tx*4), a 2-stage cp.async
// (LDGSTS) shared-memory ring, LDS.128 fragments and sm_100 FFMA2 (packed fp32x2 FMA).
// (BK 32 x 2 stages measured 54.8 TFLOP/s at 8192^3 against 50.4 for BK 16 x 3, 51.2 for
// 32 x 3, 52.6 for 16 x 4, 49.8 for 48 x 2: half the CTA barriers per FMA, 2 CTAs/SM.)  Every
// element accumulates c = fma(a_k, b_k, c) in ascending k, which is exactly the fused
// sequential inner product of Eq 15 / §IV-D -- the FP32 product is bit-identical to the
// definition.  Same three tile types as the FP64 kernel (C, Ccol, Crow).  Fault injection
// (Alg 3) is a separate instantiation (FAULTS = true, launched only with a fault
// list) and is instruction-exact: a thread owning a fault whose k_step falls in the current
// k-tile replays that k-tile step by step in scalar code -- site 4 rounds the product on its
// own and XORs it ("errorVecMul"), sites 1 / 3 hit the accumulator right after step k_step
// ("errorVecAdd1") -- so a faulty FP32 product equals the oracle's dot_fault bit for bit.
#include <atomic>

#include "common.cuh"

namespace aabft {
namespace {

#ifndef AABFT_F32_BN
#define AABFT_F32_BN 128
#endif
#ifndef AABFT_F32_BK
#define AABFT_F32_BK 32
#endif
#ifndef AABFT_F32_STAGES
#define AABFT_F32_STAGES 2
#endif
constexpr int BM = 128, BN = AABFT_F32_BN, BK = AABFT_F32_BK, STAGES = AABFT_F32_STAGES;
constexpr int TX = BN / 8, THREADS = 16 * TX;   // 16 x TX threads, 8 x 8 outputs each
constexpr int HN = BN / 2;                      // column offset of the second 4-wide half
constexpr int MAXF = BM * BN / 64;  // faults per tile kept in smem (one per 8x8 block)
constexpr int RING32 = STAGES * (BM + BN) * BK * 4;
constexpr int TILE32 = BM * (BN + 1) * 4;  // fused-sum epilogue staging (reuses the ring)
constexpr int SMEM32 = (RING32 > TILE32 ? RING32 : TILE32) + MAXF * (int)sizeof(aabft_fault);
#ifndef AABFT_F32_SCALAR
#define AABFT_F32_SCALAR 0
#endif
#ifndef AABFT_F32_JOUTER
#define AABFT_F32_JOUTER 1  // measured 20.42 vs 20.61 ms at 8192^3
#endif
#ifndef AABFT_F32_GROUP_M
#define AABFT_F32_GROUP_M 8
#endif
constexpr int GROUP_M = AABFT_F32_GROUP_M;

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
  double *Rcol;  // fused reference sums (NULL = unfused): (M/bs) x N, M x (N/bs)
  double *Rrow;
  int bs;
  unsigned long long *check_acc;  // the following aabft_check's counter accumulator: zeroed
};

__device__ __forceinline__ float xor_bits(float v, uint64_t m) {
  return __int_as_float(__float_as_int(v) ^ (int)(uint32_t)m);
}

// 16-byte cp.async (LDGSTS) with zero-fill of the bytes beyond `valid` (0..16)
__device__ __forceinline__ void cp_async16(void *smem, const void *gmem, int valid) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(smem)),
               "l"(gmem), "r"(valid)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

template <bool FAULTS>
#ifndef AABFT_F32_MINB
#define AABFT_F32_MINB (THREADS >= 512 ? 1 : 2)
#endif
__global__ void __launch_bounds__(THREADS, AABFT_F32_MINB) gemm_f32_kernel(const SgemmArgs args) {
  // cp.async ring: A tile [128 rows][BK k] (k contiguous, as in memory), B tile
  // [BK k][128 cols].  A fragments are LDS.128 along k (4 k-steps of one row), B fragments
  // LDS.128 along n; the 8 x 8 micro-tile runs as 32 FFMA2 per k-step (sm_100 packed fp32x2
  // FMA, A broadcast) -- each lane rounded once, exactly fmaf.
  extern __shared__ __align__(16) uint8_t smem32[];
  auto As = reinterpret_cast<float(*)[BM][BK]>(smem32);                          // [STAGES]
  auto Bs = reinterpret_cast<float(*)[BK][BN]>(smem32 + STAGES * BM * BK * 4);   // [STAGES]
  aabft_fault *s_f = reinterpret_cast<aabft_fault *>(smem32 + (RING32 > TILE32 ? RING32 : TILE32));
  __shared__ int s_nf;

  if (blockIdx.x == 0 && threadIdx.x < 10 && args.check_acc) args.check_acc[threadIdx.x] = 0ull;
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

  const int tid = threadIdx.x, tx = tid % TX, ty = tid / TX;

  int nf = 0;
  if (FAULTS && args.nfaults > 0) {
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

  // tile loaders: 2 x 16-byte chunks of A and of B per thread per k-tile
  auto load_tile = [&](int stage, int kt) {
    const int64_t k0 = (int64_t)kt * BK;
#pragma unroll
    for (int c = 0; c < BM * BK / 4 / THREADS; ++c) {
      const int e = tid + c * THREADS;
      const int ar = e / (BK / 4), ak = (e % (BK / 4)) * 4;  // A: row ar, k ak..ak+3
      const int64_t gr = m0 + ar, gk = k0 + ak;
      const int av = (gr < rows_valid && gk < K) ? (int)((K - gk) * 4 < 16 ? (K - gk) * 4 : 16) : 0;
      cp_async16(&As[stage][ar][ak], av ? (const void *)(Ap + gr * lda + gk) : (const void *)Ap, av);
    }
#pragma unroll
    for (int c = 0; c < BK * BN / 4 / THREADS; ++c) {
      const int e = tid + c * THREADS;
      const int bk = e / (BN / 4), bn = (e % (BN / 4)) * 4;  // B: k row bk, cols bn..bn+3
      const int64_t gkb = k0 + bk, gn = n0 + bn;
      const int bv = (gkb < K && gn < cols_valid) ? (int)((cols_valid - gn) * 4 < 16 ? (cols_valid - gn) * 4 : 16) : 0;
      cp_async16(&Bs[stage][bk][bn], bv ? (const void *)(Bp + gkb * ldb + gn) : (const void *)Bp, bv);
    }
  };

  float2 acc2[8][4];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc2[i][j] = make_float2(0.f, 0.f);
#define ACC(i, j) (((j) & 1) ? acc2[i][(j) >> 1].y : acc2[i][(j) >> 1].x)

  const int nk = (int)((K + BK - 1) / BK);
#pragma unroll
  for (int st = 0; st < STAGES - 1; ++st) {
    if (st < nk) load_tile(st, st);
    cp_async_commit();
  }
  for (int kt = 0; kt < nk; ++kt) {
    cp_async_wait<STAGES - 2>();
    __syncthreads();  // tile kt visible to all; the stage consumed at kt-1 is free
    if (kt + STAGES - 1 < nk) load_tile((kt + STAGES - 1) % STAGES, kt + STAGES - 1);
    cp_async_commit();
    const int cur = kt % STAGES;
    if (FAULTS && nf > 0) {
      // this thread's in-loop faults (sites 1, 3, 4) whose k_step falls inside k-tile kt
      int myf[4], nmy = 0;
      for (int f = 0; f < nf; ++f) {
        const aabft_fault &ft = s_f[f];
        if ((ft.site == 1 || ft.site == 3 || ft.site == 4) && ft.k_step / BK == kt &&
            ((ft.row & 63) >> 2) == ty && ((ft.col % HN) >> 2) == tx && nmy < 4)
          myf[nmy++] = f;
      }
      if (nmy > 0) {  // scalar replay of this k-tile, step by step (ascending k, as Alg 3)
        for (int kk = 0; kk < BK; ++kk) {
          const int64_t k = (int64_t)kt * BK + kk;
          if (k >= K) break;
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const int r = i < 4 ? ty * 4 + i : 64 + ty * 4 + (i - 4);
            const float av = As[cur][r][kk];
#pragma unroll
            for (int j = 0; j < 8; ++j) {
              const int c = j < 4 ? tx * 4 + j : HN + tx * 4 + (j - 4);
              const float bv = Bs[cur][kk][c];
              float acc = ACC(i, j);
              int site = -1;
              uint64_t mask = 0;
              double add = 0.0;
              for (int q = 0; q < nmy; ++q) {
                const aabft_fault &ft = s_f[myf[q]];
                if (ft.row == r && ft.col == c && ft.k_step == k) {
                  site = ft.site; mask = ft.xor_mask; add = ft.add;
                }
              }
              if (site == 4) acc = __fadd_rn(acc, xor_bits(__fmul_rn(av, bv), mask));
              else acc = __fmaf_rn(av, bv, acc);
              if (site == 1) acc = xor_bits(acc, mask);
              if (site == 3) acc = (float)((double)acc + add);
              ACC(i, j) = acc;
            }
          }
        }
        continue;
      }
    }
#pragma unroll
    for (int k4 = 0; k4 < BK / 4; ++k4) {
      float4 a4[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int r = i < 4 ? ty * 4 + i : 64 + ty * 4 + (i - 4);
        a4[i] = *reinterpret_cast<const float4 *>(&As[cur][r][k4 * 4]);
      }
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        const float4 b0 = *reinterpret_cast<const float4 *>(&Bs[cur][k4 * 4 + kk][tx * 4]);
        const float4 b1 = *reinterpret_cast<const float4 *>(&Bs[cur][k4 * 4 + kk][HN + tx * 4]);
        const float2 bv[4] = {make_float2(b0.x, b0.y), make_float2(b0.z, b0.w),
                              make_float2(b1.x, b1.y), make_float2(b1.z, b1.w)};
#if AABFT_F32_JOUTER  // experiment: the B pair is the operand re-used by consecutive FFMA2
#pragma unroll
        for (int j = 0; j < 4; ++j)
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const float av = kk == 0 ? a4[i].x : (kk == 1 ? a4[i].y : (kk == 2 ? a4[i].z : a4[i].w));
#if AABFT_F32_SCALAR  // experiment: scalar FFMA (higher pipe ceiling, twice the instructions)
            acc2[i][j].x = __fmaf_rn(av, bv[j].x, acc2[i][j].x);
            acc2[i][j].y = __fmaf_rn(av, bv[j].y, acc2[i][j].y);
#else
            acc2[i][j] = __ffma2_rn(make_float2(av, av), bv[j], acc2[i][j]);
#endif
          }
#else
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const float av = kk == 0 ? a4[i].x : (kk == 1 ? a4[i].y : (kk == 2 ? a4[i].z : a4[i].w));
#pragma unroll
          for (int j = 0; j < 4; ++j) acc2[i][j] = __ffma2_rn(make_float2(av, av), bv[j], acc2[i][j]);
        }
#endif
      }
    }
  }
  cp_async_wait<0>();

  if (FAULTS && nf > 0) {  // sites 0 / 2: the stored result ("errorVecAdd2")
    for (int f = 0; f < nf; ++f) {
      const aabft_fault ft = s_f[f];
      if (ft.site != 0 && ft.site != 2) continue;
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int r = (i < 4 ? ty * 4 + i : 64 + ty * 4 + i - 4);
          const int c = (j < 4 ? tx * 4 + j : HN + tx * 4 + j - 4);
          if (r == ft.row && c == ft.col)
            ACC(i, j) = ft.site == 0 ? xor_bits(ACC(i, j), ft.xor_mask)
                                     : (float)((double)ACC(i, j) + ft.add);
        }
    }
  }
  if (type == 0 && args.Rcol != nullptr) {
    // ---- fused reference sums (Eq 4, in double, reading R12) of the BS x BS blocks of this
    // 128 x 128 tile, from the registers about to be stored (after any injected fault): the
    // check compares them instead of re-reading C (the FP64 kernel's design).  The tile goes
    // through shared memory (the drained cp.async ring; odd pitch 129: conflict-free column AND
    // row walks), then thread c < 128 sums column c down each block and thread 128 + r sums
    // row r across each block, both in ascending order -- the definition's sequential order,
    // so these sums equal the unfused check's bit for bit.
    const int bs = args.bs;
    __syncthreads();  // every warp is done with the stage buffers
    float *s_tile = reinterpret_cast<float *>(smem32);  // [BM][BN + 1]
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int r = i < 4 ? ty * 4 + i : 64 + ty * 4 + i - 4;
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const int c = j < 4 ? tx * 4 + j : HN + tx * 4 + (j - 4);
        s_tile[r * (BN + 1) + c] = ACC(i, j);
      }
    }
    __syncthreads();
    if (tid < BN) {  // column sums: rows of each block in ascending order
      const int c = tid;
      const int64_t col = n0 + c;
      for (int r0 = 0; r0 < BM; r0 += bs) {
        double sum = 0.0;
        for (int r = r0; r < r0 + bs; ++r) sum = sum + (double)s_tile[r * (BN + 1) + c];
        if (m0 + r0 < args.M && col < args.N) args.Rcol[((m0 + r0) / bs) * args.N + col] = sum;
      }
    } else if (tid < BN + BM) {  // row sums: columns of each block in ascending order
      const int r = tid - BN;
      const int64_t row = m0 + r, nJ = args.N / bs;
      for (int c0 = 0; c0 < BN; c0 += bs) {
        double sum = 0.0;
        for (int c = c0; c < c0 + bs; ++c) sum = sum + (double)s_tile[r * (BN + 1) + c];
        const int64_t J = (n0 + c0) / bs;
        if (row < args.M && J < nJ) args.Rrow[row * nJ + J] = sum;
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
      const int64_t c = n0 + h * HN + tx * 4;
      float *p = out + r * ld + c;
      if (c + 3 < cols_valid && vec_ok) {
        *reinterpret_cast<float4 *>(p) =
            make_float4(ACC(i, h * 4), ACC(i, h * 4 + 1), ACC(i, h * 4 + 2), ACC(i, h * 4 + 3));
      } else {
#pragma unroll
        for (int j = 0; j < 4; ++j)
          if (c + j < cols_valid) p[j] = ACC(i, h * 4 + j);
      }
    }
  }
#undef ACC
}

}  // namespace

aabft_status launch_gemm_f32(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                             int64_t ldb, const aabft_encoded *enc, const aabft_product *out,
                             const aabft_fault *faults, int32_t nfaults, bool plain,
                             unsigned long long *check_acc, cudaStream_t st) {
  const int64_t M = cfg->M, N = cfg->N, K = cfg->K, bs = cfg->bs;
  SgemmArgs a{};
  a.check_acc = plain ? nullptr : check_acc;
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
  a.bs = (int)bs;
  const bool fused = !plain && out->Rcol && out->Rrow && fused_check_ok(cfg);
  a.Rcol = fused ? out->Rcol : nullptr;
  a.Rrow = fused ? out->Rrow : nullptr;
  const int64_t tiles = a.n0 + a.n1 + a.n2;
  static std::atomic<bool> attr_dev[64];  // per device (function attributes are per context)
  int dev = 0;
  cudaGetDevice(&dev);
  if (!attr_dev[dev & 63].load(std::memory_order_relaxed)) {
    if (cudaFuncSetAttribute(gemm_f32_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM32) != cudaSuccess ||
        cudaFuncSetAttribute(gemm_f32_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM32) != cudaSuccess)
      return check_launch("gemm_f32 smem attribute");
    attr_dev[dev & 63].store(true, std::memory_order_relaxed);
  }
  if (tiles > 0) {
    if (a.nfaults > 0) gemm_f32_kernel<true><<<(unsigned)tiles, THREADS, SMEM32, st>>>(a);
    else gemm_f32_kernel<false><<<(unsigned)tiles, THREADS, SMEM32, st>>>(a);
    next_launch();
  }
  return check_launch("aabft_gemm(f32)");
}

}  // namespace aabft
