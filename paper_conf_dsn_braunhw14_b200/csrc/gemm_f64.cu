// gemm_f64.cu -- step 2 of A-ABFT (Eq 3) on sm_100a: the checksum-augmented
// FP64 GEMM on the DMMA tensor-core pipe, with Alg 3 fault-injection hooks.
//
// B200 design:
//  * tcgen05.mma has no f64 kind, so the FP64 tensor path is warp-level
//    mma.sync.aligned.m16n8k4.row.col.f64 (SASS DMMA); measured issue ceiling 37.0 TFLOP/s
//    (profiles/r01_step0_pipes.jsonl) vs 34 TFLOP/s for DFMA.
//  * One elected thread issues TMA (cp.async.bulk.tensor) into a 4-stage shared-memory ring
//    guarded by full/empty mbarriers; 8 MMA warps (2 x 4, 64 x 32 warp tiles) read swizzled
//    fragments with conflict-free 64-bit LDS and issue 16 DMMAs per k4-step.
//    A tiles use the 128B swizzle (box 16 k x 128 rows), B tiles are 16 boxes of 8 columns x
//    16 k with the 64B swizzle -- both make the m16n8k4 fragment loads bank-conflict free.
//  * One launch computes all three products of Eq 3 with partitioned checksums: C = A.B,
//    Ccol = Acs.B (checksum rows as their own tiles), Crow = A.Bcs (checksum columns as
//    their own tiles).  The corner Acs.Bcs is never formed (reading R17).
//  * Fault hooks: a CTA copies the faults that hit its tile into shared memory; site 1 XORs
//    the accumulator after the k-tile containing k_step, sites 0/2 act on the stored value.
#include <cudaTypedefs.h>

#include "common.cuh"

namespace aabft {
namespace {

constexpr int BM = 128, BN = 128, BK = 16, STAGES = 4;
constexpr int NCW = 8;                     // MMA warps (2 x 4)
constexpr int THREADS = NCW * 32;          // 256: 2 warps / SMSP -> up to 255 registers
constexpr int A_BYTES = BM * BK * 8;       // 16 KiB
constexpr int B_BYTES = BK * BN * 8;       // 16 KiB
constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
constexpr int MAXF = 16;                   // faults per tile kept in smem
constexpr int SMEM_BYTES = STAGES * STAGE_BYTES + 1024 /*align*/ + 256 /*barriers*/ +
                           MAXF * (int)sizeof(aabft_fault) + 16;
constexpr int GROUP_M = 8;

struct GemmArgs {
  int64_t M, N, K, Mcs, Ncs;
  double *C;
  int64_t ldc;
  double *Ccol;
  int64_t ld_ccol;
  double *Crow;
  int64_t ld_crow;
  int64_t n0, n1, n2;       // tiles of type 0 (data), 1 (column checksums), 2 (row checksums)
  int tm0, tn0, tm1, tn2;   // tile grid dims
  int nk;
  const aabft_fault *faults;
  int nfaults;
};

__device__ __forceinline__ int swz128(int r, int k) {  // A tile [128 rows][16 k] doubles
  return r * 16 + ((((k >> 1) ^ (r & 7)) << 1) | (k & 1));
}
__device__ __forceinline__ int swz64(int k, int n) {   // B sub-box [16 k][8 n] doubles
  return k * 8 + ((((n >> 1) ^ ((k >> 1) & 3)) << 1) | (n & 1));
}

__device__ __forceinline__ void dmma(double (&c)[4], double a0, double a1, double b) {
  asm volatile(
      "mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, "
      "{%0,%1,%2,%3};"
      : "+d"(c[0]), "+d"(c[1]), "+d"(c[2]), "+d"(c[3])
      : "d"(a0), "d"(a1), "d"(b));
}

__device__ __forceinline__ double xor_bits(double v, uint64_t m) {
  return __longlong_as_double(__double_as_longlong(v) ^ (long long)m);
}

__global__ void __launch_bounds__(THREADS, 1)
    gemm_f64_kernel(const __grid_constant__ CUtensorMap tmA,
                    const __grid_constant__ CUtensorMap tmAcs,
                    const __grid_constant__ CUtensorMap tmB,
                    const __grid_constant__ CUtensorMap tmBcs, const GemmArgs args) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                              ~uintptr_t(1023));
  uint64_t *full = reinterpret_cast<uint64_t *>(smem + STAGES * STAGE_BYTES);
  uint64_t *empty = full + STAGES;
  int *s_nf = reinterpret_cast<int *>(empty + STAGES);
  aabft_fault *s_f = reinterpret_cast<aabft_fault *>(smem + STAGES * STAGE_BYTES + 256);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  // ---- tile decode (type 0 grouped raster for L2 reuse)
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
  const int m0 = tm * BM, n0 = tn * BN;
  const int64_t rows_valid = type == 1 ? args.Mcs : args.M;
  const int64_t cols_valid = type == 2 ? args.Ncs : args.N;

  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], NCW);
    }
    *s_nf = 0;
    fence_barrier_init();
  }
  __syncthreads();

  // Producer role: thread 0 issues TMA.  Prologue fills the ring; afterwards, at the top of
  // k-tile kt it refills the slot consumed at kt-1 once all 8 warps released it (empty
  // barrier), so the refill lags the slowest warp by one k-tile and never blocks the MMAs of
  // the stages already resident.  (A dedicated 9th producer warp would cap registers at 168:
  // 3 warps on one SMSP.)
  const CUtensorMap *ta = type == 1 ? &tmAcs : &tmA;
  const CUtensorMap *tb = type == 2 ? &tmBcs : &tmB;
  auto issue = [&](int kt) {
    const int s = kt % STAGES;
    uint8_t *sa = smem + s * STAGE_BYTES;
    uint8_t *sb = sa + A_BYTES;
    mbar_arrive_expect_tx(&full[s], STAGE_BYTES);
    tma_load_2d(sa, ta, &full[s], kt * BK, m0);
#pragma unroll
    for (int b = 0; b < BN / 8; ++b) tma_load_2d(sb + b * 1024, tb, &full[s], n0 + b * 8, kt * BK);
  };
  if (threadIdx.x == 0) {
    tma_prefetch_desc(ta);
    tma_prefetch_desc(tb);
    for (int kt = 0; kt < STAGES && kt < args.nk; ++kt) issue(kt);
  }

  // ================= consumers
  const int wm = warp >> 2, wn = warp & 3;  // 2 x 4 warps, 64 x 32 warp tiles
  const int g = lane >> 2, tig = lane & 3;

  // collect faults that hit this tile (C_fc coordinates -> tile-local)
  int nf = 0;
  if (args.nfaults > 0) {
    for (int f = threadIdx.x; f < args.nfaults; f += NCW * 32) {
      const aabft_fault ft = args.faults[f];
      int64_t r = ft.row, c = ft.col;
      bool hit;
      if (type == 0) hit = r < args.M && c < args.N;
      else if (type == 1) { hit = r >= args.M && c < args.N; r -= args.M; }
      else { hit = c >= args.N && r < args.M; c -= args.N; }
      if (hit && r >= m0 && r < m0 + BM && c >= n0 && c < n0 + BN) {
        const int slot = atomicAdd(s_nf, 1);
        if (slot < MAXF) {
          aabft_fault loc = ft;
          loc.row = r - m0;
          loc.col = c - n0;
          s_f[slot] = loc;
        }
      }
    }
    __syncthreads();
    nf = min(*s_nf, MAXF);
  }

  double acc[4][4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j)
#pragma unroll
      for (int q = 0; q < 4; ++q) acc[i][j][q] = 0.0;

  for (int kt = 0; kt < args.nk; ++kt) {
    const int s = kt % STAGES;
    if (threadIdx.x == 0 && kt >= 1 && kt - 1 + STAGES < args.nk) {
      mbar_wait(&empty[(kt - 1) % STAGES], ((kt - 1) / STAGES) & 1);
      issue(kt - 1 + STAGES);
    }
    mbar_wait(&full[s], (kt / STAGES) & 1);
    const double *sa = reinterpret_cast<const double *>(smem + s * STAGE_BYTES);
    const double *sb = reinterpret_cast<const double *>(smem + s * STAGE_BYTES + A_BYTES);
#pragma unroll
    for (int ks = 0; ks < BK / 4; ++ks) {
      const int k = ks * 4 + tig;
      double a[4][2], b[4];
#pragma unroll
      for (int mt = 0; mt < 4; ++mt) {
        const int r = wm * 64 + mt * 16 + g;
        a[mt][0] = sa[swz128(r, k)];
        a[mt][1] = sa[swz128(r + 8, k)];
      }
#pragma unroll
      for (int nt = 0; nt < 4; ++nt) b[nt] = sb[(wn * 4 + nt) * 128 + swz64(k, g)];
#pragma unroll
      for (int mt = 0; mt < 4; ++mt)
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) dmma(acc[mt][nt], a[mt][0], a[mt][1], b[nt]);
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[s]);
    if (nf > 0) {  // Alg 3 errorVecAdd1 at k-tile granularity
      for (int f = 0; f < nf; ++f) {
        const aabft_fault ft = s_f[f];
        if (ft.site != 1 || ft.k_step / BK != kt) continue;
#pragma unroll
        for (int mt = 0; mt < 4; ++mt)
#pragma unroll
          for (int nt = 0; nt < 4; ++nt)
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const int r = wm * 64 + mt * 16 + g + (q >> 1) * 8;
              const int c = wn * 32 + nt * 8 + tig * 2 + (q & 1);
              if (r == ft.row && c == ft.col) acc[mt][nt][q] = xor_bits(acc[mt][nt][q], ft.xor_mask);
            }
      }
    }
  }

  // ================= epilogue: faults on the stored value, then masked 16-byte stores
  if (nf > 0) {
    for (int f = 0; f < nf; ++f) {
      const aabft_fault ft = s_f[f];
      if (ft.site == 1) continue;
#pragma unroll
      for (int mt = 0; mt < 4; ++mt)
#pragma unroll
        for (int nt = 0; nt < 4; ++nt)
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            const int r = wm * 64 + mt * 16 + g + (q >> 1) * 8;
            const int c = wn * 32 + nt * 8 + tig * 2 + (q & 1);
            if (r == ft.row && c == ft.col)
              acc[mt][nt][q] = ft.site == 0 ? xor_bits(acc[mt][nt][q], ft.xor_mask)
                                            : acc[mt][nt][q] + ft.add;
          }
    }
  }
  double *out;
  int64_t ld;
  if (type == 0) { out = args.C; ld = args.ldc; }
  else if (type == 1) { out = args.Ccol; ld = args.ld_ccol; }
  else { out = args.Crow; ld = args.ld_crow; }
  const bool vec_ok = (ld % 2 == 0) && ((reinterpret_cast<uintptr_t>(out) & 15) == 0);
#pragma unroll
  for (int mt = 0; mt < 4; ++mt)
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int64_t r = m0 + wm * 64 + mt * 16 + g + h * 8;
      if (r >= rows_valid) continue;
#pragma unroll
      for (int nt = 0; nt < 4; ++nt) {
        const int64_t c = n0 + wn * 32 + nt * 8 + tig * 2;
        double *p = out + r * ld + c;
        const double v0 = acc[mt][nt][h * 2], v1 = acc[mt][nt][h * 2 + 1];
        if (c + 1 < cols_valid && vec_ok) {
          *reinterpret_cast<double2 *>(p) = make_double2(v0, v1);
        } else {
          if (c < cols_valid) p[0] = v0;
          if (c + 1 < cols_valid) p[1] = v1;
        }
      }
    }
}

PFN_cuTensorMapEncodeTiled_v12000 get_encoder() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void *p = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) ==
            cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  }
  return fn;
}

bool make_map(CUtensorMap *m, const void *base, uint64_t inner, uint64_t outer, uint64_t ld_elems,
              uint32_t box_inner, uint32_t box_outer, CUtensorMapSwizzle sw) {
  auto enc = get_encoder();
  if (!enc) {
    set_error("cuTensorMapEncodeTiled unavailable");
    return false;
  }
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {ld_elems * 8};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, const_cast<void *>(base), dims, strides,
                   box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    set_error("cuTensorMapEncodeTiled failed (%d): inner=%llu outer=%llu ld=%llu", (int)r,
              (unsigned long long)inner, (unsigned long long)outer,
              (unsigned long long)ld_elems);
    return false;
  }
  return true;
}

}  // namespace

aabft_status launch_gemm_f64(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                             int64_t ldb, const aabft_encoded *enc, const aabft_product *out,
                             const aabft_fault *faults, int32_t nfaults, bool plain,
                             cudaStream_t st) {
  static bool attr_set = false;
  if (!attr_set) {
    if (cudaFuncSetAttribute(gemm_f64_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             SMEM_BYTES) != cudaSuccess)
      return check_launch("gemm_f64 smem attribute");
    attr_set = true;
  }
  const int64_t M = cfg->M, N = cfg->N, K = cfg->K, bs = cfg->bs;
  GemmArgs a{};
  a.M = M; a.N = N; a.K = K;
  a.Mcs = plain ? 0 : M / bs;
  a.Ncs = plain ? 0 : N / bs;
  a.C = static_cast<double *>(out->C); a.ldc = out->ldc;
  a.Ccol = plain ? nullptr : static_cast<double *>(out->Ccol);
  a.ld_ccol = plain ? 0 : out->ld_ccol;
  a.Crow = plain ? nullptr : static_cast<double *>(out->Crow);
  a.ld_crow = plain ? 0 : out->ld_crow;
  a.tm0 = (int)((M + BM - 1) / BM);
  a.tn0 = (int)((N + BN - 1) / BN);
  a.tm1 = plain ? 0 : (int)((a.Mcs + BM - 1) / BM);
  a.tn2 = plain ? 0 : (int)((a.Ncs + BN - 1) / BN);
  a.n0 = (int64_t)a.tm0 * a.tn0;
  a.n1 = (int64_t)a.tm1 * a.tn0;
  a.n2 = (int64_t)a.tm0 * a.tn2;
  a.nk = (int)((K + BK - 1) / BK);
  a.faults = faults;
  a.nfaults = faults ? nfaults : 0;

  CUtensorMap tA, tAcs, tB, tBcs;
  if (!make_map(&tA, A, K, M, lda, BK, BM, CU_TENSOR_MAP_SWIZZLE_128B)) return AABFT_EINVAL;
  if (!make_map(&tB, B, N, K, ldb, 8, BK, CU_TENSOR_MAP_SWIZZLE_64B)) return AABFT_EINVAL;
  if (plain) {
    tAcs = tA;
    tBcs = tB;
  } else {
    if (!make_map(&tAcs, enc->Acs, K, a.Mcs, enc->ld_acs, BK, BM, CU_TENSOR_MAP_SWIZZLE_128B))
      return AABFT_EINVAL;
    if (!make_map(&tBcs, enc->Bcs, a.Ncs, K, enc->ld_bcs, 8, BK, CU_TENSOR_MAP_SWIZZLE_64B))
      return AABFT_EINVAL;
  }
  const int64_t tiles = a.n0 + a.n1 + a.n2;
  if (tiles > 0) {
    gemm_f64_kernel<<<(unsigned)tiles, THREADS, SMEM_BYTES, st>>>(tA, tAcs, tB, tBcs, a);
    next_launch();
  }
  return check_launch("aabft_gemm(f64)");
}

}  // namespace aabft
