// gemm_f64.cu -- step 2 of A-ABFT (Eq 3) on sm_100a: the checksum-augmented
// FP64 GEMM on the DMMA tensor-core pipe, with Alg 3 fault-injection hooks.
//
// B200 design:
//  * tcgen05.mma has no f64 kind, so the FP64 tensor path is warp-level
//    mma.sync.aligned.m16n8k4.row.col.f64 (SASS DMMA.8x8x4: 512 flop, one per 16 cycles per
//    SM sub-partition; measured ceiling 37.0 TFLOP/s, profiles/r01_step0_pipes.jsonl).
//  * The DMMA pipe is kept busy by many INDEPENDENT warps rather than big register tiles:
//    64 x 64 CTA tiles, 4 MMA warps (2 x 2, 32 x 32 warp tiles, 128 registers) + 1 TMA
//    producer warp, 3 CTAs per SM, each with its own ring -- a stall in one CTA never blocks
//    another.
//  * All three products of Eq 3 with partitioned checksums use the same 64 x 64 tile:
//    C = A.B, Ccol = Acs.B (M/BS checksum rows), Crow = A.Bcs (N/BS checksum columns); the
//    checksum work costs its ideal 2/BS share when M/BS, N/BS are multiples of 64.  The corner
//    Acs.Bcs is never formed (reading R17).
//  * Persistent scheduling: full waves are data-parallel (grouped raster keeps a wave's A/B
//    panels L2-resident); the ragged remainder is split along K (stream-K) so every CTA gets
//    the same number of k-tiles.  Split tiles are reduced deterministically: the CTA holding
//    k-chunk 0 adds the partials of the following CTAs in ascending k order.
//  * A dedicated producer warp per CTA streams TMA (cp.async.bulk.tensor) copies through a
//    4-stage full/empty mbarrier ring (across tile boundaries), one box per lane.  A tiles use the 128B swizzle (box 16 k x 64 rows), B tiles are 8 boxes of 8
//    columns x 16 k with the 64B swizzle; with the k-permutation below every 64-bit fragment
//    LDS is bank-conflict free.
//  * Fault hooks (Alg 3): site 1 XORs the accumulator after the k-tile containing k_step (in
//    a split tile: the partial accumulator of the CTA that owns that k-tile); sites 0/2 act
//    on the stored value.
#include <cudaTypedefs.h>

#include <algorithm>
#include <atomic>

#include "common.cuh"

namespace aabft {

namespace {

#ifndef AABFT_F64_STAGES
#define AABFT_F64_STAGES 4
#endif
#ifndef AABFT_F64_PROD_FIRST
#define AABFT_F64_PROD_FIRST 0
#endif
#ifndef AABFT_F64_B3D
#define AABFT_F64_B3D 0
#endif
#ifndef AABFT_F64_GROUP_M
#define AABFT_F64_GROUP_M 16
#endif
#ifndef AABFT_F64_TN
#define AABFT_F64_TN 64
#endif
constexpr int TM = 64, TN = AABFT_F64_TN, BK = 16, STAGES = AABFT_F64_STAGES;  // CTA tile TM x TN
constexpr int TILE = TM;  // rows of a CTA tile (fused check: bs <= TILE)
// B tiles as 4 TMA boxes of 16 columns x 16 k with the 128B swizzle (B16) instead of 8 boxes of
// 8 columns with the 64B swizzle: half the copies per stage; needs its own k-permutation
#ifndef AABFT_F64_B16
#define AABFT_F64_B16 1
#endif
constexpr bool B16 = AABFT_F64_B16 != 0;
#ifndef AABFT_F64_L2PROMO
#define AABFT_F64_L2PROMO CU_TENSOR_MAP_L2_PROMOTION_L2_128B
#endif
#ifndef AABFT_F64_EARLY_RELEASE
#define AABFT_F64_EARLY_RELEASE 0
#endif
#ifndef AABFT_F64_KROT
#define AABFT_F64_KROT 0
#endif
#ifndef AABFT_F64_C_STREAM
#define AABFT_F64_C_STREAM 0
#endif
#ifndef AABFT_F64_NT
#define AABFT_F64_NT 4
#endif
constexpr int NT = AABFT_F64_NT;            // n8 fragments per warp (warp tile 32 x 8*NT)
constexpr int MT = 2;                       // m16 fragments per warp
constexpr int WTN = NT * 8;                 // warp tile columns
constexpr int WARPS_N = TN / WTN;           // warps across the tile's columns
constexpr int NCW = 2 * WARPS_N;            // MMA warps per CTA (2 x WARPS_N)
constexpr int THREADS = NCW * 32;           // MMA threads (named barrier 1)
constexpr int CTA_THREADS = THREADS + 32;   // + 1 TMA producer warp
#ifndef AABFT_F64_CTAS
#define AABFT_F64_CTAS (NCW == 4 ? 3 : 2)
#endif
constexpr int CTAS_PER_SM = AABFT_F64_CTAS;  // 15 / 18 warps per SM (128 / <= 102 registers)
// BS = 64 on a 64 x 64 tile of 2 x 2 warps: the block is the CTA tile, and the epilogue
// completes its column / row reference sums inside the CTA (shared memory, one barrier) --
// otherwise a block larger than a warp tile leaves per-warp "parts" in the workspace
#ifndef AABFT_F64_CTA_SUMS
#define AABFT_F64_CTA_SUMS 1
#endif
constexpr bool kCtaSums = AABFT_F64_CTA_SUMS && TM == 64 && TN == 64 && WTN == 32;
constexpr int COL_PARTS = kCtaSums ? 1 : 2;           // fused column sums of a BS = 64 block
constexpr int ROW_PARTS = kCtaSums ? 1 : 64 / WTN;    // fused row sums of a BS = 64 block
constexpr int A_BYTES = TILE * BK * 8;      // 8 KiB
constexpr int B_BYTES = BK * TN * 8;        // 8 KiB (TN 64) / 4 KiB (TN 32)
constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
constexpr int MAXF = 64;                    // faults per 64x64 tile kept in smem (one per 8x8 block)
constexpr int BOOK = 128;                   // barriers, counters, cursor
constexpr int SUMBUF = 4 * 64 * 8;           // BS = 64 epilogue exchange (kCtaSums)
// [ring][bookkeeping][BS = 64 sum exchange][fault list: FAULTS instantiation only -- the
// production kernel leaves ~23 KB per SM free for the overlapped encode's CTA]
constexpr int SMEM_PROD = STAGES * STAGE_BYTES + 1024 /*align*/ + BOOK + SUMBUF;
constexpr int SMEM_FAULTS = SMEM_PROD + MAXF * (int)sizeof(aabft_fault);
constexpr int smem_bytes(bool faults) { return faults ? SMEM_FAULTS : SMEM_PROD; }
constexpr int GROUP_M = AABFT_F64_GROUP_M;
constexpr int kMaxCtas = 1024;              // >= resident CTAs; sizes the split-K partial slots
constexpr int ACC = MT * NT * 4;            // accumulators per thread
constexpr int kTpMaxP = 4;                  // top-p selection in the GEMM for p <= 4

struct GemmArgs {
  int64_t M, N, K, Mcs, Ncs;
  double *C;
  int64_t ldc;
  double *Ccol;
  int64_t ld_ccol;
  double *Crow;
  int64_t ld_crow;
  int tm0, tn0, tm1, tn2;             // tile grids: data tm0 x tn0, Ccol tm1 x tn0, Crow tm0 x tn2
  int n0, n1, n2, ntiles;
  int nk;                             // k-tiles per tile
  int waves;                          // data-parallel waves
  int64_t sk_iters;                   // k-tiles in the stream-K remainder
  double *partials;                   // [kMaxCtas][ACC][THREADS]
  int *flags;                         // [kMaxCtas]
  const aabft_fault *faults;
  int nfaults;
  double *Rcol;                       // fused reference sums (NULL = unfused): (M/bs) x N
  double *Rrow;                       //                                         M x (N/bs)
  double *Rcol2;                      // BS = 64: partials of the wm = 1 warps (workspace)
  double *Rrow2;                      //          partials of the wn = 1 warps (workspace)
  int bs;
  // top-p selection fused into the operand stream (TP > 0; DESIGN.md 6.1 "top-p in the GEMM")
  double *topA_v;                     // (M + M/bs) x TP  final tables (aabft_encoded)
  int *topA_i;
  double *topB_v;                     // (N + N/bs) x TP
  int *topB_i;
  double *tp_v;                       // [kMaxCtas][128 lists][TP] stream-K partial lists
  int *tp_i;
  int *tp_flags;                      // [kMaxCtas]
  int b3d, bcs3d;                     // B / Bcs tiles as ONE 3-D TMA box (8 cols x 16 k x 8 groups)
  unsigned long long *check_acc;      // the following aabft_check's counter accumulator: zeroed
};

struct Tile {
  int type, m0, n0;
};

__device__ __forceinline__ Tile tile_of(const GemmArgs &a, int t) {
  Tile r;
  if (t < a.n0) {
    r.type = 0;
    const int group = GROUP_M * a.tn0;
    const int g = t / group;
    const int first_m = g * GROUP_M;
    const int gm = min(a.tm0 - first_m, GROUP_M);
    const int in = t % group;
    r.m0 = (first_m + in % gm) * TM;
    r.n0 = (in / gm) * TN;
  } else if (t < a.n0 + a.n1) {
    t -= a.n0;
    r.type = 1;
    r.m0 = (t / a.tn0) * TM;
    r.n0 = (t % a.tn0) * TN;
  } else {
    t -= a.n0 + a.n1;
    r.type = 2;
    r.m0 = (t / a.tn2) * TM;
    r.n0 = (t % a.tn2) * TN;
  }
  return r;
}

__device__ __forceinline__ int64_t sk_begin(const GemmArgs &a, int64_t c) {
  return a.sk_iters * c / gridDim.x;
}

// the CTA's j-th k-tile: (tile index, k-tile index)
__device__ __forceinline__ void iter_of(const GemmArgs &a, int j, int64_t sk0, int &tile, int &kt) {
  const int dp = a.waves * a.nk;
  if (j < dp) {
    tile = (int)blockIdx.x + (j / a.nk) * (int)gridDim.x;
    kt = j % a.nk;
  } else {
    const int64_t it = sk0 + (j - dp);
    tile = a.waves * (int)gridDim.x + (int)(it / a.nk);
    kt = (int)(it % a.nk);
  }
}

__device__ __forceinline__ void dmma(double (&c)[4], double a0, double a1, double b) {
  asm volatile(
      "mma.sync.aligned.m16n8k4.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5}, {%6}, "
      "{%0,%1,%2,%3};"
      : "+d"(c[0]), "+d"(c[1]), "+d"(c[2]), "+d"(c[3])
      : "d"(a0), "d"(a1), "d"(b));
}

// barrier among the 4 MMA warps only (the producer warp never joins)
__device__ __forceinline__ void mma_sync_bar() {
  asm volatile("bar.sync 1, %0;" ::"n"(THREADS) : "memory");
}

__device__ __forceinline__ double xor_bits(double v, uint64_t m) {
  return __longlong_as_double(__double_as_longlong(v) ^ (long long)m);
}

// FAULTS: the Alg 3 injection instantiation (launched only with a fault list); the production
// instantiation carries no fault bookkeeping in its k-loop.
// ------------------------------------------------------------------ top-p in the GEMM
// Step 1's top-p selection (Alg 1; the paper runs its global reduction "in
// parallel to the matrix multiplication kernel", P:L320 / P:L368) taken from the operand
// tiles the GEMM already streams through shared memory: the tiles of block-column 0 see every
// row of A (type 0) and of Acs (type 1) over the whole K, the tiles of block-row 0 every
// column of B (type 0) and of Bcs (type 2).  The TMA producer warp -- otherwise idle on the
// empty barriers -- scans a stage kScanLag jobs after issuing it (the stage is refilled only
// STAGES jobs later, by the same warp), lane l owning rows / columns l and l + 32.
// MEASURED SLOWER than selecting in aabft_encode (the ~130 scanning CTAs
// become stragglers, +0.35 ms on a 4.17 ms c2 GEMM against ~0.05 ms of top-p work in the
// encode), so it is opt-in (AABFT_FLAG_TOPP_IN_GEMM) and ProtectedGemm leaves it off.  Within a segment k ascends, so the branch-free tp_push (new
// element loses every tie) gives the sequential scan's list; stream-K partial lists are
// parked like the accumulators and merged by the tile's owner with the full comparator.  No
// extra HBM traffic; the encode stage keeps only the checksums.
constexpr int kScanLag = STAGES - 1;  // measured best of 1..3 (tools/variants_time.sh)

template <int P>
struct TopScan {
  int tile, kt0;
  bool sa, sb;
  Tile tl;
  unsigned long long ka[2][P], kb[2][P];  // |value| bit patterns (integer-ALU selection)
  double va[2][P], vb[2][P];              // values at the segment end (merge / store)
  int ia[2][P], ib[2][P];
};

__device__ __forceinline__ void sk_owner_contributors_end(const GemmArgs &a, int tile, int64_t &it_end) {
  it_end = (int64_t)(tile - a.waves * (int)gridDim.x + 1) * a.nk;
}

template <int P>
__device__ __forceinline__ void tp_store(double *v_out, int *i_out, const double (&v)[P],
                                         const int (&ix)[P]) {
#pragma unroll
  for (int r = 0; r < P; ++r) { v_out[r] = v[r]; i_out[r] = ix[r]; }
}

template <int P>
__device__ __forceinline__ void tp_merge_from(double (&v)[P], int (&ix)[P], const double *sv,
                                             const int *si) {
#pragma unroll
  for (int r = 0; r < P; ++r) tp_insert<P>(v, ix, __ldcg(sv + r), __ldcg(si + r));
}

template <int P>
__device__ void scan_flush(const GemmArgs &a, TopScan<P> &sc, int kt_last, int lane) {
  const bool first = sc.kt0 == 0, last = kt_last == a.nk - 1;
#pragma unroll
  for (int h = 0; h < 2; ++h)
#pragma unroll
    for (int r = 0; r < P; ++r) {  // empty slots keep the tp_init sentinel (-1.0, -1)
      sc.va[h][r] = sc.ia[h][r] < 0 ? -1.0 : __longlong_as_double((long long)(sc.ka[h][r] - 1));
      sc.vb[h][r] = sc.ib[h][r] < 0 ? -1.0 : __longlong_as_double((long long)(sc.kb[h][r] - 1));
    }
  if (!first) {  // stream-K contributor: park the partial lists, then signal the tile's owner
    double *pv = a.tp_v + (int64_t)blockIdx.x * 128 * P;
    int *pi = a.tp_i + (int64_t)blockIdx.x * 128 * P;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      if (sc.sa) tp_store<P>(pv + (lane + 32 * h) * P, pi + (lane + 32 * h) * P, sc.va[h], sc.ia[h]);
      if (sc.sb) tp_store<P>(pv + (64 + lane + 32 * h) * P, pi + (64 + lane + 32 * h) * P, sc.vb[h], sc.ib[h]);
    }
    __threadfence();
    __syncwarp();
    if (lane == 0) atomicExch(&a.tp_flags[blockIdx.x], 1);
    return;
  }
  if (!last) {  // owner of a split tile: merge the following CTAs' partial lists
    int64_t it_end;
    sk_owner_contributors_end(a, sc.tile, it_end);
    for (int64_t c = blockIdx.x + 1; c < gridDim.x && sk_begin(a, c) < it_end; ++c) {
      if (sk_begin(a, c + 1) == sk_begin(a, c)) continue;  // empty slice
      if (lane == 0) {
        while (atomicAdd(&a.tp_flags[c], 0) == 0) __nanosleep(64);
        atomicExch(&a.tp_flags[c], 0);  // re-arm for the next launch
        __threadfence();
      }
      __syncwarp();
      const double *pv = a.tp_v + c * 128 * P;
      const int *pi = a.tp_i + c * 128 * P;
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        if (sc.sa) tp_merge_from<P>(sc.va[h], sc.ia[h], pv + (lane + 32 * h) * P, pi + (lane + 32 * h) * P);
        if (sc.sb) tp_merge_from<P>(sc.vb[h], sc.ib[h], pv + (64 + lane + 32 * h) * P, pi + (64 + lane + 32 * h) * P);
      }
    }
  }
  // complete lists: data vectors first, then checksum vectors (aabft_encoded layout)
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    const int r = lane + 32 * h;
    if (sc.sa) {
      int64_t row = -1;
      if (sc.tl.type == 0 && sc.tl.m0 + r < a.M) row = sc.tl.m0 + r;
      if (sc.tl.type == 1 && sc.tl.m0 + r < a.Mcs) row = a.M + sc.tl.m0 + r;
      if (row >= 0) tp_store<P>(a.topA_v + row * P, a.topA_i + row * P, sc.va[h], sc.ia[h]);
    }
    if (sc.sb) {
      int64_t col = -1;
      if (sc.tl.type == 0 && sc.tl.n0 + r < a.N) col = sc.tl.n0 + r;
      if (sc.tl.type == 2 && sc.tl.n0 + r < a.Ncs) col = a.N + sc.tl.n0 + r;
      if (col >= 0) tp_store<P>(a.topB_v + col * P, a.topB_i + col * P, sc.vb[h], sc.ib[h]);
    }
  }
}

template <int P>
__device__ __forceinline__ void scan_job(const GemmArgs &a, const uint8_t *smem, uint64_t *full,
                                         int js, int njobs, int64_t sk0, TopScan<P> &sc,
                                         int lane) {
  int tile, kt;
  iter_of(a, js, sk0, tile, kt);
  if (tile != sc.tile) {  // a new segment of consecutive k-tiles of one tile
    sc.tile = tile;
    sc.kt0 = kt;
    sc.tl = tile_of(a, tile);
    sc.sa = (sc.tl.type == 0 || sc.tl.type == 1) && sc.tl.n0 == 0;
    sc.sb = (sc.tl.type == 0 || sc.tl.type == 2) && sc.tl.m0 == 0;
#pragma unroll
    for (int h = 0; h < 2; ++h)
#pragma unroll
      for (int r = 0; r < P; ++r) {  // key = |x| bits + 1, so the empty key 0 loses to |x| = 0
        sc.ka[h][r] = 0ull; sc.kb[h][r] = 0ull; sc.ia[h][r] = -1; sc.ib[h][r] = -1;
      }
  }
  if (sc.sa || sc.sb) {
    const int s = js % STAGES;
    mbar_wait(&full[s], (uint32_t)((js / STAGES) & 1));
    const uint8_t *st = smem + s * STAGE_BYTES;
    const int kbase = kt * BK;
    const int lim = a.K - kbase < BK ? (int)(a.K - kbase) : BK;  // TMA zero-fills k >= K
    if (sc.sa) {
      // A tile: row r, column k at r*128 + ((k/2 ^ r%8) * 16) + (k%2)*8 (128B swizzle)
#pragma unroll
      for (int k = 0; k < BK; ++k) {
        if (k < lim) {
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int r = lane + 32 * h;
            const double x = *reinterpret_cast<const double *>(
                st + r * 128 + ((((k >> 1) ^ (r & 7)) << 4) | ((k & 1) << 3)));
            tp_push_bits<P>(sc.ka[h], sc.ia[h], abs_bits(x) + 1, kbase + k);
          }
        }
      }
    }
    if (sc.sb) {
      // B tile: 8 boxes of 8 columns; column c, row k at box*1024 + k*64 +
      // (((c%8)/2 ^ (k/2)%4) * 16) + (c%2)*8 (64B swizzle), or the B16 layout
#pragma unroll
      for (int k = 0; k < BK; ++k) {
        if (k < lim) {
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int c = lane + 32 * h, cc = c & 7, c16 = c & 15;
            // B16: 4 boxes of 16 columns, row k at box*2048 + k*128, 128B swizzle
            const double x = *reinterpret_cast<const double *>(
                B16 ? st + A_BYTES + (c >> 4) * 2048 + k * 128 +
                          ((((c16 >> 1) ^ (k & 7)) << 4) | ((c16 & 1) << 3))
                    : st + A_BYTES + (c >> 3) * 1024 + k * 64 +
                          ((((cc >> 1) ^ ((k >> 1) & 3)) << 4) | ((cc & 1) << 3)));
            tp_push_bits<P>(sc.kb[h], sc.ib[h], abs_bits(x) + 1, kbase + k);
          }
        }
      }
    }
  }
  if (kt == a.nk - 1 || js == njobs - 1) {  // segment end
    if (sc.sa || sc.sb) scan_flush<P>(a, sc, kt, lane);
    sc.tile = -1;
  }
}

#ifndef AABFT_F64_EVICT_LAST
#define AABFT_F64_EVICT_LAST 0
#endif
// TMA load with an L2 evict-last hint (operand panels are re-read by many CTAs)
__device__ __forceinline__ void tma_load_2d_el(void *smem_dst, const CUtensorMap *tm, uint64_t *bar,
                                               int c0, int c1) {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1, {%3, %4}], [%2], %5;" ::"r"(smem_u32(smem_dst)),
      "l"(reinterpret_cast<uint64_t>(tm)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "l"(pol)
      : "memory");
}

// one stage of a job: expect the bytes, then the A box and the B tile (one 3-D box, or 2-D
// boxes of 8 / 16 columns), all from the calling thread
__device__ __forceinline__ void issue_stage(const GemmArgs &a, const CUtensorMap *tmA,
                                            const CUtensorMap *tmAcs, const CUtensorMap *tmB,
                                            const CUtensorMap *tmBcs, uint8_t *sa, uint64_t *bar,
                                            const Tile &tl, int k) {
  mbar_arrive_expect_tx(bar, STAGE_BYTES);
  const CUtensorMap *mb = tl.type == 2 ? tmBcs : tmB;
  if (!B16 && (tl.type == 2 ? a.bcs3d : a.b3d)) {
    // the 8 column groups of the 64-column tile in one copy: smem [group][k][8 cols], the same
    // bytes and 64B swizzle as 8 separate 2-D boxes
    tma_load_3d(sa + A_BYTES, mb, bar, 0, k, tl.n0 / 8);
  } else if (B16) {
#pragma unroll
    for (int b = 0; b < TN / 16; ++b) {
#if AABFT_F64_EVICT_LAST
      tma_load_2d_el(sa + A_BYTES + b * 2048, mb, bar, tl.n0 + b * 16, k);
#else
      tma_load_2d(sa + A_BYTES + b * 2048, mb, bar, tl.n0 + b * 16, k);
#endif
    }
  } else {
#pragma unroll
    for (int b = 0; b < TN / 8; ++b) tma_load_2d(sa + A_BYTES + b * 1024, mb, bar, tl.n0 + b * 8, k);
  }
#if AABFT_F64_EVICT_LAST
  tma_load_2d_el(sa, tl.type == 1 ? tmAcs : tmA, bar, k, tl.m0);
#else
  tma_load_2d(sa, tl.type == 1 ? tmAcs : tmA, bar, k, tl.m0);
#endif
}

#ifdef AABFT_OV_PROBE
// timing diagnosis: [0] first CTA start, [1] last producer end, [2] latest encode-wait return
__device__ unsigned long long g_gemm_probe[3] = {~0ull, 0ull, 0ull};
__device__ __forceinline__ unsigned long long gemm_gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#endif

template <bool FAULTS, int TP>
__global__ void __launch_bounds__(CTA_THREADS, CTAS_PER_SM)
    gemm_f64_kernel(const __grid_constant__ CUtensorMap tmA,
                    const __grid_constant__ CUtensorMap tmAcs,
                    const __grid_constant__ CUtensorMap tmB,
                    const __grid_constant__ CUtensorMap tmBcs, const GemmArgs args) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  // 1024-B aligned ring (swizzle atoms); offset applied to the __shared__ array itself so the
  // compiler keeps the shared address space (32-bit LDS, not generic 64-bit loads)
  const uint32_t pad = (1024u - (smem_u32(smem_raw) & 1023u)) & 1023u;
  uint8_t *smem = smem_raw + pad;
  uint64_t *full = reinterpret_cast<uint64_t *>(smem + STAGES * STAGE_BYTES);
  uint64_t *empty = full + STAGES;
  int *s_nf = reinterpret_cast<int *>(empty + STAGES);
  static_assert(16 * STAGES + 8 <= BOOK, "bookkeeping fits");
  double *s_csum = reinterpret_cast<double *>(smem + STAGES * STAGE_BYTES + BOOK);  // [2][64] column parts
  double *s_rsum = s_csum + 128;                                                   // [2][64] row parts
  aabft_fault *s_f = reinterpret_cast<aabft_fault *>(s_csum + 256);  // FAULTS only

  // warp roles: the producer is the CTA's last warp (AABFT_F64_PROD_FIRST: its first);
  // mtid / mwarp index the 4 MMA warps
  const int warp_hw = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int prod_warp = AABFT_F64_PROD_FIRST ? 0 : NCW;
  const int warp = AABFT_F64_PROD_FIRST ? (warp_hw == 0 ? NCW : warp_hw - 1) : warp_hw;
  const int mtid = warp * 32 + lane;  // MMA thread index 0..THREADS-1 (producer: THREADS..)
  const int g = lane >> 2, tig = lane & 3;
  const int wm = warp / WARPS_N, wn = warp % WARPS_N;

  // this CTA's k-tile sequence: its data-parallel tiles, then its stream-K slice
  const int64_t sk0 = sk_begin(args, blockIdx.x), sk1 = sk_begin(args, blockIdx.x + 1);
  // data-parallel tiles of this CTA (the last wave may be partial when there is no stream-K
  // tail: AABFT_FLAG_GEMM_HALF_GRID), then its stream-K slice
  const int my_dp = min(args.waves, ((int)args.ntiles - (int)blockIdx.x + (int)gridDim.x - 1) / (int)gridDim.x);
  const int njobs = my_dp * args.nk + (int)(sk1 - sk0);

#ifdef AABFT_OV_PROBE
  if (threadIdx.x == 0) atomicMin(&g_gemm_probe[0], gemm_gtime());
#endif
  if (threadIdx.x == 0 && blockIdx.x == 0 && args.check_acc) {
    // the check of this product accumulates its counters here (no memset between the kernels)
#pragma unroll
    for (int w = 0; w < 10; ++w) args.check_acc[w] = 0ull;
  }
  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], NCW);
    }
    fence_barrier_init();
  }
  __syncthreads();

  // ---------------- TMA producer warp: streams every job of this CTA through the ring,
  // refilling a stage as soon as the 4 MMA warps released it (empty mbarrier).  The box
  // copies are spread over the lanes (one cp.async.bulk.tensor per lane).
  if (warp_hw == prod_warp) {
    if (lane == 0) {
      tma_prefetch_desc(&tmA);
      tma_prefetch_desc(&tmB);
      tma_prefetch_desc(&tmAcs);
      tma_prefetch_desc(&tmBcs);
    }
    int tile = -1, kt = 0;
    Tile tl{0, 0, 0};
    bool enc_ready = false;  // griddepcontrol.wait done (AABFT_FLAG_OVERLAP_ENCODE)
#ifdef AABFT_OV_PROBE
    unsigned long long first_cs_wait_end = 0;
#endif
    constexpr int SP = TP > 0 ? TP : 1;
    TopScan<SP> sc;
    sc.tile = -1;
    for (int jn = 0; jn < njobs; ++jn) {
      if (tile < 0 || kt + 1 >= args.nk || jn == args.waves * args.nk) {
        iter_of(args, jn, sk0, tile, kt);
        tl = tile_of(args, tile);
      } else {
        ++kt;
      }
      const int s = jn % STAGES;
      if (jn >= STAGES) mbar_wait(&empty[s], (uint32_t)(((jn / STAGES) & 1) ^ 1));
      uint8_t *sa = smem + s * STAGE_BYTES;
      // AABFT_F64_KROT (experiment): the CTAs sharing an SM start their data-parallel tiles at
      // k offsets 0, nk/3, 2nk/3 so their k-tile boundaries do not coincide
      int kphys = kt;
      if (AABFT_F64_KROT && !FAULTS && TP == 0 && jn < args.waves * args.nk) {
        const int rot = (int)(((long long)blockIdx.x * 3) / gridDim.x) * (args.nk / 3);
        kphys = (kt + rot) % args.nk;
      }
      const int k = kphys * BK;
      if (lane == 0) {
        // checksum tiles read Acs / Bcs, which a programmatically-dependent launch may still
        // be producing: wait for the preceding grid (no-op without PDL).  Data tiles read only
        // A and B and never wait.
        if (tl.type != 0 && !enc_ready) {
          griddep_wait();
          enc_ready = true;
#ifdef AABFT_OV_PROBE
          first_cs_wait_end = gemm_gtime();
#endif
        }
        issue_stage(args, &tmA, &tmAcs, &tmB, &tmBcs, sa, &full[s], tl, k);
      }
      __syncwarp();
      if (TP > 0 && jn >= kScanLag) scan_job<SP>(args, smem, full, jn - kScanLag, njobs, sk0, sc, lane);
    }
    if (TP > 0)
      for (int js = max(0, njobs - kScanLag); js < njobs; ++js)
        scan_job<SP>(args, smem, full, js, njobs, sk0, sc, lane);
    // the grid never completes before the grid it depends on (stream order is kept for the
    // kernels after it, e.g. aabft_check reading the top-p tables)
    if (lane == 0 && !enc_ready) griddep_wait();
#ifdef AABFT_OV_PROBE
    if (lane == 0) {
      atomicMax(&g_gemm_probe[1], gemm_gtime());           // last producer done
      atomicMax(&g_gemm_probe[2], first_cs_wait_end);      // latest return from the encode wait
    }
#endif
    return;
  }

  // Fragment addressing.  The mma k index (= tig) of k4-step ks maps to the k-tile column
  //   k = pi(ks, tig) = (tig&1) | (ks&1)<<1 | ((tig>>1)^(ks>>1))<<2 | (tig>>1)<<3
  // (a bijection of [0,16); the same permutation for A and B leaves the product unchanged).
  // With the 128B-swizzled A tile and the 64B-swizzled B boxes every half-warp of a 64-bit
  // LDS touches 16 distinct 8-byte bank slots (conflict-free: 2 wavefronts).
  // (offsets recomputed per load: cheaper than holding 8 registers across the k-loop)
  // B16: k = pi16(ks, tig) from {0,3,12,15}, {1,2,13,14}, {4,7,8,11}, {5,6,9,10}: per k4-step
  // the four tig give distinct (k>>3, k&1) -- conflict-free 128B-swizzled A rows -- and
  // distinct (k>>1)&3 -- conflict-free 128B-swizzled 16-column B rows.
  auto kperm = [&](int ks) -> int {
    if (B16) {
      constexpr uint64_t tab = 0xA965B874ED21FC30ull;  // nibble 4*ks + tig
      return (int)((tab >> (4 * (4 * ks + tig))) & 15);
    }
    return (tig & 1) | ((ks & 1) << 1) | ((((tig >> 1) ^ (ks >> 1)) & 1) << 2) | ((tig >> 1) << 3);
  };
  auto offA = [&](int ks) -> uint32_t {
    const int k = kperm(ks);
    return (uint32_t)(((wm * 32 + g) * 16 + ((((k >> 1) ^ g) << 1) | (k & 1))) * 8);
  };
  auto offB = [&](int ks) -> uint32_t {
    const int k = kperm(ks);
    if (B16)  // nt-independent part; odd nt flips chunk bit 2 (see load)
      return (uint32_t)(A_BYTES + wn * (WTN / 16) * 2048 + k * 128 + ((((g >> 1) ^ (k & 7)) << 4) | ((g & 1) << 3)));
    return (uint32_t)(A_BYTES + wn * NT * 1024 + (k * 8 + ((((g >> 1) ^ ((k >> 1) & 3)) << 1) | (g & 1))) * 8);
  };

  double acc[MT][NT][4];
  int j = 0;
  while (j < njobs) {
    // ---------------- segment = consecutive k-tiles of one tile
    int tile, kt0;
    iter_of(args, j, sk0, tile, kt0);
    const Tile tl = tile_of(args, tile);
    const int seg_len = min(args.nk - kt0, njobs - j);
    const int kt_end = kt0 + seg_len;  // exclusive
    const int64_t rbase = (int64_t)tl.m0 + wm * 32, cbase = (int64_t)tl.n0 + wn * WTN;

    // faults that hit this tile (output coordinates of the tile's product)
    int nf = 0;
    if (FAULTS && args.nfaults > 0) {
      mma_sync_bar();
      if (mtid == 0) *s_nf = 0;
      mma_sync_bar();
      for (int f = mtid; f < args.nfaults; f += THREADS) {
        aabft_fault ft = args.faults[f];
        int64_t r = ft.row, c = ft.col;
        int ftype;
        if (r < args.M && c < args.N) ftype = 0;
        else if (r >= args.M && c < args.N) { ftype = 1; r -= args.M; }
        else if (c >= args.N && r < args.M) { ftype = 2; c -= args.N; }
        else ftype = -1;
        if (ftype == tl.type && r >= tl.m0 && r < tl.m0 + TM && c >= tl.n0 && c < tl.n0 + TN) {
          const int slot = atomicAdd(s_nf, 1);
          if (slot < MAXF) {
            ft.row = r;
            ft.col = c;
            s_f[slot] = ft;
          }
        }
      }
      mma_sync_bar();
      nf = min(*s_nf, MAXF);
    }

#pragma unroll
    for (int i = 0; i < MT; ++i)
#pragma unroll
      for (int jj = 0; jj < NT; ++jj)
#pragma unroll
        for (int q = 0; q < 4; ++q) acc[i][jj][q] = 0.0;

    // Fragments are double-buffered in registers across k4-steps AND across k-tiles: the
    // ks = 0 fragments of k-tile kt+1 are loaded (after its full barrier) while the ks = 3
    // DMMAs of k-tile kt issue, so no warp idles on LDS latency at a k-tile boundary.
    double a[2][MT][2], b[2][NT];
    auto load = [&](const uint8_t *st, int buf, int ks) {
#pragma unroll
      for (int mt = 0; mt < MT; ++mt) {
        a[buf][mt][0] = *reinterpret_cast<const double *>(st + offA(ks) + mt * 2048);
        a[buf][mt][1] = *reinterpret_cast<const double *>(st + offA(ks) + mt * 2048 + 1024);
      }
      if (B16) {
        const uint32_t ob = offB(ks);
#pragma unroll
        for (int nt = 0; nt < NT; ++nt)
          b[buf][nt] = *reinterpret_cast<const double *>(st + ((ob + (nt >> 1) * 2048) ^ ((nt & 1) << 6)));
      } else {
#pragma unroll
        for (int nt = 0; nt < NT; ++nt)
          b[buf][nt] = *reinterpret_cast<const double *>(st + offB(ks) + nt * 1024);
      }
    };
    {
      const int s0 = j % STAGES;
      mbar_wait(&full[s0], (uint32_t)((j / STAGES) & 1));
      load(smem + s0 * STAGE_BYTES, 0, 0);
    }
    for (int kt = kt0; kt < kt_end; ++kt, ++j) {
      const int s = j % STAGES;
      const uint8_t *st = smem + s * STAGE_BYTES;
#pragma unroll
      for (int ks = 0; ks < BK / 4; ++ks) {
        if (ks + 1 < BK / 4) {
          load(st, (ks + 1) & 1, ks + 1);
#if AABFT_F64_EARLY_RELEASE
          if (ks + 2 == BK / 4) {  // the stage's last fragments are loaded: release it now
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[s]);
          }
#endif
        } else if (kt + 1 < kt_end) {
          const int s1 = (j + 1) % STAGES;
          mbar_wait(&full[s1], (uint32_t)(((j + 1) / STAGES) & 1));
          load(smem + s1 * STAGE_BYTES, 0, 0);
        }
#pragma unroll
        for (int mt = 0; mt < MT; ++mt)
#pragma unroll
          for (int nt = 0; nt < NT; ++nt)
            dmma(acc[mt][nt], a[ks & 1][mt][0], a[ks & 1][mt][1], b[ks & 1][nt]);
      }
#if !AABFT_F64_EARLY_RELEASE
      // release the stage to the producer (its last fragments were consumed by the ks = 3 DMMAs)
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[s]);
#endif
#ifdef AABFT_F64_KSYNC
      if ((kt & (AABFT_F64_KSYNC - 1)) == 0) mma_sync_bar();  // experiment: MMA warps in lockstep
#endif
      if (FAULTS && nf > 0) {  // Alg 3 errorVecAdd1 at k-tile granularity
        for (int f = 0; f < nf; ++f) {
          const aabft_fault ft = s_f[f];
          if ((ft.site != 1 && ft.site != 3) || ft.k_step / BK != kt) continue;
#pragma unroll
          for (int mt = 0; mt < MT; ++mt)
#pragma unroll
            for (int nt = 0; nt < NT; ++nt)
#pragma unroll
              for (int q = 0; q < 4; ++q) {
                const int64_t r = rbase + mt * 16 + g + (q >> 1) * 8;
                const int64_t c = cbase + nt * 8 + tig * 2 + (q & 1);
                if (r == ft.row && c == ft.col)
                  acc[mt][nt][q] = ft.site == 1 ? xor_bits(acc[mt][nt][q], ft.xor_mask)
                                                : acc[mt][nt][q] + ft.add;
              }
        }
      }
    }

    // ---------------- segment epilogue
    const bool first = kt0 == 0, last = kt_end == args.nk;
    if (!first) {
      // contributor: park the partial accumulators, then signal the owner
      double *slot = args.partials + (int64_t)blockIdx.x * ACC * THREADS + mtid;
#pragma unroll
      for (int mt = 0; mt < MT; ++mt)
#pragma unroll
        for (int nt = 0; nt < NT; ++nt)
#pragma unroll
          for (int q = 0; q < 4; ++q) slot[((mt * NT + nt) * 4 + q) * THREADS] = acc[mt][nt][q];
      __threadfence();
      mma_sync_bar();
      if (mtid == 0) atomicExch(&args.flags[blockIdx.x], 1);
      continue;
    }
    if (!last) {
      // owner of a split tile: add the partials of the following CTAs in ascending k order
      const int64_t tile_it_end = (int64_t)(tile - args.waves * (int)gridDim.x + 1) * args.nk;
      for (int64_t c = blockIdx.x + 1; c < gridDim.x && sk_begin(args, c) < tile_it_end; ++c) {
        if (sk_begin(args, c + 1) == sk_begin(args, c)) continue;  // empty slice: no partial
        if (mtid == 0) {
          while (atomicAdd(&args.flags[c], 0) == 0) __nanosleep(64);
          atomicExch(&args.flags[c], 0);  // re-arm for the next launch
          __threadfence();
        }
        mma_sync_bar();
        const double *slot = args.partials + c * ACC * THREADS + mtid;
#pragma unroll
        for (int mt = 0; mt < MT; ++mt)
#pragma unroll
          for (int nt = 0; nt < NT; ++nt)
#pragma unroll
            for (int q = 0; q < 4; ++q)
              acc[mt][nt][q] += __ldcg(slot + ((mt * NT + nt) * 4 + q) * THREADS);
        mma_sync_bar();
      }
    }
    if (FAULTS && nf > 0) {
      for (int f = 0; f < nf; ++f) {
        const aabft_fault ft = s_f[f];
        if (ft.site != 0 && ft.site != 2) continue;
#pragma unroll
        for (int mt = 0; mt < MT; ++mt)
#pragma unroll
          for (int nt = 0; nt < NT; ++nt)
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const int64_t r = rbase + mt * 16 + g + (q >> 1) * 8;
              const int64_t c = cbase + nt * 8 + tig * 2 + (q & 1);
              if (r == ft.row && c == ft.col)
                acc[mt][nt][q] = ft.site == 0 ? xor_bits(acc[mt][nt][q], ft.xor_mask)
                                              : acc[mt][nt][q] + ft.add;
            }
      }
    }
    if (args.Rcol != nullptr && tl.type == 0) {
      // ---- fused reference sums (Eq 4) of the BS x BS blocks touching this 64 x 64 C tile,
      // taken from the registers about to be stored (after any injected fault), in a fixed
      // order: 8-row / 8-column shuffle trees, then pairwise over fragments.  A block larger
      // than the warp tile (rows > 32 or columns > WTN) is left as per-warp partials ("parts",
      // part 0 in Rcol/Rrow, the others in the workspace) that aabft_check adds in part order.
      const int bs = args.bs;
      const int64_t nJ = args.N / bs;
      const bool cta64 = kCtaSums && bs == 64;  // block == CTA tile: complete the sums here
      // column sums: per (nt, e) column, 8-row trees over g, then (h, mt) pairwise
#pragma unroll
      for (int nt = 0; nt < NT; ++nt)
#pragma unroll
        for (int e = 0; e < 2; ++e) {
          double c8[MT][2];
#pragma unroll
          for (int mt = 0; mt < MT; ++mt)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              double v = acc[mt][nt][h * 2 + e];
              v += __shfl_xor_sync(0xffffffffu, v, 4);
              v += __shfl_xor_sync(0xffffffffu, v, 8);
              v += __shfl_xor_sync(0xffffffffu, v, 16);
              c8[mt][h] = v;  // rows mt*16 + h*8 + (0..7)
            }
          const double c16a = c8[0][0] + c8[0][1], c16b = c8[1][0] + c8[1][1];
          const double c32 = c16a + c16b;
          const int64_t col = cbase + nt * 8 + tig * 2 + e;
          if (g == 0 && col < args.N) {
            if (bs == 8) {
#pragma unroll
              for (int mt = 0; mt < MT; ++mt)
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                  const int64_t I = (rbase + mt * 16 + h * 8) / 8;
                  if (I * 8 < args.M) args.Rcol[I * args.N + col] = c8[mt][h];
                }
            } else if (bs == 16) {
              const int64_t I0 = rbase / 16;
              if (I0 * 16 < args.M) args.Rcol[I0 * args.N + col] = c16a;
              if ((I0 + 1) * 16 < args.M) args.Rcol[(I0 + 1) * args.N + col] = c16b;
            } else if (cta64) {  // each 32-row half of the column into the exchange buffer
              s_csum[wm * 64 + wn * 32 + nt * 8 + tig * 2 + e] = c32;
            } else {  // 32 or 64: one value per warp; part = which 32-row half of the block
              const int64_t I = rbase / bs;
              const int part = (int)((rbase % bs) / 32);
              double *dst = part == 0 ? args.Rcol : args.Rcol2;
              if (rbase < args.M) dst[I * args.N + col] = c32;
            }
          }
        }
      // row sums: per (mt, h) row, pairwise over e, 4-lane tree over tig, then over nt
#pragma unroll
      for (int mt = 0; mt < MT; ++mt)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          double r8[NT];
#pragma unroll
          for (int nt = 0; nt < NT; ++nt) {
            double v = acc[mt][nt][h * 2] + acc[mt][nt][h * 2 + 1];
            v += __shfl_xor_sync(0xffffffffu, v, 1);
            v += __shfl_xor_sync(0xffffffffu, v, 2);
            r8[nt] = v;  // columns nt*8 + (0..7)
          }
          // pairwise tree over the warp's NT column groups: r16[q] covers 16 columns
          double r16[NT / 2 > 0 ? NT / 2 : 1];
#pragma unroll
          for (int q = 0; q < NT / 2; ++q) r16[q] = r8[2 * q] + r8[2 * q + 1];
          double rw = NT == 4 ? r16[0] + r16[1] : r16[0];  // the warp's WTN columns
          const int64_t row = rbase + mt * 16 + h * 8 + g;
          if (tig == 0 && row < args.M) {
            if (bs == 8) {
#pragma unroll
              for (int nt = 0; nt < NT; ++nt) {
                const int64_t J = (cbase + nt * 8) / 8;
                if (J < nJ) args.Rrow[row * nJ + J] = r8[nt];
              }
            } else if (bs == 16) {
#pragma unroll
              for (int q = 0; q < NT / 2; ++q) {
                const int64_t J = (cbase + q * 16) / 16;
                if (J < nJ) args.Rrow[row * nJ + J] = r16[q];
              }
            } else if (cta64) {  // each 32-column half of the row into the exchange buffer
              s_rsum[wn * 64 + wm * 32 + mt * 16 + h * 8 + g] = rw;
            } else if (bs < WTN) {  // bs = 32 inside a 32-column warp tile (NT == 4)
              const int64_t J = cbase / 32;
              if (J < nJ) args.Rrow[row * nJ + J] = rw;
            } else {  // block spans bs / WTN warp columns: part = which one
              const int64_t J = cbase / bs;
              const int part = (int)((cbase % bs) / WTN);
              double *dst = part == 0 ? args.Rrow : args.Rrow2 + (int64_t)(part - 1) * args.M * nJ;
              if (J < nJ) dst[row * nJ + J] = rw;
            }
          }
        }
      if (cta64) {
        // complete the block's sums in part order (rows / columns 0..31 first, then 32..63)
        mma_sync_bar();
        const int64_t I = tl.m0 / 64, J = tl.n0 / 64;
        const int t = mtid;  // 128 MMA threads: column t / 64 ... one value each
        if (t < 64) args.Rcol[I * args.N + tl.n0 + t] = s_csum[t] + s_csum[64 + t];
        else args.Rrow[(tl.m0 + (t - 64)) * nJ + J] = s_rsum[t - 64] + s_rsum[t];
        mma_sync_bar();  // the exchange buffers are free for the next tile
      }
    }
    double *out;
    int64_t ld, rows_valid, cols_valid;
    if (tl.type == 0) { out = args.C; ld = args.ldc; rows_valid = args.M; cols_valid = args.N; }
    else if (tl.type == 1) { out = args.Ccol; ld = args.ld_ccol; rows_valid = args.Mcs; cols_valid = args.N; }
    else { out = args.Crow; ld = args.ld_crow; rows_valid = args.M; cols_valid = args.Ncs; }
    const bool vec_ok = (ld % 2 == 0) && ((reinterpret_cast<uintptr_t>(out) & 15) == 0);
#pragma unroll
    for (int mt = 0; mt < MT; ++mt)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int64_t r = rbase + mt * 16 + g + h * 8;
        if (r >= rows_valid) continue;
#pragma unroll
        for (int nt = 0; nt < NT; ++nt) {
          const int64_t c = cbase + nt * 8 + tig * 2;
          double *p = out + r * ld + c;
          const double v0 = acc[mt][nt][h * 2], v1 = acc[mt][nt][h * 2 + 1];
          if (c + 1 < cols_valid && vec_ok) {
#if AABFT_F64_C_STREAM
            __stcs(reinterpret_cast<double2 *>(p), make_double2(v0, v1));  // evict-first: keep L2 for operands
#else
            *reinterpret_cast<double2 *>(p) = make_double2(v0, v1);
#endif
          } else {
            if (c < cols_valid) p[0] = v0;
            if (c + 1 < cols_valid) p[1] = v1;
          }
        }
      }
  }
}

const void *kernel_for(bool faults, int tp) {
  static const void *tab[2][kTpMaxP + 1] = {
      {(const void *)gemm_f64_kernel<false, 0>, (const void *)gemm_f64_kernel<false, 1>,
       (const void *)gemm_f64_kernel<false, 2>, (const void *)gemm_f64_kernel<false, 3>,
       (const void *)gemm_f64_kernel<false, 4>},
      {(const void *)gemm_f64_kernel<true, 0>, (const void *)gemm_f64_kernel<true, 1>,
       (const void *)gemm_f64_kernel<true, 2>, (const void *)gemm_f64_kernel<true, 3>,
       (const void *)gemm_f64_kernel<true, 4>}};
  return tab[faults ? 1 : 0][tp];
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

// B as a 3-D tensor {8 columns, K rows, N/8 column groups} with strides {ldb, 8} elements: one
// box {8, 16, 8} is a 64-column x 16-k tile laid out [group][k][col] (64B swizzle per 64-byte
// row), i.e. exactly the 8 two-dimensional boxes of 8 columns.  Needs N % 8 == 0 (no group
// straddles the row end).  Returns false (caller falls back to 2-D boxes) if not encodable.
bool make_map_b3d(CUtensorMap *m, const void *base, uint64_t N, uint64_t K, uint64_t ld_elems) {
  auto enc = get_encoder();
  if (!enc || N % 8 != 0) return false;
  cuuint64_t dims[3] = {8, K, N / 8};
  cuuint64_t strides[2] = {ld_elems * 8, 64};
  cuuint32_t box[3] = {8, BK, TN / 8};
  cuuint32_t es[3] = {1, 1, 1};
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, const_cast<void *>(base), dims, strides, box,
             es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B, AABFT_F64_L2PROMO,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
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
                   box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw, AABFT_F64_L2PROMO,
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

#ifdef AABFT_OV_PROBE
extern "C" int aabft_debug_gemm_probe(unsigned long long *out3) {
  cudaMemcpyFromSymbol(out3, g_gemm_probe, 24);
  const unsigned long long init[3] = {~0ull, 0ull, 0ull};
  cudaMemcpyToSymbol(g_gemm_probe, init, 24);
  return 0;
}
#endif

bool make_tma_2d_f64(CUtensorMap *m, const void *base, uint64_t inner, uint64_t outer,
                     uint64_t ld_elems, uint32_t box_inner, uint32_t box_outer,
                     CUtensorMapSwizzle sw) {
  return make_map(m, base, inner, outer, ld_elems, box_inner, box_outer, sw);
}

static size_t r256z(size_t b) { return (b + 255) / 256 * 256; }
// [split-K accumulator partials][flags][top-p flags][top-p partial values][indices][R planes]
static size_t flags_off() { return r256z((size_t)kMaxCtas * ACC * THREADS * sizeof(double)); }
static size_t tpv_off() { return flags_off() + r256z(2 * (size_t)kMaxCtas * sizeof(int)); }
static size_t tpi_off() { return tpv_off() + r256z((size_t)kMaxCtas * 128 * kTpMaxP * sizeof(double)); }
static size_t red_off() { return tpi_off() + r256z((size_t)kMaxCtas * 128 * kTpMaxP * sizeof(int)); }
bool gemm_f64_topp_ok(const aabft_config *cfg) {
  return TN == 64 && cfg->dtype == AABFT_F64 && cfg->p <= kTpMaxP;  // producer-warp scan, 64-col tiles
}
size_t gemm_f64_ws_bytes(const aabft_config *cfg) {
  // the fused reference-sum planes exist only where the fused check can run (bs <= 64)
  if (cfg->bs > TILE) return red_off() + 256;
  return red_off() + r256z((size_t)(cfg->M / cfg->bs) * cfg->N * 8 * (COL_PARTS - 1)) +
         r256z((size_t)cfg->M * (cfg->N / cfg->bs) * 8 * (ROW_PARTS - 1)) + 256;
}
// the unprotected GEMM: split-K partial slots and flags only
size_t gemm_f64_plain_ws_bytes() { return tpv_off() + 256; }
int gemm_f64_fused_parts(int bs, int *row_parts) {
  if (kCtaSums) {  // every block's sums are complete after the epilogue
    *row_parts = 1;
    return 1;
  }
  *row_parts = bs > WTN ? bs / WTN : 1;
  return bs > 32 ? bs / 32 : 1;
}
void gemm_f64_red_ptrs(const aabft_config *cfg, void *ws, double **rcol2, double **rrow2) {
  char *w = static_cast<char *>(ws) + red_off();
  *rcol2 = reinterpret_cast<double *>(w);
  *rrow2 = reinterpret_cast<double *>(w + r256z((size_t)(cfg->M / cfg->bs) * cfg->N * 8 * (COL_PARTS - 1)));
}

aabft_status launch_gemm_f64(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                             int64_t ldb, const aabft_encoded *enc, const aabft_product *out,
                             const aabft_fault *faults, int32_t nfaults, bool plain, void *ws,
                             unsigned long long *check_acc, cudaStream_t st) {
  // per-device one-time setup (function attributes belong to the device's context); a racing
  // first call computes the same value twice, which is benign
  static std::atomic<int> max_ctas_dev[64];
  int dev = 0;
  cudaGetDevice(&dev);
  int max_ctas = max_ctas_dev[dev & 63].load(std::memory_order_relaxed);
  if (!max_ctas) {
    int sms = 0, per_sm = 0;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess)
      return check_launch("gemm_f64 SM count");
    per_sm = 1 << 30;  // every instantiation must keep every CTA resident
    for (int f = 0; f < 2; ++f)
      for (int tp = 0; tp <= kTpMaxP; ++tp) {
        const void *fn = kernel_for(f != 0, tp);
        int n = 0;
        if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes(f != 0)) !=
                cudaSuccess ||
            cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout,
                                 cudaSharedmemCarveoutMaxShared) != cudaSuccess)
          return check_launch("gemm_f64 smem attribute");
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, fn, CTA_THREADS, smem_bytes(f != 0)) !=
                cudaSuccess || n < 1)
          return check_launch("gemm_f64 occupancy");
        per_sm = std::min(per_sm, n);
      }
    // every CTA must be resident (split-tile owners wait on later CTAs)
    max_ctas = std::min(sms * per_sm, kMaxCtas);
    max_ctas_dev[dev & 63].store(max_ctas, std::memory_order_relaxed);
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
  const int64_t tm0 = (M + TM - 1) / TM, tn0 = (N + TN - 1) / TN;
  const int64_t tm1 = (a.Mcs + TM - 1) / TM, tn2 = (a.Ncs + TN - 1) / TN;
  const int64_t ntiles = tm0 * tn0 + tm1 * tn0 + tm0 * tn2;
  const int64_t nk = (K + BK - 1) / BK;
  if (ntiles * nk >= ((int64_t)1 << 31) || M >= ((int64_t)1 << 31) || N >= ((int64_t)1 << 31)) {
    set_error("gemm_f64: problem too large for 32-bit tile/iteration indices");
    return AABFT_EINVAL;
  }
  a.tm0 = (int)tm0; a.tn0 = (int)tn0; a.tm1 = (int)tm1; a.tn2 = (int)tn2;
  a.n0 = (int)(tm0 * tn0); a.n1 = (int)(tm1 * tn0); a.n2 = (int)(tm0 * tn2);
  a.ntiles = (int)ntiles;
  a.nk = (int)nk;
  const int64_t total = ntiles * nk;
  // AABFT_FLAG_GEMM_HALF_GRID: half the persistent grid, so two launches can share the GPU
  const int cap = (cfg->flags & AABFT_FLAG_GEMM_HALF_GRID) ? std::max(1, max_ctas / 2) : max_ctas;
  // small problems: at least kMinIters k-tiles per CTA, so a split tile has few contributors
  // (the owner adds their partials one after another: at 128^3 every tile was split 8 ways)
  constexpr int64_t kMinIters = 4;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(cap, std::max<int64_t>(ntiles, total / kMinIters)));
  // full data-parallel waves, keeping at least ~1/2 wave of tiles for the stream-K tail so
  // every CTA's k-slice stays long enough to amortise its fixup
  int waves = (int)(ntiles / grid);
  if (waves > 0 && ntiles % grid != 0 && (ntiles % grid) * 2 < grid) waves -= 1;
  a.waves = waves;
  a.sk_iters = std::max<int64_t>(0, ntiles - (int64_t)waves * grid) * nk;
  a.partials = static_cast<double *>(ws);
  a.flags = reinterpret_cast<int *>(static_cast<char *>(ws) + flags_off());
  a.tp_flags = a.flags + kMaxCtas;
  a.tp_v = reinterpret_cast<double *>(static_cast<char *>(ws) + tpv_off());
  a.tp_i = reinterpret_cast<int *>(static_cast<char *>(ws) + tpi_off());
  // top-p in the GEMM (aabft_config flag; FP64, p <= 4): the tables of `enc`
  const int tp = (!plain && (cfg->flags & AABFT_FLAG_TOPP_IN_GEMM) && gemm_f64_topp_ok(cfg) &&
                  enc->topA_val && enc->topB_val) ? cfg->p : 0;
  a.topA_v = tp ? enc->topA_val : nullptr;
  a.topA_i = tp ? enc->topA_idx : nullptr;
  a.topB_v = tp ? enc->topB_val : nullptr;
  a.topB_i = tp ? enc->topB_idx : nullptr;
  a.faults = faults;
  a.nfaults = faults ? nfaults : 0;
  a.check_acc = plain ? nullptr : check_acc;
  a.bs = (int)bs;
  const bool fused = !plain && out->Rcol && out->Rrow && bs <= TILE;
  a.Rcol = fused ? out->Rcol : nullptr;
  a.Rrow = fused ? out->Rrow : nullptr;
  gemm_f64_red_ptrs(cfg, ws, &a.Rcol2, &a.Rrow2);

  CUtensorMap tA, tAcs, tB, tBcs;
  if (!make_map(&tA, A, K, M, lda, BK, TILE, CU_TENSOR_MAP_SWIZZLE_128B)) return AABFT_EINVAL;
  a.b3d = a.bcs3d = 0;
  if (AABFT_F64_B3D && !B16 && make_map_b3d(&tB, B, N, K, ldb)) {
    a.b3d = 1;
  } else if (!make_map(&tB, B, N, K, ldb, B16 ? 16 : 8, BK,
                       B16 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B)) {
    return AABFT_EINVAL;
  }
  if (plain) {
    tAcs = tA;
    tBcs = tB;
    a.bcs3d = a.b3d;
  } else {
    if (!make_map(&tAcs, enc->Acs, K, a.Mcs, enc->ld_acs, BK, TILE, CU_TENSOR_MAP_SWIZZLE_128B))
      return AABFT_EINVAL;
    if (AABFT_F64_B3D && !B16 &&
        make_map_b3d(&tBcs, enc->Bcs, (uint64_t)a.Ncs, K, enc->ld_bcs)) {
      a.bcs3d = 1;
    } else if (!make_map(&tBcs, enc->Bcs, a.Ncs, K, enc->ld_bcs, B16 ? 16 : 8, BK,
                         B16 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B)) {
      return AABFT_EINVAL;
    }
  }
  if (total > 0) {
    // AABFT_FLAG_OVERLAP_ENCODE (protected product): a programmatic dependent launch of the
    // preceding aabft_encode; the flag words are zero on entry by contract (workspace zeroed
    // once, every launch re-arms the words it used), so no reset sits between the two grids
    const bool overlap = !plain && (cfg->flags & AABFT_FLAG_OVERLAP_ENCODE);
    if (!overlap && a.sk_iters > 0 &&
        cudaMemsetAsync(a.flags, 0, 2 * kMaxCtas * sizeof(int), st) != cudaSuccess)
      return check_launch("gemm_f64 flag reset");
    // split-tile owners spin on flags set by later CTAs: with a stream-K tail the launch is
    // COOPERATIVE, so a grid that cannot be co-resident (other kernels, MPS, green contexts)
    // waits for room or fails instead of hanging.  Overlapped with the encode it
    // is a plain launch: the encode grid it may share the GPU with never waits on the GEMM,
    // so every GEMM CTA becomes resident at the latest when the encode's CTAs exit.
    cudaLaunchConfig_t lc = {};
    lc.gridDim = dim3((unsigned)grid);
    lc.blockDim = dim3(CTA_THREADS);
    lc.dynamicSmemBytes = smem_bytes(a.nfaults > 0);
    lc.stream = st;
    cudaLaunchAttribute attr[1];
    if (overlap) {
      attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
      attr[0].val.programmaticStreamSerializationAllowed = 1;
    } else {
      attr[0].id = cudaLaunchAttributeCooperative;
      attr[0].val.cooperative = a.sk_iters > 0 ? 1 : 0;
    }
    lc.attrs = attr;
    lc.numAttrs = 1;
    void *params[] = {&tA, &tAcs, &tB, &tBcs, &a};
    cudaError_t e = cudaLaunchKernelExC(&lc, kernel_for(a.nfaults > 0, tp), params);
    if (e != cudaSuccess) return check_launch("aabft_gemm(f64) launch");
    next_launch();
  }
  return check_launch("aabft_gemm(f64)");
}

}  // namespace aabft
