// common.cuh -- shared device/host helpers of the sm_100a A-ABFT library (CUDA path only;
// nothing here is shared with oracle/).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/aabft.h"

namespace aabft {

// ----------------------------------------------------------------------------- host side
void set_error(const char *fmt, ...);
int64_t next_launch(int64_t n = 1);  // bumps the library launch counter
aabft_status check_launch(const char *what);
aabft_status validate(const aabft_config *cfg);
int eff_t(const aabft_config *cfg);
size_t elem_size(const aabft_config *cfg);

// the GEMM epilogue forms the reference sums of the check (fused check): FP64 with bs <= 64
// (64 x 64 tiles), FP32 with bs <= 128 (128 x 128 tiles)
inline bool fused_check_ok(const aabft_config *cfg) {
  return (cfg->dtype == AABFT_F64 && cfg->bs <= 64) || (cfg->dtype == AABFT_F32 && cfg->bs <= 128);
}

// sigma coefficient sqrt(F(K)) (Eq 28 P:L219 / P:L287) evaluated in double on the host
// (compiled without FMA contraction); passed to kernels as a parameter.
double sigma_coeff(int64_t K, int fma_model);

struct BoundParams {
  double s;          // sqrt(F(K))
  double two_mt;     // 2^-t
  double two_m2t;    // 2^-2t
  double omega;
  double ev_coeff;   // K/3 (only used when fma_model == 0)
  int fma_model;
  int p;
};
BoundParams make_bound_params(const aabft_config *cfg);

// Encode-stage chunking (shared by workspace sizing and the launcher).
constexpr int kEncAChunk = 128;   // columns of A per encode CTA (one thread per column)
#ifndef AABFT_ENC_BCHUNK
#define AABFT_ENC_BCHUNK 256
#endif
constexpr int kEncBChunk = AABFT_ENC_BCHUNK;  // rows of B per encode CTA
inline int64_t enc_a_chunks(int64_t K) { return (K + kEncAChunk - 1) / kEncAChunk; }
inline int64_t enc_b_chunks(int64_t K) { return (K + kEncBChunk - 1) / kEncBChunk; }

// launchers (defined in the .cu files)
aabft_status launch_encode(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                           int64_t ldb, const aabft_encoded *out, void *ws, cudaStream_t st);
aabft_status launch_bound(const aabft_config *cfg, const aabft_encoded *enc, double *eps_col,
                          double *sig_col, double *eps_row, double *sig_row, cudaStream_t st);
// check_acc (protected product): the check accumulator the kernel zeroes (see launch_check)
aabft_status launch_gemm_f64(const aabft_config *cfg, const void *A, int64_t lda,
                             const void *B, int64_t ldb, const aabft_encoded *enc,
                             const aabft_product *out, const aabft_fault *faults,
                             int32_t nfaults, bool plain, void *ws,
                             unsigned long long *check_acc, cudaStream_t st);
size_t encode_ws_bytes(const aabft_config *cfg);
// AABFT_FLAG_OVERLAP_ENCODE honoured by aabft_encode (FP64, 16 <= bs <= 64, p <= 4)
bool encode_overlap_ok(const aabft_config *cfg);
// 2-D FP64 TMA descriptor {inner, outer} with row pitch ld_elems (gemm_f64.cu)
bool make_tma_2d_f64(CUtensorMap *m, const void *base, uint64_t inner, uint64_t outer,
                     uint64_t ld_elems, uint32_t box_inner, uint32_t box_outer,
                     CUtensorMapSwizzle sw);
aabft_status launch_counts_sum(const aabft_counts *parts, int n, aabft_counts *out, cudaStream_t st);
size_t gemm_f64_ws_bytes(const aabft_config *cfg);
size_t gemm_f64_plain_ws_bytes();
bool gemm_f64_topp_ok(const aabft_config *cfg);  // AABFT_FLAG_TOPP_IN_GEMM honoured
void gemm_f64_red_ptrs(const aabft_config *cfg, void *gemm_ws, double **rcol2, double **rrow2);
int gemm_f64_fused_parts(int bs, int *row_parts);  // returns column parts
aabft_status launch_gemm_f32(const aabft_config *cfg, const void *A, int64_t lda,
                             const void *B, int64_t ldb, const aabft_encoded *enc,
                             const aabft_product *out, const aabft_fault *faults,
                             int32_t nfaults, bool plain, unsigned long long *check_acc,
                             cudaStream_t st);
aabft_status launch_bound_elements(const aabft_config *cfg, const aabft_encoded *enc,
                                   const int64_t *rows, const int64_t *cols, int64_t n,
                                   double *sig, double *eps, cudaStream_t st);
aabft_status launch_checksum_errors(const aabft_config *cfg, const void *A, int64_t lda,
                                    const void *B, int64_t ldb, const aabft_encoded *enc,
                                    const aabft_product *prod, double *err_col, double *err_row,
                                    cudaStream_t st);
// acc: the workspace's check accumulator (10 words, zeroed by aabft_gemm) or NULL (memset cnt)
aabft_status launch_check(const aabft_config *cfg, const aabft_encoded *enc,
                          const aabft_product *prod, aabft_block_report *rep,
                          aabft_counts *cnt, void *gemm_ws, unsigned long long *acc,
                          cudaStream_t st);
aabft_status launch_correct(const aabft_config *cfg, const aabft_encoded *enc,
                            const aabft_product *prod, aabft_block_report *rep,
                            aabft_counts *cnt, cudaStream_t st);
// NEXT-3 comparators (check.cu, sea.cu)
aabft_status launch_check_ext(const aabft_config *cfg, const aabft_product *prod,
                              const double *eps_col, const double *eps_row, double eps_fixed,
                              aabft_block_report *rep, aabft_counts *cnt, void *gemm_ws,
                              unsigned long long *acc, cudaStream_t st);
aabft_status launch_correct_ext(const aabft_config *cfg, const aabft_product *prod,
                                const double *eps_row, double eps_fixed, aabft_block_report *rep,
                                aabft_counts *cnt, cudaStream_t st);
size_t sea_ws_bytes(const aabft_config *cfg);
aabft_status launch_sea_bound(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                              int64_t ldb, const aabft_encoded *enc, double *eps_col,
                              double *eps_row, double *eps_corner, void *ws, cudaStream_t st);

// ----------------------------------------------------------------------------- device side
// Top-p list order: value descending, then index ascending (reading R13).  Because indices
// within one vector are distinct this is a strict total order, so any merge tree gives the
// same p survivors as a sequential scan.
__device__ __forceinline__ bool tp_better(double v1, int i1, double v2, int i2) {
  return v1 > v2 || (v1 == v2 && (unsigned)i1 < (unsigned)i2);
}

// Simple, obviously-ordered insertion used everywhere (P <= 8).
template <int P>
__device__ __forceinline__ void tp_insert(double (&v)[P], int (&ix)[P], double val, int idx) {
  if (!tp_better(val, idx, v[P - 1], ix[P - 1])) return;
  int pos = P - 1;
#pragma unroll
  for (int r = P - 2; r >= 0; --r)
    if (tp_better(val, idx, v[r], ix[r])) pos = r;
#pragma unroll
  for (int r = P - 1; r > 0; --r)
    if (r > pos) { v[r] = v[r - 1]; ix[r] = ix[r - 1]; }
#pragma unroll
  for (int r = 0; r < P; ++r)
    if (r == pos) { v[r] = val; ix[r] = idx; }
}

// Insertion of an element that loses every tie (its index is larger than all indices in the
// list: a lane scanning its own elements in ascending index order).  For small P it is
// branch-free -- g[r] = (a > v[r]) is monotone in r, and slot r takes v[r-1] if g[r-1], else a
// if g[r], else keeps v[r] -- so a warp whose lanes insert at different elements never
// diverges; larger P falls back to the early-exit insertion.
template <int P>
__device__ __forceinline__ void tp_push(double (&v)[P], int (&ix)[P], double a, int idx) {
  if (P <= 4) {
    bool g[P];
#pragma unroll
    for (int r = 0; r < P; ++r) g[r] = a > v[r];
#pragma unroll
    for (int r = P - 1; r >= 1; --r) {
      const double vr = g[r - 1] ? v[r - 1] : (g[r] ? a : v[r]);
      const int ir = g[r - 1] ? ix[r - 1] : (g[r] ? idx : ix[r]);
      v[r] = vr;
      ix[r] = ir;
    }
    v[0] = g[0] ? a : v[0];
    ix[0] = g[0] ? idx : ix[0];
  } else {
    if (a > v[P - 1]) tp_insert<P>(v, ix, a, idx);
  }
}

// tp_push on the bit patterns of |x|: for non-negative doubles the unsigned 64-bit order of
// the bits is the value order, so the selection runs on the integer ALU (ISETP/SEL) instead
// of the FP64 pipe -- which the FP64 GEMM keeps busy with DMMA.  Same list as tp_push.
template <int P>
__device__ __forceinline__ void tp_push_bits(unsigned long long (&v)[P], int (&ix)[P],
                                             unsigned long long a, int idx) {
  bool g[P];
#pragma unroll
  for (int r = 0; r < P; ++r) g[r] = a > v[r];
#pragma unroll
  for (int r = P - 1; r >= 1; --r) {
    const unsigned long long vr = g[r - 1] ? v[r - 1] : (g[r] ? a : v[r]);
    const int ir = g[r - 1] ? ix[r - 1] : (g[r] ? idx : ix[r]);
    v[r] = vr;
    ix[r] = ir;
  }
  v[0] = g[0] ? a : v[0];
  ix[0] = g[0] ? idx : ix[0];
}
__device__ __forceinline__ unsigned long long abs_bits(double x) {
  return (unsigned long long)__double_as_longlong(x) & 0x7FFFFFFFFFFFFFFFull;
}

template <int P>
__device__ __forceinline__ void tp_init(double (&v)[P], int (&ix)[P]) {
#pragma unroll
  for (int r = 0; r < P; ++r) { v[r] = -1.0; ix[r] = -1; }
}

// merge the partner lane's list (xor-shuffle) into ours
template <int P>
__device__ __forceinline__ void tp_shfl_merge(double (&v)[P], int (&ix)[P], int lane_mask,
                                              unsigned member = 0xffffffffu) {
  double ov[P];
  int oi[P];
#pragma unroll
  for (int r = 0; r < P; ++r) {
    ov[r] = __shfl_xor_sync(member, v[r], lane_mask);
    oi[r] = __shfl_xor_sync(member, ix[r], lane_mask);
  }
#pragma unroll
  for (int r = 0; r < P; ++r) tp_insert<P>(v, ix, ov[r], oi[r]);
}

// ----------------------------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void fence_barrier_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
  uint32_t addr = smem_u32(bar);
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra WAIT_%=;\n"
      "}\n" ::"r"(addr),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_prefetch_desc(const CUtensorMap *tm) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(tm)) : "memory");
}
// 2D tiled TMA load global -> shared, completion on an mbarrier (complete_tx::bytes)
__device__ __forceinline__ void tma_load_2d(void *smem_dst, const CUtensorMap *tm, uint64_t *bar,
                                            int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(smem_u32(smem_dst)),
      "l"(reinterpret_cast<uint64_t>(tm)), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
      : "memory");
}

// programmatic dependent launch: wait for the preceding grid's completion (and its memory)
__device__ __forceinline__ void griddep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void griddep_launch_dependents() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

// 3D tiled TMA load global -> shared (complete_tx on an mbarrier)
__device__ __forceinline__ void tma_load_3d(void *smem_dst, const CUtensorMap *tm, uint64_t *bar,
                                            int c0, int c1, int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(smem_u32(smem_dst)),
      "l"(reinterpret_cast<uint64_t>(tm)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2)
      : "memory");
}


}  // namespace aabft
