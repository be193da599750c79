// api.cu -- the C ABI of include/aabft.h: validation, workspace sizing, dispatch, errors.
// No C++ exception crosses the ABI; every entry point is stream-ordered and never allocates.
#include <cstdlib>
#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>
#include <vector>

#include "common.cuh"

namespace aabft {

namespace {
thread_local char g_err[512] = "";
std::atomic<int64_t> g_launches{0};
int g_dev_ok[64] = {0};  // 0 unknown, 1 ok, 2 unsupported

inline size_t r256(size_t b) { return (b + 255) / 256 * 256; }

bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; }
}  // namespace

void set_error(const char *fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof g_err, fmt, ap);
  va_end(ap);
}

int64_t next_launch(int64_t n) { return g_launches.fetch_add(n) + n; }

aabft_status check_launch(const char *what) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    set_error("%s: %s", what, cudaGetErrorString(e));
    return AABFT_ECUDA;
  }
  return AABFT_OK;
}

int eff_t(const aabft_config *cfg) {
  if (cfg->t > 0) return cfg->t;
  return cfg->dtype == AABFT_F64 ? 52 : 23;
}

size_t elem_size(const aabft_config *cfg) { return cfg->dtype == AABFT_F64 ? 8 : 4; }

double sigma_coeff(int64_t K, int fma_model) {
  const double dn = (double)K;
  double F;
  if (fma_model) F = ((dn * (dn + 1.0)) * (2.0 * dn + 1.0)) / 48.0;
  else F = ((dn * (dn + 1.0)) * (dn + 0.5) + 2.0 * dn) / 24.0;
  return std::sqrt(F);
}

BoundParams make_bound_params(const aabft_config *cfg) {
  BoundParams b;
  const int t = eff_t(cfg);
  b.s = sigma_coeff(cfg->K, cfg->fma_model);
  b.two_mt = std::ldexp(1.0, -t);
  b.two_m2t = std::ldexp(1.0, -2 * t);
  b.omega = cfg->omega;
  b.ev_coeff = (double)cfg->K / 3.0;
  b.fma_model = cfg->fma_model;
  b.p = cfg->p;
  return b;
}

aabft_status validate(const aabft_config *c) {
  if (!c) { set_error("config is NULL"); return AABFT_EINVAL; }
  if (c->dtype != AABFT_F64 && c->dtype != AABFT_F32) { set_error("dtype %d", c->dtype); return AABFT_EINVAL; }
  if (c->M < 1 || c->N < 1 || c->K < 1) { set_error("M, N, K must be >= 1"); return AABFT_EINVAL; }
  if (c->K >= (int64_t)1 << 31) { set_error("K must be < 2^31"); return AABFT_EINVAL; }
  if (c->bs < 8 || c->bs > 256 || (c->bs & (c->bs - 1))) { set_error("bs=%d must be a power of 2 in [8,256]", c->bs); return AABFT_EINVAL; }
  if (c->M % c->bs || c->N % c->bs) { set_error("M and N must be multiples of bs (zero-pad, P:L353)"); return AABFT_EINVAL; }
  if (c->p < 1 || c->p > 8 || c->p > c->K) { set_error("p=%d must be in [1, min(8, K)]", c->p); return AABFT_EINVAL; }
  if (!(c->omega > 0.0) || !std::isfinite(c->omega)) { set_error("omega must be positive and finite"); return AABFT_EINVAL; }
  if (c->t < 0 || c->t > 200) { set_error("t=%d out of range", c->t); return AABFT_EINVAL; }
  if (c->fma_model != 0 && c->fma_model != 1) { set_error("fma_model must be 0 or 1"); return AABFT_EINVAL; }
  if ((c->M / c->bs) * (c->N / c->bs) >= ((int64_t)1 << 31)) { set_error("too many blocks"); return AABFT_EINVAL; }
  // launch-geometry limit (gridDim.y <= 65535): block-rows of A in the streaming check
  if (c->M / c->bs > 65535) { set_error("M/bs = %lld exceeds 65535 block-rows", (long long)(c->M / c->bs)); return AABFT_EINVAL; }
  return AABFT_OK;
}

static aabft_status device_ok() {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return check_launch("cudaGetDevice");
  if (dev < 0 || dev >= 64) return AABFT_EUNSUPPORTED;
  if (g_dev_ok[dev] == 0) {
    int major = 0, minor = 0;
    cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
    cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev);
    g_dev_ok[dev] = (major == 10 && minor == 0) ? 1 : 2;
    if (g_dev_ok[dev] == 2) set_error("device %d is sm_%d%d; this library is built for sm_100a", dev, major, minor);
  }
  if (g_dev_ok[dev] != 1) {
    set_error("device is not sm_100 (B200); library built for sm_100a only");
    return AABFT_EUNSUPPORTED;
  }
  return AABFT_OK;
}

// rows of a row-major operand fed to TMA / vector loads: base 16-B aligned, pitch 16-B multiple
static size_t gemm_ws_bytes(const aabft_config *c) {
  return c->dtype == AABFT_F64 ? gemm_f64_ws_bytes(c) : 0;
}
// [encode partial top-p lists | SEA norms][FP64 GEMM split-K partials + flags]
static size_t front_ws_bytes(const aabft_config *c) {
  return r256(std::max(encode_ws_bytes(c), sea_ws_bytes(c)));
}
static void *gemm_ws(const aabft_config *c, void *ws) {
  return static_cast<char *>(ws) + front_ws_bytes(c);
}

// the check's counter accumulator: the workspace's trailing 256 bytes (10 words used),
// zeroed by aabft_gemm of the protected product and re-armed by the check's last CTA
static unsigned long long *check_acc(const aabft_config *c, void *ws) {
  return reinterpret_cast<unsigned long long *>(static_cast<char *>(ws) + front_ws_bytes(c) +
                                                r256(gemm_ws_bytes(c)));
}

static bool pitch_ok(const aabft_config *c, const void *p, int64_t ld) {
  return aligned16(p) && ((size_t)ld * elem_size(c)) % 16 == 0;
}

}  // namespace aabft

using namespace aabft;

#define AABFT_GUARD_BEGIN try {
#define AABFT_GUARD_END                                     \
  }                                                         \
  catch (...) {                                             \
    set_error("internal error (exception caught at ABI)"); \
    return AABFT_EINTERNAL;                                 \
  }

extern "C" {

size_t aabft_workspace_bytes(const aabft_config *cfg) {
  if (validate(cfg) != AABFT_OK) return 0;
  return front_ws_bytes(cfg) + r256(gemm_ws_bytes(cfg)) + 256;
}

size_t aabft_gemm_plain_workspace_bytes(const aabft_config *cfg) {
  if (validate(cfg) != AABFT_OK) return 0;
  return cfg->dtype == AABFT_F64 ? r256(gemm_f64_plain_ws_bytes()) : 256;
}

aabft_status aabft_encode(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                          int64_t ldb, const aabft_encoded *out, void *ws, size_t ws_bytes,
                          void *stream) {
  AABFT_GUARD_BEGIN
  aabft_status s = validate(cfg);
  if (s != AABFT_OK) return s;
  if (!out) { set_error("out is NULL"); return AABFT_EINVAL; }
  if (!A && !B) { set_error("A and B are both NULL"); return AABFT_EINVAL; }
  // top-p tables: both pointers or neither (neither = checksums only, NEXT-3 comparators)
  if (A && (lda < cfg->K || !out->Acs || out->ld_acs < cfg->K || (!out->topA_val != !out->topA_idx))) {
    set_error("encode A: need lda >= K, Acs (ld_acs >= K), topA_val and topA_idx both set or both NULL");
    return AABFT_EINVAL;
  }
  if (B && (ldb < cfg->N || !out->Bcs || out->ld_bcs < cfg->N / cfg->bs || (!out->topB_val != !out->topB_idx))) {
    set_error("encode B: need ldb >= N, Bcs (ld_bcs >= N/bs), topB_val and topB_idx both set or both NULL");
    return AABFT_EINVAL;
  }
  if ((A && !pitch_ok(cfg, A, lda)) || (B && !pitch_ok(cfg, B, ldb))) {
    set_error("encode: A/B must be 16-byte aligned with row pitches that are multiples of 16 bytes");
    return AABFT_EINVAL;
  }
  if (!ws || ws_bytes < aabft_workspace_bytes(cfg)) {
    set_error("workspace too small: need %zu bytes", aabft_workspace_bytes(cfg));
    return AABFT_EWORKSPACE;
  }
  if ((s = device_ok()) != AABFT_OK) return s;
  return launch_encode(cfg, A, lda, B, ldb, out, ws, (cudaStream_t)stream);
  AABFT_GUARD_END
}

aabft_status aabft_bound(const aabft_config *cfg, const aabft_encoded *enc, double *eps_col,
                         double *sig_col, double *eps_row, double *sig_row, void *stream) {
  AABFT_GUARD_BEGIN
  aabft_status s = validate(cfg);
  if (s != AABFT_OK) return s;
  if (!enc || !enc->topA_val || !enc->topA_idx || !enc->topB_val || !enc->topB_idx) {
    set_error("bound: top-p tables required");
    return AABFT_EINVAL;
  }
  if ((s = device_ok()) != AABFT_OK) return s;
  return launch_bound(cfg, enc, eps_col, sig_col, eps_row, sig_row, (cudaStream_t)stream);
  AABFT_GUARD_END
}

aabft_status aabft_bound_elements(const aabft_config *cfg, const aabft_encoded *enc,
                                  const int64_t *rows, const int64_t *cols, int64_t n,
                                  double *sig, double *eps, void *stream) {
  AABFT_GUARD_BEGIN
  aabft_status s = validate(cfg);
  if (s != AABFT_OK) return s;
  if (!enc || !enc->topA_val || !enc->topA_idx || !enc->topB_val || !enc->topB_idx) {
    set_error("bound_elements: top-p tables required");
    return AABFT_EINVAL;
  }
  if (n < 0 || (n > 0 && (!rows || !cols || (!sig && !eps)))) {
    set_error("bound_elements: rows, cols and sig or eps required");
    return AABFT_EINVAL;
  }
  if ((s = device_ok()) != AABFT_OK) return s;
  return launch_bound_elements(cfg, enc, rows, cols, n, sig, eps, (cudaStream_t)stream);
  AABFT_GUARD_END
}

aabft_status aabft_checksum_errors(const aabft_config *cfg, const void *A, int64_t lda,
                                   const void *B, int64_t ldb, const aabft_encoded *enc,
                                   const aabft_product *prod, double *err_col, double *err_row,
                                   void *stream) {
  AABFT_GUARD_BEGIN
  aabft_status s = validate(cfg);
  if (s != AABFT_OK) return s;
  if (!A || !B || !enc || !enc->Acs || !enc->Bcs || !prod || !prod->Ccol || !prod->Crow ||
      !err_col || !err_row || lda < cfg->K || ldb < cfg->N) {
    set_error("checksum_errors: A, B, Acs, Bcs, Ccol, Crow, err_col, err_row required");
    return AABFT_EINVAL;
  }
  if ((s = device_ok()) != AABFT_OK) return s;
  return launch_checksum_errors(cfg, A, lda, B, ldb, enc, prod, err_col, err_row, (cudaStream_t)stream);
  AABFT_GUARD_END
}

static aabft_status gemm_common(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                                int64_t ldb, const aabft_encoded *enc, const aabft_product *out,
                                const aabft_fault *faults, int32_t nfaults, bool plain,
                                void *ws, size_t ws_bytes, void *stream) {
  aabft_status s = validate(cfg);
  if (s != AABFT_OK) return s;
  const size_t need = plain ? aabft_gemm_plain_workspace_bytes(cfg) : aabft_workspace_bytes(cfg);
  if (!ws || ws_bytes < need) {
    set_error("workspace too small: need %zu bytes", need);
    return AABFT_EWORKSPACE;
  }
  if (!A || !B || !out || !out->C) { set_error("gemm: A, B, C required"); return AABFT_EINVAL; }
  if (lda < cfg->K || ldb < cfg->N || out->ldc < cfg->N) { set_error("gemm: lda >= K, ldb >= N, ldc >= N required"); return AABFT_EINVAL; }
  if (!pitch_ok(cfg, A, lda) || !pitch_ok(cfg, B, ldb) || !aligned16(out->C)) {
    set_error("gemm: A/B/C must be 16-byte aligned with row pitches that are multiples of 16 bytes");
    return AABFT_EINVAL;
  }
  if (!plain) {
    if (!enc || !enc->Acs || !enc->Bcs || !out->Ccol || !out->Crow) { set_error("gemm: Acs, Bcs, Ccol, Crow required"); return AABFT_EINVAL; }
    if (enc->ld_acs < cfg->K || enc->ld_bcs < cfg->N / cfg->bs || out->ld_ccol < cfg->N || out->ld_crow < cfg->N / cfg->bs) {
      set_error("gemm: checksum leading dimensions too small");
      return AABFT_EINVAL;
    }
    if (!pitch_ok(cfg, enc->Acs, enc->ld_acs) || !pitch_ok(cfg, enc->Bcs, enc->ld_bcs)) {
      set_error("gemm: Acs/Bcs must be 16-byte aligned with 16-byte-multiple row pitches (pad ld_bcs)");
      return AABFT_EINVAL;
    }
    if (nfaults < 0 || (nfaults > 0 && !faults)) { set_error("gemm: bad fault list"); return AABFT_EINVAL; }
  }
  if ((s = device_ok()) != AABFT_OK) return s;
  if (cfg->dtype == AABFT_F64)
    return launch_gemm_f64(cfg, A, lda, B, ldb, enc, out, plain ? nullptr : faults, plain ? 0 : nfaults, plain,
                           plain ? ws : gemm_ws(cfg, ws), plain ? nullptr : check_acc(cfg, ws),
                           (cudaStream_t)stream);
  return launch_gemm_f32(cfg, A, lda, B, ldb, enc, out, plain ? nullptr : faults, plain ? 0 : nfaults, plain,
                         plain ? nullptr : check_acc(cfg, ws), (cudaStream_t)stream);
}

aabft_status aabft_gemm(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                        int64_t ldb, const aabft_encoded *enc, const aabft_product *out,
                        const aabft_fault *faults, int32_t nfaults, void *ws, size_t ws_bytes,
                        void *stream) {
  AABFT_GUARD_BEGIN
  return gemm_common(cfg, A, lda, B, ldb, enc, out, faults, nfaults, false, ws, ws_bytes, stream);
  AABFT_GUARD_END
}

aabft_status aabft_gemm_plain(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                              int64_t ldb, void *C, int64_t ldc, void *ws, size_t ws_bytes,
                              void *stream) {
  AABFT_GUARD_BEGIN
  aabft_product out{};
  out.C = C;
  out.ldc = ldc;
  return gemm_common(cfg, A, lda, B, ldb, nullptr, &out, nullptr, 0, true, ws, ws_bytes, stream);
  AABFT_GUARD_END
}

static aabft_status check_common(const aabft_config *cfg, const aabft_encoded *enc,
                                 const aabft_product *prod, aabft_block_report *rep,
                                 aabft_counts *cnt) {
  aabft_status s = validate(cfg);
  if (s != AABFT_OK) return s;
  if (!enc || !enc->topA_val || !enc->topA_idx || !enc->topB_val || !enc->topB_idx) { set_error("check: top-p tables required"); return AABFT_EINVAL; }
  if (!prod || !prod->C || !prod->Ccol || !prod->Crow || !rep || !cnt) { set_error("check: C, Ccol, Crow, reports, counts required"); return AABFT_EINVAL; }
  if (prod->ldc < cfg->N || prod->ld_ccol < cfg->N || prod->ld_crow < cfg->N / cfg->bs) { set_error("check: leading dimensions too small"); return AABFT_EINVAL; }
  return device_ok();
}

aabft_status aabft_check(const aabft_config *cfg, const aabft_encoded *enc,
                         const aabft_product *prod, aabft_block_report *reports,
                         aabft_counts *counts, void *ws, size_t ws_bytes, void *stream) {
  AABFT_GUARD_BEGIN
  aabft_status s = check_common(cfg, enc, prod, reports, counts);
  if (s != AABFT_OK) return s;
  const bool fused = prod->Rcol && prod->Rrow && fused_check_ok(cfg);
  if (fused && (!ws || ws_bytes < aabft_workspace_bytes(cfg))) {
    set_error("check (fused): the aabft_gemm workspace is required");
    return AABFT_EWORKSPACE;
  }
  // fused: the GEMM's workspace, whose check accumulator that GEMM zeroed (no memset here)
  return launch_check(cfg, enc, prod, reports, counts, fused ? gemm_ws(cfg, ws) : nullptr,
                      fused ? check_acc(cfg, ws) : nullptr, (cudaStream_t)stream);
  AABFT_GUARD_END
}

aabft_status aabft_correct(const aabft_config *cfg, const aabft_encoded *enc,
                           const aabft_product *prod, aabft_block_report *reports,
                           aabft_counts *counts, void *stream) {
  AABFT_GUARD_BEGIN
  aabft_status s = check_common(cfg, enc, prod, reports, counts);
  if (s != AABFT_OK) return s;
  return launch_correct(cfg, enc, prod, reports, counts, (cudaStream_t)stream);
  AABFT_GUARD_END
}

// ------------------------------------------------------------------ NEXT-3 comparators
aabft_status aabft_sea_bound(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                             int64_t ldb, const aabft_encoded *enc, double *eps_col,
                             double *eps_row, double *eps_corner, void *ws, size_t ws_bytes,
                             void *stream) {
  AABFT_GUARD_BEGIN
  aabft_status s = validate(cfg);
  if (s != AABFT_OK) return s;
  if (!A || !B || !enc || !enc->Acs || !enc->Bcs || lda < cfg->K || ldb < cfg->N ||
      enc->ld_acs < cfg->K || enc->ld_bcs < cfg->N / cfg->bs) {
    set_error("sea_bound: A (lda >= K), B (ldb >= N), Acs, Bcs required");
    return AABFT_EINVAL;
  }
  if (!eps_col && !eps_row && !eps_corner) { set_error("sea_bound: no output"); return AABFT_EINVAL; }
  if (!pitch_ok(cfg, A, lda) || !pitch_ok(cfg, enc->Acs, enc->ld_acs)) {
    set_error("sea_bound: A / Acs must be 16-byte aligned with 16-byte-multiple row pitches");
    return AABFT_EINVAL;
  }
  if (!ws || ws_bytes < aabft_workspace_bytes(cfg)) {
    set_error("workspace too small: need %zu bytes", aabft_workspace_bytes(cfg));
    return AABFT_EWORKSPACE;
  }
  if ((s = device_ok()) != AABFT_OK) return s;
  return launch_sea_bound(cfg, A, lda, B, ldb, enc, eps_col, eps_row, eps_corner, ws,
                          (cudaStream_t)stream);
  AABFT_GUARD_END
}

static aabft_status ext_common(const aabft_config *cfg, const aabft_product *prod,
                               double eps_fixed, aabft_block_report *rep, aabft_counts *cnt) {
  aabft_status s = validate(cfg);
  if (s != AABFT_OK) return s;
  if (!prod || !prod->C || !prod->Ccol || !prod->Crow || !rep || !cnt) { set_error("check_ext: C, Ccol, Crow, reports, counts required"); return AABFT_EINVAL; }
  if (prod->ldc < cfg->N || prod->ld_ccol < cfg->N || prod->ld_crow < cfg->N / cfg->bs) { set_error("check_ext: leading dimensions too small"); return AABFT_EINVAL; }
  if (!(eps_fixed >= 0.0)) { set_error("check_ext: eps_fixed must be >= 0"); return AABFT_EINVAL; }
  return device_ok();
}

aabft_status aabft_check_ext(const aabft_config *cfg, const aabft_product *prod,
                             const double *eps_col, const double *eps_row, double eps_fixed,
                             aabft_block_report *reports, aabft_counts *counts, void *ws,
                             size_t ws_bytes, void *stream) {
  AABFT_GUARD_BEGIN
  aabft_status s = ext_common(cfg, prod, eps_fixed, reports, counts);
  if (s != AABFT_OK) return s;
  const bool fused = prod->Rcol && prod->Rrow && fused_check_ok(cfg);
  if (fused && (!ws || ws_bytes < aabft_workspace_bytes(cfg))) {
    set_error("check_ext (fused): the aabft_gemm workspace is required");
    return AABFT_EWORKSPACE;
  }
  return launch_check_ext(cfg, prod, eps_col, eps_row, eps_fixed, reports, counts,
                          fused ? gemm_ws(cfg, ws) : nullptr, fused ? check_acc(cfg, ws) : nullptr,
                          (cudaStream_t)stream);
  AABFT_GUARD_END
}

aabft_status aabft_correct_ext(const aabft_config *cfg, const aabft_product *prod,
                               const double *eps_row, double eps_fixed,
                               aabft_block_report *reports, aabft_counts *counts, void *stream) {
  AABFT_GUARD_BEGIN
  aabft_status s = ext_common(cfg, prod, eps_fixed, reports, counts);
  if (s != AABFT_OK) return s;
  return launch_correct_ext(cfg, prod, eps_row, eps_fixed, reports, counts, (cudaStream_t)stream);
  AABFT_GUARD_END
}

}  // extern "C"

// ------------------------------------------------------------------ host end-to-end entry point
// Pipelined: A is split into S row slabs and B into S column panels (S <= 4, multiples of
// lcm(bs, 64)); the S x S blocks of C are protected GEMMs of their own (every BS x BS block
// lies in exactly one of them, so the check is unchanged).  Host->device copies run on a copy
// stream in the order A0, B0, B1, A1, ..., B(S-1), A(S-1), the compute stream starts block
// (i, j) as soon as A_i and B_j have landed (encode of a slab / panel runs once), and each
// finished C block is
// copied back on a third stream -- PCIe in both directions overlaps the DMMA GEMMs.
namespace {
constexpr int kMaxSplit = 8, kDefaultSplit = 4;
struct Split {
  int S;
  int64_t ms, ns;  // slab rows / panel cols (last may be shorter)
};
Split plan_split(const aabft_config *c) {
  // slab rows: multiples of lcm(bs, 64) = max(bs, 64) (bs is a power of two); panel columns
  // additionally keep the Bcs / Crow column offsets 16-byte aligned (4 x (N/bs) granules)
  const int64_t unit = std::max<int64_t>(64, c->bs), unit_n = 4 * unit;
  Split sp;
  // S x S blocks: finer splits start the GEMMs earlier and leave less work after the last
  // host->device copy, at the cost of smaller GEMM launches (AABFT_HOST_SPLIT overrides the cap)
  static const int cap = [] {
    const char *e = std::getenv("AABFT_HOST_SPLIT");
    const int v = e ? std::atoi(e) : 0;
    return v >= 1 && v <= kMaxSplit ? v : kDefaultSplit;
  }();
  sp.S = (int)std::max<int64_t>(1, std::min<int64_t>(cap, std::min(c->M / (4 * unit), c->N / unit_n)));
  sp.ms = (c->M / sp.S + unit - 1) / unit * unit;
  sp.ns = (c->N / sp.S + unit_n - 1) / unit_n * unit_n;
  return sp;
}
int64_t piece(int64_t total, int64_t step, int i) {
  const int64_t lo = step * i;
  return lo >= total ? 0 : std::min(step, total - lo);
}
struct Arena {
  int64_t lda, ldb, ldc, ld_acs, ld_bcs, ld_ccol, ld_crow;
  size_t oA, oB, oC, oAcs, oBcs, oCcol, oCrow, oRcol, oRrow, oTav, oTai, oTbv, oTbi, oRep, oCnt,
      oCntAll, oWs, oWs2, total;
};
Arena plan_arena(const aabft_config *c) {
  Arena a;
  const size_t es = elem_size(c);
  const int64_t q = 16 / (int64_t)es;  // elements per 16 bytes
  auto rnd = [q](int64_t n) { return (n + q - 1) / q * q; };
  a.lda = rnd(c->K); a.ldb = rnd(c->N); a.ldc = rnd(c->N);
  a.ld_acs = rnd(c->K); a.ld_bcs = rnd(c->N / c->bs);
  a.ld_ccol = rnd(c->N); a.ld_crow = rnd(c->N / c->bs);
  const Split sp = plan_split(c);
  size_t o = 0;
  auto take = [&o](size_t bytes) { size_t r = o; o += r256(bytes); return r; };
  a.oA = take(c->M * a.lda * es);
  a.oB = take(c->K * a.ldb * es);
  a.oC = take(c->M * a.ldc * es);
  a.oAcs = take((c->M / c->bs) * a.ld_acs * es);
  a.oBcs = take(c->K * a.ld_bcs * es);
  a.oCcol = take((c->M / c->bs) * a.ld_ccol * es);
  a.oCrow = take(c->M * a.ld_crow * es);
  a.oRcol = take((c->M / c->bs) * c->N * 8 + 256 * sp.S * sp.S);
  a.oRrow = take(c->M * (c->N / c->bs) * 8 + 256 * sp.S * sp.S);
  a.oTav = take((c->M + c->M / c->bs) * c->p * 8 + 256 * sp.S);
  a.oTai = take((c->M + c->M / c->bs) * c->p * 4 + 256 * sp.S);
  a.oTbv = take((c->N + c->N / c->bs) * c->p * 8 + 256 * sp.S);
  a.oTbi = take((c->N + c->N / c->bs) * c->p * 4 + 256 * sp.S);
  a.oRep = take((c->M / c->bs) * (c->N / c->bs) * sizeof(aabft_block_report) + 256 * sp.S * sp.S);
  a.oCnt = take(sizeof(aabft_counts) * sp.S * sp.S);
  a.oCntAll = take(sizeof(aabft_counts));
  a.oWs = take(aabft_workspace_bytes(c));
  a.oWs2 = take(aabft_workspace_bytes(c));  // the second compute stream's workspace
  a.total = o;
  return a;
}
struct HostPipe {  // per-device copy / compute streams + event pool (created once)
  cudaStream_t in = nullptr, out = nullptr, c2 = nullptr;
  cudaEvent_t ev[2 * kMaxSplit + kMaxSplit * kMaxSplit + 2];
  cudaEvent_t enc[2 * kMaxSplit + 2];  // encode of A_i / B_j done; second stream done
  bool ok = false;
};
HostPipe &host_pipe() {
  static thread_local HostPipe hp[64];
  int dev = 0;
  cudaGetDevice(&dev);
  HostPipe &h = hp[dev & 63];
  if (!h.ok) {
    if (cudaStreamCreateWithFlags(&h.in, cudaStreamNonBlocking) != cudaSuccess ||
        cudaStreamCreateWithFlags(&h.out, cudaStreamNonBlocking) != cudaSuccess ||
        cudaStreamCreateWithFlags(&h.c2, cudaStreamNonBlocking) != cudaSuccess)
      return h;
    for (auto &e : h.ev)
      if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return h;
    for (auto &e : h.enc)
      if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return h;
    h.ok = true;
  }
  return h;
}
}  // namespace

extern "C" {

size_t aabft_host_arena_bytes(const aabft_config *cfg) {
  if (validate(cfg) != AABFT_OK) return 0;
  return plan_arena(cfg).total;
}

aabft_status aabft_protected_gemm_host(const aabft_config *cfg, const void *A_host,
                                       const void *B_host, void *C_host,
                                       aabft_counts *counts_host, void *arena,
                                       size_t arena_bytes, void *stream) {
  AABFT_GUARD_BEGIN
  aabft_status s = validate(cfg);
  if (s != AABFT_OK) return s;
  if (!A_host || !B_host || !C_host) { set_error("host buffers required"); return AABFT_EINVAL; }
  const Arena a = plan_arena(cfg);
  if (!arena || arena_bytes < a.total) { set_error("arena too small: need %zu bytes", a.total); return AABFT_EWORKSPACE; }
  if (!aligned16(arena)) { set_error("arena must be 16-byte aligned"); return AABFT_EINVAL; }
  HostPipe &hp = host_pipe();
  if (!hp.ok) return check_launch("copy stream / event creation");
  cudaStream_t st = (cudaStream_t)stream;
  char *base = static_cast<char *>(arena);
  const size_t es = elem_size(cfg);
  const int64_t M = cfg->M, N = cfg->N, K = cfg->K, bs = cfg->bs, p = cfg->p;
  const Split sp = plan_split(cfg);
  const int S = sp.S;
  cudaEvent_t *evA = hp.ev, *evB = hp.ev + kMaxSplit, *evC = hp.ev + 2 * kMaxSplit;  // S*S
  cudaEvent_t evStart = hp.ev[2 * kMaxSplit + kMaxSplit * kMaxSplit];
  cudaEvent_t evOutDone = hp.ev[2 * kMaxSplit + kMaxSplit * kMaxSplit + 1];
  // the copy streams start after whatever the caller enqueued before this call
  if (cudaEventRecord(evStart, st) != cudaSuccess || cudaStreamWaitEvent(hp.in, evStart, 0) != cudaSuccess ||
      cudaStreamWaitEvent(hp.out, evStart, 0) != cudaSuccess ||
      cudaStreamWaitEvent(hp.c2, evStart, 0) != cudaSuccess)
    return check_launch("pipeline start");
  // two compute streams: consecutive blocks alternate between them and each FP64 GEMM runs on
  // half the persistent grid (AABFT_FLAG_GEMM_HALF_GRID), so one block's stream-K tail
  // overlaps the next block's data-parallel waves instead of idling SMs
  const bool two = cfg->dtype == AABFT_F64 && sp.S > 1 && !std::getenv("AABFT_HOST_ONE_STREAM");
  cudaEvent_t *evEncA = hp.enc, *evEncB = hp.enc + kMaxSplit;
  cudaEvent_t evC2Done = hp.enc[2 * kMaxSplit];
  // AABFT_HOST_TRACE=1: timing events per copy / block, printed to stderr after the call
  // (diagnostics for the pipeline's schedule; no effect on results)
  static const bool trace = std::getenv("AABFT_HOST_TRACE") != nullptr;
  struct Mark { cudaEvent_t e; char what[24]; };
  std::vector<Mark> marks;
  auto mark = [&](cudaStream_t on, const char *what, int x, int y) {
    if (!trace) return;
    Mark m;
    cudaEventCreate(&m.e);
    cudaEventRecord(m.e, on);
    std::snprintf(m.what, sizeof m.what, "%s %d %d", what, x, y);
    marks.push_back(m);
  };
  mark(st, "start", 0, 0);
  // host -> device in the order A0, B0, B1, A1, B2, A2, ..., B(S-1), A(S-1): every piece after
  // the first pair unlocks GEMM blocks at once, and the last one (an A slab) unlocks only one
  // block-row, so the work left after the final copy is S blocks rather than 2S - 1
  int ord_kind[2 * kMaxSplit], ord_idx[2 * kMaxSplit];  // kind 0 = A slab, 1 = B panel
  for (int i = 0; i < S; ++i) {
    ord_kind[2 * i] = i == 0 ? 0 : 1;
    ord_kind[2 * i + 1] = i == 0 ? 1 : 0;
    ord_idx[2 * i] = ord_idx[2 * i + 1] = i;
  }
  for (int o = 0; o < 2 * S; ++o) {
    const int i = ord_idx[o];
    if (ord_kind[o] == 0) {
      const int64_t mi = piece(M, sp.ms, i);
      if (mi > 0 && cudaMemcpy2DAsync(base + a.oA + (size_t)(i * sp.ms) * a.lda * es, a.lda * es,
                                      static_cast<const char *>(A_host) + (size_t)(i * sp.ms) * K * es,
                                      K * es, K * es, mi, cudaMemcpyHostToDevice, hp.in) != cudaSuccess)
        return check_launch("host->device copy (A)");
      cudaEventRecord(evA[i], hp.in);
      mark(hp.in, "h2d A", i, 0);
    } else {
      const int64_t nj = piece(N, sp.ns, i);
      if (nj > 0 && cudaMemcpy2DAsync(base + a.oB + (size_t)(i * sp.ns) * es, a.ldb * es,
                                      static_cast<const char *>(B_host) + (size_t)(i * sp.ns) * es,
                                      N * es, nj * es, K, cudaMemcpyHostToDevice, hp.in) != cudaSuccess)
        return check_launch("host->device copy (B)");
      cudaEventRecord(evB[i], hp.in);
      mark(hp.in, "h2d B", i, 0);
    }
  }
  const size_t wsb = aabft_workspace_bytes(cfg);
  auto *cnt_blocks = reinterpret_cast<aabft_counts *>(base + a.oCnt);
  // per-slab / per-panel top-p tables and per-block reference sums / reports (dense, block-major)
  auto tav = [&](int i) { return reinterpret_cast<double *>(base + a.oTav) + (i * sp.ms + i * (sp.ms / bs)) * p; };
  auto tai = [&](int i) { return reinterpret_cast<int32_t *>(base + a.oTai) + (i * sp.ms + i * (sp.ms / bs)) * p; };
  auto tbv = [&](int j) { return reinterpret_cast<double *>(base + a.oTbv) + (j * sp.ns + j * (sp.ns / bs)) * p; };
  auto tbi = [&](int j) { return reinterpret_cast<int32_t *>(base + a.oTbi) + (j * sp.ns + j * (sp.ns / bs)) * p; };
  size_t rcol_off = 0, rrow_off = 0, rep_off = 0;
  bool encA[kMaxSplit] = {}, encB[kMaxSplit] = {};
  int nblk = 0;
  // compute order = arrival order: each piece runs the blocks it completes, so block (i, j)
  // starts as soon as both A_i and B_j are resident
  auto run_block = [&](int i, int j) -> aabft_status {
      const int64_t mi = piece(M, sp.ms, i), nj = piece(N, sp.ns, j);
      if (mi <= 0 || nj <= 0) return AABFT_OK;
      aabft_status s;
      aabft_config cb = *cfg;
      cb.M = mi;
      cb.N = nj;
      if (two) cb.flags |= AABFT_FLAG_GEMM_HALF_GRID;
      cb.flags |= AABFT_FLAG_CHECK_CORRECTS;  // correction inside the check kernel
      const bool second = two && (nblk & 1);
      cudaStream_t cs = second ? hp.c2 : st;
      void *ws = base + (second ? a.oWs2 : a.oWs);
      const void *Ai = base + a.oA + (size_t)(i * sp.ms) * a.lda * es;
      const void *Bj = base + a.oB + (size_t)(j * sp.ns) * es;
      aabft_encoded enc{base + a.oAcs + (size_t)(i * sp.ms / bs) * a.ld_acs * es, a.ld_acs,
                        base + a.oBcs + (size_t)(j * sp.ns / bs) * es, a.ld_bcs,
                        tav(i), tai(i), tbv(j), tbi(j)};
      // encode a newly arrived slab / panel once (on this block's stream); blocks on the other
      // stream wait for that encode's event
      if (!encA[i]) {
        cudaStreamWaitEvent(cs, evA[i], 0);
        if ((s = aabft_encode(&cb, Ai, a.lda, nullptr, 0, &enc, ws, wsb, cs)) != AABFT_OK) return s;
        cudaEventRecord(evEncA[i], cs);
        encA[i] = true;
      } else {
        cudaStreamWaitEvent(cs, evEncA[i], 0);
      }
      if (!encB[j]) {
        cudaStreamWaitEvent(cs, evB[j], 0);
        if ((s = aabft_encode(&cb, nullptr, 0, Bj, a.ldb, &enc, ws, wsb, cs)) != AABFT_OK) return s;
        cudaEventRecord(evEncB[j], cs);
        encB[j] = true;
      } else {
        cudaStreamWaitEvent(cs, evEncB[j], 0);
      }
      aabft_product prod{base + a.oC + ((size_t)(i * sp.ms) * a.ldc + (size_t)(j * sp.ns)) * es, a.ldc,
                         base + a.oCcol + ((size_t)(i * sp.ms / bs) * a.ld_ccol + (size_t)(j * sp.ns)) * es, a.ld_ccol,
                         base + a.oCrow + ((size_t)(i * sp.ms) * a.ld_crow + (size_t)(j * sp.ns / bs)) * es, a.ld_crow,
                         reinterpret_cast<double *>(base + a.oRcol + rcol_off),
                         reinterpret_cast<double *>(base + a.oRrow + rrow_off)};
      auto *rep = reinterpret_cast<aabft_block_report *>(base + a.oRep + rep_off);
      rcol_off += r256((size_t)(mi / bs) * nj * 8);
      rrow_off += r256((size_t)mi * (nj / bs) * 8);
      rep_off += r256((size_t)(mi / bs) * (nj / bs) * sizeof(aabft_block_report));
      aabft_counts *cnt = cnt_blocks + nblk;
      if ((s = aabft_gemm(&cb, Ai, a.lda, Bj, a.ldb, &enc, &prod, nullptr, 0, ws, wsb, cs)) != AABFT_OK) return s;
      if ((s = aabft_check(&cb, &enc, &prod, rep, cnt, ws, wsb, cs)) != AABFT_OK) return s;
      // device -> host of the finished (corrected) C block on the copy-out stream
      cudaEventRecord(evC[nblk], cs);
      mark(cs, "block done", i, j);
      cudaStreamWaitEvent(hp.out, evC[nblk], 0);
      if (cudaMemcpy2DAsync(static_cast<char *>(C_host) + ((size_t)(i * sp.ms) * N + (size_t)(j * sp.ns)) * es,
                            N * es, prod.C, a.ldc * es, nj * es, mi, cudaMemcpyDeviceToHost, hp.out) != cudaSuccess)
        return check_launch("device->host copy (C)");
      mark(hp.out, "d2h", i, j);
      ++nblk;
      return AABFT_OK;
  };
  bool haveA[kMaxSplit] = {}, haveB[kMaxSplit] = {};
  for (int o = 0; o < 2 * S; ++o) {
    const int x = ord_idx[o];
    (ord_kind[o] == 0 ? haveA : haveB)[x] = true;
    for (int y = 0; y < S; ++y) {
      const bool other = ord_kind[o] == 0 ? haveB[y] : haveA[y];
      if (!other) continue;
      if ((s = ord_kind[o] == 0 ? run_block(x, y) : run_block(y, x)) != AABFT_OK) return s;
    }
  }
  // global counters = sum over the blocks (SUM n, MAX max_ratio), after both compute streams
  if (two) {
    cudaEventRecord(evC2Done, hp.c2);
    cudaStreamWaitEvent(st, evC2Done, 0);
  }
  auto *cnt_all = reinterpret_cast<aabft_counts *>(base + a.oCntAll);
  if ((s = launch_counts_sum(cnt_blocks, nblk, cnt_all, st)) != AABFT_OK) return s;
  if (counts_host && cudaMemcpyAsync(counts_host, cnt_all, sizeof(aabft_counts), cudaMemcpyDeviceToHost, st) != cudaSuccess)
    return check_launch("counts copy");
  cudaEventRecord(evOutDone, hp.out);
  cudaStreamWaitEvent(st, evOutDone, 0);
  if (cudaStreamSynchronize(st) != cudaSuccess) return check_launch("stream sync");
  if (trace) {
    for (auto &m : marks) {
      float ms = 0.f;
      cudaEventElapsedTime(&ms, marks[0].e, m.e);
      std::fprintf(stderr, "[aabft host trace] %8.3f ms  %s\n", ms, m.what);
    }
    for (auto &m : marks) cudaEventDestroy(m.e);
  }
  return AABFT_OK;
  AABFT_GUARD_END
}

const char *aabft_status_str(aabft_status s) {
  switch (s) {
    case AABFT_OK: return "AABFT_OK";
    case AABFT_EINVAL: return "AABFT_EINVAL: invalid argument";
    case AABFT_EUNSUPPORTED: return "AABFT_EUNSUPPORTED: device is not sm_100";
    case AABFT_ECUDA: return "AABFT_ECUDA: CUDA error";
    case AABFT_EWORKSPACE: return "AABFT_EWORKSPACE: workspace missing or too small";
    case AABFT_EINTERNAL: return "AABFT_EINTERNAL: internal error";
  }
  return "unknown aabft_status";
}

const char *aabft_last_error(void) { return g_err; }
const char *aabft_version(void) { return "aabft-b200 0.1 (sm_100a; DMMA f64 / FFMA f32)"; }
int64_t aabft_launch_count(void) { return g_launches.load(); }

}  // extern "C"
