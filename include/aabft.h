/*
 * aabft.h -- C ABI of the B200-native (sm_100a) A-ABFT hot path.
 *
 * A-ABFT: Braun, Halder, Wunderlich, "A-ABFT: Autonomous Algorithm-Based Fault Tolerance
 * for Matrix Multiplications on Graphics Processing Units", DSN 2014.  "P:Lnn" cites line
 * nn of the paper text; section / equation / algorithm given beside it.
 *
 * The path (§V):
 *   1. aabft_encode   -- partitioned checksums of A (column checksums per BS rows, Eq 1) and
 *                        of B (row checksums per BS columns, Eq 2) fused with the top-p
 *                        largest |values| of every row of A / column of B and of every
 *                        checksum row / column (Alg 1; step 3 global reduction)
 *   2. aabft_gemm     -- checksum-augmented product C_fc = A_cc . B_rc (Eq 3): C, the carried
 *                        column checksums Ccol = Acs.B and row checksums Crow = A.Bcs
 *   3. aabft_check    -- bound (§IV, Eq 28 / P:L287, upper bound y §IV-E), reference sums
 *                        (Eq 4), comparison (Eq 6) and 3-class classification
 *   4. aabft_correct  -- locate a single critical error at the intersection of the
 *                        mismatching row and column and correct it (Alg 2 output,
 *                        P:L385)
 * plus aabft_bound (the bound alone, §IV-E last paragraph P:L307) and aabft_gemm_plain (the
 * unprotected GEMM of the same kernel family; the overhead denominator).
 *
 * Conventions (all entry points):
 *  - Every matrix is ROW-MAJOR; "ld" is the row pitch in ELEMENTS.  All array pointers are
 *    DEVICE pointers unless the name ends in _host.  The caller owns all memory: the library
 *    never allocates, frees or synchronises (except aabft_protected_gemm_host, which
 *    synchronises its stream before returning because it writes host memory).
 *  - Every call is asynchronous on `stream` (a cudaStream_t passed as void*; NULL = legacy
 *    default stream).  AABFT_OK means "validated and enqueued".
 *  - Parameter checks run before any launch and return AABFT_EINVAL with a message in
 *    aabft_last_error().  Launch failures return AABFT_ECUDA.  A device that is not sm_100
 *    returns AABFT_EUNSUPPORTED.  No C++ exception crosses this ABI.
 *  - Inputs must be finite; non-finite RESULTS are always classified CRITICAL (reading R9).
 *  - Thread safety: calls are safe concurrently on distinct streams and buffers.
 */
#ifndef AABFT_H
#define AABFT_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  AABFT_OK = 0,
  AABFT_EINVAL = 1,        /* bad argument (dimension, ld, alignment, NULL, range) */
  AABFT_EUNSUPPORTED = 2,  /* not an sm_100 device */
  AABFT_ECUDA = 3,         /* CUDA launch / runtime error (message in aabft_last_error) */
  AABFT_EWORKSPACE = 4,    /* workspace NULL or too small */
  AABFT_EINTERNAL = 5
} aabft_status;

typedef enum { AABFT_F64 = 0, AABFT_F32 = 1 } aabft_dtype;

/* Problem description.  C[M x N] = A[M x K] . B[K x N].
 *  bs        checksum block size BS (partitioned encoding, P:L91 ref [20]); power of two in
 *            [8, 256]; M % bs == 0 and N % bs == 0 (the caller zero-pads: "padded matrix A",
 *            Alg 1; reading R20).  K is free (>= 1).
 *  p         numMax, the number of largest |values| per vector; 1..8, p <= K.
 *  omega     confidence scale of Eq 7; the paper uses 3.
 *  t         eps_M = 2^-t; 0 selects 52 (F64) / 23 (F32) (reading R1).
 *  fma_model 1: sigma of Eq 28 (FMA hardware, §IV-D) -- the default;
 *            0: sigma of P:L287 plus |EV_Prod| of Eq 43 (separately rounded products). */
typedef struct {
  int32_t dtype;  /* aabft_dtype: element type of A, B, C, Acs, Bcs, Ccol, Crow */
  int32_t bs;
  int64_t M, N, K;
  int32_t p;
  int32_t t;
  double omega;
  int32_t fma_model;
  int32_t flags;  /* AABFT_FLAG_* (0 = defaults) */
} aabft_config;

/* AABFT_FLAG_TOPP_IN_GEMM: move the top-p selection of step 1 (Alg 1) from
 * aabft_encode into aabft_gemm, which takes it from the operand tiles it already streams
 * through shared memory -- the paper runs this reduction "in parallel to the matrix
 * multiplication kernel".  Honoured where the GEMM supports it (FP64,
 * p <= 4); elsewhere aabft_encode selects as usual.  Either way the top-p tables of
 * aabft_encoded are complete once aabft_gemm (stream-ordered) has run, with identical
 * contents (value desc, index asc; bit-exact).  Opt-in: on B200 it measured slower than the
 * selection in aabft_encode. */
#define AABFT_FLAG_TOPP_IN_GEMM 1
/* AABFT_FLAG_GEMM_HALF_GRID: the FP64 aabft_gemm / aabft_gemm_plain launch uses half of the
 * persistent grid (1.5 CTAs per SM) so that two such calls on two streams can run side by side
 * (the host entry point's pipelined blocks use it).  A launch with a stream-K tail is
 * cooperative, so each grid is fully resident before it starts.  Results are identical up to
 * the FP64 summation order of split tiles (parity by tolerance, as always for FP64). */
#define AABFT_FLAG_GEMM_HALF_GRID 2
/* AABFT_FLAG_OVERLAP_ENCODE: step 1 runs CONCURRENTLY with the following aabft_gemm on the same
 * stream (the paper overlaps its top-p reduction with the multiplication, P:L320 / P:L368;
 * here the whole encode does).  aabft_encode (FP64, 16 <= bs <= 64, p <= 4, A, B and both
 * top-p tables given; otherwise the flag is ignored) launches a one-CTA-per-SM kernel small
 * enough to sit next to the GEMM's CTAs and marks the GEMM as a programmatic dependent launch;
 * aabft_gemm (FP64) then streams its data tiles at once and waits for the encode grid only
 * before its first checksum tile.  Results are bit-identical to the unflagged calls.  Pass
 * the flag to BOTH calls (and to aabft_check / aabft_correct, which ignore it).  Contract:
 * the workspace must be zero-filled once before its first flagged aabft_gemm (the kernel
 * leaves its split-K flag words zero after every launch, so no per-call reset -- which would
 * sit between the two kernels and serialise them -- is needed).  Opt-in: measured SLOWER on
 * B200 -- the encode's FP64 additions share the FP64 datapath with the GEMM's
 * DMMA instructions, which stretches the co-resident encode 7x and costs the GEMM more than
 * the serial encode takes. */
#define AABFT_FLAG_OVERLAP_ENCODE 4
/* AABFT_FLAG_CHECK_CORRECTS: aabft_check also corrects every block it locates as SINGLE, in the
 * same kernel (Alg 2 classifies and corrects per block): the block's report leaves
 * the check as AABFT_BLK_CORRECTED or AABFT_BLK_UNCORRECTABLE (the correction is re-verified
 * exactly as aabft_correct does), the counters include the corrections, and a following
 * aabft_correct finds nothing left to do.  Without the flag aabft_check only classifies and
 * locates (AABFT_BLK_SINGLE) and aabft_correct corrects. */
#define AABFT_FLAG_CHECK_CORRECTS 8

/* Output of aabft_encode.  Acs: (M/bs) x K, ld_acs >= K.  Bcs: K x (N/bs), ld_bcs >= N/bs.
 * topA_val/topA_idx: (M + M/bs) x p -- data rows 0..M-1, then checksum rows; |value|
 *   (as double) in descending order, ties to the lowest index; idx = column k.
 * topB_val/topB_idx: (N + N/bs) x p -- data columns, then checksum columns; idx = row k. */
typedef struct {
  void *Acs;
  int64_t ld_acs;
  void *Bcs;
  int64_t ld_bcs;
  double *topA_val;
  int32_t *topA_idx;
  double *topB_val;
  int32_t *topB_idx;
} aabft_encoded;

/* Output of aabft_gemm.  C: M x N (ldc >= N); Ccol: (M/bs) x N (ld_ccol >= N) carried column
 * checksums c_{m+1,j} per block-row; Crow: M x (N/bs) (ld_crow >= N/bs) carried row
 * checksums c_{i,q+1} per block-column (Eq 3 with partitioned encoding; corner not formed,
 * reading R17).
 * Rcol / Rrow (optional, double, dense (M/bs) x N and M x (N/bs)): when both are non-NULL and
 * the path supports it (FP64 with bs <= 64, FP32 with bs <= 128), aabft_gemm also forms the
 * REFERENCE checksums of Eq 4 (c*_{m+1,j}, c*_{i,q+1}) from its epilogue registers and
 * aabft_check -- which then needs the same workspace -- compares those instead of re-reading C
 * ("fused check"; fault model: DESIGN.md 6.4); after aabft_check Rcol / Rrow hold the
 * complete reference sums.  NULL = unfused: aabft_check re-sums C. */
typedef struct {
  void *C;
  int64_t ldc;
  void *Ccol;
  int64_t ld_ccol;
  void *Crow;
  int64_t ld_crow;
  double *Rcol;
  double *Rrow;
} aabft_product;

/* Per-block (BS x BS sub-matrix of C, "one threadblock for each submatrix of C")
 * report, row-major over blocks: report[I * (N/bs) + J]. */
enum {
  AABFT_BLK_CLEAN = 0,          /* no critical check */
  AABFT_BLK_CORRECTED = 1,      /* one critical row x one critical column, corrected */
  AABFT_BLK_CHECKSUM_ONLY = 2,  /* only row checks or only column checks tripped: the
                                   carried checksum itself is faulty, data untouched */
  AABFT_BLK_UNCORRECTABLE = 3,  /* several rows and columns, or correction did not verify */
  AABFT_BLK_SINGLE = 4          /* located by aabft_check, awaiting aabft_correct */
};
typedef struct {
  uint8_t status;      /* AABFT_BLK_* */
  uint8_t worst_class; /* 0 rounding, 1 tolerable, 2 critical (reading R10) */
  uint16_t n_bad_rows; /* critical row checks in the block */
  uint16_t n_bad_cols; /* critical column checks in the block */
  uint16_t reserved;
  int32_t row, col;    /* global (i, j) of the located element, else -1 */
  float max_ratio;     /* max |d| / eps over the block's 2*bs checks (inf if eps = 0 < |d|) */
} aabft_block_report;  /* 20 bytes */

/* Device-side counters, reducible with a SUM all-reduce (n) and a MAX all-reduce
 * (max_ratio): n = {blocks, clean, corrected, checksum_only, uncorrectable,
 * checks_rounding, checks_tolerable, checks_critical}. */
typedef struct {
  int64_t n[8];
  double max_ratio;
} aabft_counts;

/* Fault descriptor for injection campaigns (Alg 3).
 * (row, col) are C_fc coordinates: row in [M, M + M/bs) hits Ccol row row-M;
 * col in [N, N + N/bs) hits Crow column col-N.
 *  site 0: XOR xor_mask into the stored result ("errorVecAdd2")
 *  site 1: XOR xor_mask into the accumulator ("errorVecAdd1").  FP32 (FFMA):
 *          right after step k_step, instruction-exact.  FP64 (DMMA): after the k-tile
 *          (16 steps) that contains k_step -- products inside the DMMA unit are not
 *          addressable (R23)
 *  site 2: add `add` to the stored result (magnitude sweep)
 *  site 3: add `add` to the accumulator, at the same point as site 1
 *  site 4: FP32 only ("errorVecMul"): at step k_step the product is rounded on
 *          its own, XOR-ed with xor_mask and added (c = c + (fl(a*b) ^ mask)); the FP64
 *          kernel ignores it
 * Capacity: the FP64 kernel applies at most 64 faults per 64 x 64 tile of C / Ccol / Crow, the
 * FP32 kernel at most 256 per 128 x 128 tile (i.e. one per 8 x 8 block); extra faults in the
 * same tile are ignored. */
typedef struct {
  int64_t row, col;
  int32_t site;
  int32_t reserved;
  int64_t k_step;
  uint64_t xor_mask;
  double add;
} aabft_fault; /* 48 bytes */

/* Bytes of device workspace needed by aabft_encode / aabft_gemm / aabft_gemm_plain /
 * aabft_check (one buffer serves all of them; 256-byte aligned; contents need no
 * initialisation -- except under AABFT_FLAG_OVERLAP_ENCODE, see there).  A fused aabft_check
 * must get the workspace of the aabft_gemm that produced its product: that GEMM zeroes the
 * check's counter accumulator (the workspace's last 256 bytes), the check's CTAs add into it
 * and its last CTA moves the totals to *counts and re-arms it.  Returns 0 on an invalid
 * config. */
size_t aabft_workspace_bytes(const aabft_config *cfg);

/* Step 1 (Alg 1).  A (lda >= K) or B (ldb >= N) may be NULL to encode only the
 * other; the corresponding outputs are then untouched.  Checksums are summed sequentially
 * in ascending order in the working precision, so Acs/Bcs, top-p values and hence every
 * bound are bit-identical to the definition (reading R11).
 * topA_val and topA_idx (likewise topB_*) both NULL: checksums only, no top-p selection --
 * the encoding of the fixed-eps and SEA-ABFT comparators (Table I); setting only
 * one of the pair is AABFT_EINVAL. */
aabft_status aabft_encode(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                          int64_t ldb, const aabft_encoded *out, void *ws, size_t ws_bytes,
                          void *stream);

/* Bound of arbitrary elements of C_fc (§IV-E last paragraph: "for each element c_ij of
 * the full-checksum result matrix C_fc, this upper bound gives an expectation value and a
 * variance"): for n DEVICE (row, col) pairs in C_fc coordinates (row >= M: checksum row of A,
 * col >= N: checksum column of B) writes sigma and eps (double, device, n each). */
aabft_status aabft_bound_elements(const aabft_config *cfg, const aabft_encoded *enc,
                                  const int64_t *rows, const int64_t *cols, int64_t n,
                                  double *sig, double *eps, void *stream);

/* Bound alone (§IV-E): eps for every carried checksum element.
 * eps_col: (M/bs) x N dense, eps_row: M x (N/bs) dense (either may be NULL); sig_* likewise.
 * eps = omega * sqrt(F(K)) * y * 2^-t (+ K/3 * 2^-2t * y when fma_model = 0). */
aabft_status aabft_bound(const aabft_config *cfg, const aabft_encoded *enc, double *eps_col,
                         double *sig_col, double *eps_row, double *sig_row, void *stream);

/* Step 2 (Eq 3).  FP64: DMMA (mma.sync .f64) tensor-core tiles fed by TMA;
 * FP32: FFMA SIMT tiles (no TF32: it would change the rounding model, north_star).
 * faults: DEVICE array of nfaults aabft_fault (NULL / 0 = none). */
aabft_status aabft_gemm(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                        int64_t ldb, const aabft_encoded *enc, const aabft_product *out,
                        const aabft_fault *faults, int32_t nfaults, void *ws, size_t ws_bytes,
                        void *stream);

/* Unprotected C = A.B with the same kernel family and scheduler (overhead denominator).
 * ws: device workspace of aabft_gemm_plain_workspace_bytes(cfg) bytes (split-K partial
 * slots and flags only; no checksum, top-p or reference-sum space).  Only cfg's dtype, M, N,
 * K are used (bs and p must still validate). */
size_t aabft_gemm_plain_workspace_bytes(const aabft_config *cfg);
aabft_status aabft_gemm_plain(const aabft_config *cfg, const void *A, int64_t lda,
                              const void *B, int64_t ldb, void *C, int64_t ldc, void *ws,
                              size_t ws_bytes, void *stream);

/* Step 3 (Alg 2; Eq 4-6).  Writes (M/bs)*(N/bs) reports and overwrites *counts
 * (device) with this check's totals (AABFT_FLAG_CHECK_CORRECTS: also corrects SINGLE blocks).  Reference sums are in double (reading R12): unfused (prod->Rcol/Rrow
 * NULL, or FP32, or bs > 64) they re-sum C from memory in sequential ascending order -- the
 * paper's check kernel; fused they are the GEMM epilogue's sums of the registers it
 * stored (fixed shuffle-tree order, parity by tolerance) -- which sees every fault inside the
 * GEMM (Alg 3) but not a corruption of C in memory after the store. */
aabft_status aabft_check(const aabft_config *cfg, const aabft_encoded *enc,
                         const aabft_product *prod, aabft_block_report *reports,
                         aabft_counts *counts, void *ws, size_t ws_bytes, void *stream);

/* Step 4 (reading R15): for every SINGLE block,
 *   C[i][j] <- Ccol[I][j] - sum_{i' in I, i' != i} C[i'][j]   (double, ascending)
 * then re-verify row i; status becomes CORRECTED or UNCORRECTABLE and counts are updated. */
aabft_status aabft_correct(const aabft_config *cfg, const aabft_encoded *enc,
                           const aabft_product *prod, aabft_block_report *reports,
                           aabft_counts *counts, void *stream);

/* ---- NEXT-3 comparators (reporting only; the A-ABFT path above does not use them) ----------
 *
 * SEA-ABFT bound (§III, ref [28]) for every carried checksum:
 *   eps = ((n + 2m - 2) ||b||_2 sum_{i=1..m} ||a_i||_2 + n ||a_{m+1}||_2 ||b||_2) 2^-t
 * with n = K, m = bs: column checksum (I, j) -- a_i the bs rows of block-row I of A, a_{m+1}
 * = Acs[I], b = column j of B; row checksum (i, J) -- the transposed statement (a_i the bs
 * columns of block-column J of B, a_{m+1} = Bcs[:, J], b = row i of A); corner (I, J) --
 * a_{m+1} = Acs[I], b = Bcs[:, J] (reading R25; only for the Table II/III average).  Norms are
 * sequential ascending sums of squares in double (bit-identical to the definition).  Needs
 * A, B and the checksums of aabft_encode (top-p not needed).  eps_col: (M/bs) x N, eps_row:
 * M x (N/bs), eps_corner: (M/bs) x (N/bs), dense doubles, each may be NULL (not all).
 * ws: the aabft_workspace_bytes(cfg) workspace (holds the norms). */
aabft_status aabft_sea_bound(const aabft_config *cfg, const void *A, int64_t lda, const void *B,
                             int64_t ldb, const aabft_encoded *enc, double *eps_col,
                             double *eps_row, double *eps_corner, void *ws, size_t ws_bytes,
                             void *stream);

/* Check (Eq 4-6) and correction against an EXTERNAL eps instead of the A-ABFT bound (reading
 * R26): eps_col ((M/bs) x N) / eps_row (M x (N/bs)) dense device arrays -- e.g. from
 * aabft_sea_bound -- or, where an array is NULL, eps_fixed for every such check ("ABFT with
 * manually set error bounds", Table I).  An external eps carries no sigma: classes
 * are ROUNDING (|d| <= eps) and CRITICAL only.  Verdicts, reports, counts, fused reference
 * sums (prod->Rcol/Rrow + ws) and the correction rule are those of aabft_check /
 * aabft_correct; eps_fixed must be >= 0.  The fused reference sums may be checked any number
 * of times (A-ABFT and comparators over the same product). */
aabft_status aabft_check_ext(const aabft_config *cfg, const aabft_product *prod,
                             const double *eps_col, const double *eps_row, double eps_fixed,
                             aabft_block_report *reports, aabft_counts *counts, void *ws,
                             size_t ws_bytes, void *stream);
aabft_status aabft_correct_ext(const aabft_config *cfg, const aabft_product *prod,
                               const double *eps_row, double eps_fixed,
                               aabft_block_report *reports, aabft_counts *counts, void *stream);

/* Bound-quality study (NEXT-1; §VI-B, Tables II/III): the signed rounding error of
 * every carried checksum, err = carried - exact, where the exact inner product of the checksum
 * vectors (Acs[I] . B[:, j], A[i] . Bcs[:, J]) is formed in double-double on the GPU (Dot2:
 * FMA TwoProd + compensated TwoSum; the paper used GMP on the host).  err_col:
 * (M/bs) x N, err_row: M x (N/bs), dense doubles.  Needs the outputs of aabft_encode and
 * aabft_gemm.  A diagnostic, not part of the protected path. */
aabft_status aabft_checksum_errors(const aabft_config *cfg, const void *A, int64_t lda,
                                   const void *B, int64_t ldb, const aabft_encoded *enc,
                                   const aabft_product *prod, double *err_col, double *err_row,
                                   void *stream);

/* All four steps on HOST buffers (end-to-end entry point): copies A_host (M x K, dense) and
 * B_host (K x N, dense) into `arena` (device, >= aabft_host_arena_bytes), runs encode, gemm,
 * check, correct, and copies C (M x N dense) into C_host and the counts into counts_host.
 * Host buffers should be pinned for full PCIe bandwidth.  Synchronises `stream`. */
size_t aabft_host_arena_bytes(const aabft_config *cfg);
aabft_status aabft_protected_gemm_host(const aabft_config *cfg, const void *A_host,
                                       const void *B_host, void *C_host,
                                       aabft_counts *counts_host, void *arena,
                                       size_t arena_bytes, void *stream);

const char *aabft_status_str(aabft_status s);
/* Thread-local detail for the last non-OK return on this thread. */
const char *aabft_last_error(void);
/* Library version string and the number of kernel launches this thread has enqueued
 * through the library since load (used by bench.py's gpu_launches). */
const char *aabft_version(void);
int64_t aabft_launch_count(void);

#ifdef __cplusplus
}
#endif
#endif /* AABFT_H */
