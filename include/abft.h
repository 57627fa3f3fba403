/*
 * abft.h — C ABI of the B200-native two-dimensional weighted-checksum ABFT
 * hot path (Chen et al., "Fault Tolerant One-sided Matrix Decompositions on
 * Heterogeneous Systems with GPUs", SC'18).  Citations "L<n>" are lines of the
 * paper text plus the section they fall in; "c-<k>" are the
 * readings of ambiguous passages listed in DESIGN.md §4.
 *
 * Conventions (all entry points)
 *  - Matrices and checksum arrays are COLUMN-MAJOR (LAPACK/MAGMA, L536).
 *  - Every matrix / checksum / report pointer is a DEVICE pointer unless the
 *    argument says "host".  The caller owns every buffer (allocated through
 *    torch in the Python binding); the library only borrows them for the
 *    duration of the stream-ordered work.  The library owns only internal
 *    workspace (per stream), cuBLAS/cuSOLVER handles and the ft_ctx_t.
 *  - Calls are asynchronous on `stream` (a cudaStream_t; NULL = legacy
 *    default stream) and never synchronise the host, except where stated.
 *  - Return value: 0 on success; -i when argument i (1-based) is illegal
 *    (LAPACK xerbla style); a positive ABFT_E_* code on a runtime failure.
 *    Numerical outcomes (flags, fixes, LAPACK info) are written to device
 *    memory, never returned.
 *  - v1 tiles: m and n must be multiples of nb (c-22); nb must be a power of
 *    two in [32, 1024].
 *  - Tile (I, J) (0-based) is rows [I*nb, (I+1)*nb) x cols [J*nb, (J+1)*nb).
 */
#ifndef ABFT_H
#define ABFT_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define ABFT_API __attribute__((visibility("default")))
#else
#define ABFT_API
#endif

typedef struct CUstream_st *abft_stream_t; /* == cudaStream_t */

/* ---------------------------------------------------------------- enums -- */
enum { ABFT_F32 = 0, ABFT_F64 = 1 };

/* Views of a diagonal tile (c-3; off-diagonal tiles are always GENERAL).
 * GENERAL: stored block.  LOWER: upper part read as 0 (factored L_kk).
 * UNIT_LOWER: strictly-lower part + implicit unit diagonal (LU's L_kk, QR's V).
 * UPPER: lower part read as 0 (LU's U_kk, QR's R).
 * SYM_LOWER: symmetric block mirrored from the stored lower triangle,
 *   X[i][j] = A[max(i,j)][min(i,j)] (Cholesky input diagonal tiles; the
 *   maintained row checksum is then the transposed column checksum, L189). */
enum { ABFT_GENERAL = 0, ABFT_LOWER = 1, ABFT_UNIT_LOWER = 2, ABFT_UPPER = 3, ABFT_SYM_LOWER = 4 };

/* Which checksums a call encodes / checks (c-9: trailing tiles carry both,
 * column panels only c, row panels only r, L139). */
enum { ABFT_COL = 1, ABFT_ROW = 2, ABFT_BOTH = 3 };

/* Threshold kinds (c-6).  MAGNITUDE: tau_e = scale*2*gamma_nb*m where m is the
 * maintained magnitude checksum (colmag/rowmag of abft_mat_t) when present,
 * else e^T|X| of the current tile.  POSTERIORI: always e^T|X|.  In both,
 * tau_w = nb*tau_e, gamma_nb = nb*u/(1-nb*u) (L133), u = 2^-53 / 2^-24. */
enum { ABFT_TOL_MAGNITUDE = 0, ABFT_TOL_POSTERIORI = 1 };

/* Per-tile status bits (abft_report_t.status). */
enum { ABFT_ST_COL = 1, ABFT_ST_ROW = 2, ABFT_ST_NONFINITE = 4, ABFT_ST_UNCORRECTABLE = 8 };

/* Classes (c-11; L122, L145, L330-L334, L432-L434). */
enum {
  ABFT_CLS_CLEAN = 0, ABFT_CLS_0D = 1, ABFT_CLS_1D_ROW = 2, ABFT_CLS_1D_COL = 3,
  ABFT_CLS_SYM_CROSS = 4, ABFT_CLS_CHK_CORRUPT = 5, ABFT_CLS_STALE_R = 6,
  ABFT_CLS_STALE_C = 7, ABFT_CLS_2D = 8
};
/* Fix-record kinds. */
enum { ABFT_FIX_DATA = 0, ABFT_FIX_COLCHK = 1, ABFT_FIX_ROWCHK = 2 };

/* counts[] slots of abft_report_t (device int32[8], accumulated). */
enum {
  ABFT_CNT_TILES_FLAGGED = 0, ABFT_CNT_COLS_FLAGGED = 1, ABFT_CNT_ROWS_FLAGGED = 2,
  ABFT_CNT_NONFINITE = 3, ABFT_CNT_TILES_FIXED = 4, ABFT_CNT_ELEMS_FIXED = 5,
  ABFT_CNT_CHK_REPAIRED = 6, ABFT_CNT_UNCORRECTABLE = 7, ABFT_NCOUNTS = 8
};

/* Error codes (positive). */
enum {
  ABFT_OK = 0, ABFT_E_CUDA = 1, ABFT_E_CUBLAS = 2, ABFT_E_CUSOLVER = 3,
  ABFT_E_NOMEM = 4, ABFT_E_UNCORRECTABLE = 5, ABFT_E_UNSUPPORTED = 6, ABFT_E_NCCL = 7
};

/* ---------------------------------------------------------------- types -- */
/* A matrix and its maintained 2D checksum state (L108-L112, L531).
 *   A       m x n,            lda  >= m
 *   colchk  (2*m/nb) x n,     ldc  >= 2*m/nb : rows 2I (e) and 2I+1 (w) hold
 *           c(X) = [v1 v2]^T X of every tile (I, J) for its nb columns
 *   rowchk  m x (2*n/nb),     ldr  >= m      : cols 2J (e) and 2J+1 (w) hold
 *           r(X) = X [v1 v2]
 *   colmag  (m/nb) x n,       ldcm >= m/nb   : running e^T|X| per tile column (c-6), nullable
 *   rowmag  m x (n/nb),       ldrm >= m      : running |X| e per tile row (c-6), nullable
 * v1 = (1,...,1), v2 = (1,2,...,nb), tile-local and 1-based (L108, c-2).
 * Elements are fp32 or fp64 per `dtype`, all arrays the same type. */
typedef struct {
  int32_t dtype;
  int64_t m, n, nb;
  void *A;      int64_t lda;
  void *colchk; int64_t ldc;
  void *rowchk; int64_t ldr;
  void *colmag; int64_t ldcm;
  void *rowmag; int64_t ldrm;
} abft_mat_t;

/* Half-open tile ranges [I0,I1) x [J0,J1); lower_only keeps I >= J
 * (Cholesky, L464); diag_view applies to tiles with I == J. */
typedef struct {
  int32_t I0, I1, J0, J1;
  int32_t lower_only;
  int32_t diag_view;
} abft_tiles_t;

typedef struct {
  int32_t kind;    /* ABFT_TOL_* */
  double scale;    /* multiplies tau (default 1) */
  int32_t refresh; /* abft_verify: rebase every UNFLAGGED checksum entry of a checked tile on the
                      recomputed value and reset its magnitude to e^T|X| (c-6); flagged entries are
                      left for abft_locate_correct.  Keeps the magnitude bound from compounding
                      |T^-1| factors across iterations (LU/QR). */
} abft_tol_t;

/* Verification output.  status: device int32, (m/nb) x (n/nb) column-major,
 * ld_status >= m/nb; written for every tile of the range (0 = clean).
 * dcol/drow: optional device arrays with the shape and leading dimension of
 * colchk/rowchk; receive delta = maintained - recomputed (L119) for every
 * checked tile.  counts: device int32[ABFT_NCOUNTS], atomically accumulated
 * (zero it before a campaign). */
typedef struct {
  int32_t *status; int64_t ld_status;
  void *dcol; void *drow;
  int32_t *counts;
} abft_report_t;

/* One correction (device array of these).  kind DATA: element (gi, gj) of A
 * changed from `before` to `after`.  kind COLCHK: colchk e-entry of tile row
 * gi, column gj re-encoded.  kind ROWCHK: rowchk e-entry of row gi, tile
 * column gj re-encoded.  cls = ABFT_CLS_* that produced it. */
typedef struct {
  int64_t gi, gj;
  double before, after;
  int32_t cls, kind;
} abft_fix_t;

/* ------------------------------------------------------ hot path (a1-a3) -- */

/* a1 — abft_encode.  For every selected tile X (view per tiles->diag_view on
 * I == J) write c(X) = [v1 v2]^T X into colchk and/or r(X) = X [v1 v2] into
 * rowchk (`which`), and, when colmag/rowmag are non-NULL, the magnitude sums
 * e^T|X| / |X|e.  One fused HBM pass reads each tile once (L442-L454,
 * §VIII; 6 flops per element, L446/L461).  Deterministic: the same tile
 * always produces bit-identical checksums, so abft_verify right after
 * abft_encode reports delta == 0 exactly. */
ABFT_API int abft_encode(const abft_mat_t *mat, const abft_tiles_t *tiles, int32_t which,
                abft_stream_t stream);

/* a2 — abft_verify.  Recompute the checksums of every selected tile
 * (recal_c / recal_r, L116), delta = maintained - recomputed (L119), flag a
 * column j when |delta_e[j]| > tau_e[j] or |delta_w[j]| > tau_w[j] or either
 * is non-finite (L122, c-6, c-7); rows likewise.  Writes report->status for
 * every tile, optional deltas, and accumulates report->counts[0..3].  Same
 * single pass as abft_encode (the paper reuses its encoder for every check,
 * L442). */
ABFT_API int abft_verify(const abft_mat_t *mat, const abft_tiles_t *tiles, int32_t which,
                const abft_tol_t *tol, const abft_report_t *report, abft_stream_t stream);

/* Prior-art baseline (row f3; L35, L442): abft_verify with the checksums
 * recomputed as matrix products c = [v1 v2]^T X, r = X [v1 v2] by cuBLAS
 * (strided-batched GEMMs per tile column; masked diagonal views materialized
 * first), then the same test and report as abft_verify.  Needs the
 * magnitude arrays of every checked direction (ABFT_E_UNSUPPORTED
 * otherwise: a product cannot form e^T|X|); tol->refresh is ignored.  Exists
 * to measure what the fused single-pass kernel buys (the paper's L657). */
ABFT_API int abft_verify_gemm(const abft_mat_t *mat, const abft_tiles_t *tiles, int32_t which,
                const abft_tol_t *tol, const abft_report_t *report, abft_stream_t stream);

/* a3 — abft_locate_correct.  For every tile of the range whose
 * report->status has COL or ROW set: up to 3 rounds of recompute ->
 * classify (c-11: CHK_CORRUPT, STALE_R/C, 0D, 1D_ROW, 1D_COL, SYM_LOWER
 * mirrored pair, SYM_CROSS, else 2D) -> correct in place.  Location:
 * i = rint(delta_w/delta_e) - 1 with the acceptance test of c-5 (L122),
 * fallback c-7 for non-finite residuals; correction
 * x_ij <- c_e[j] - sum_{r != i} X[r][j] (c-4).  Rewrites status (0 = clean,
 * ABFT_ST_UNCORRECTABLE = 2D, L434), accumulates counts[4..7], appends fix
 * records to `fixes` (device, capacity max_fixes; *n_fixes is a device
 * counter the caller zeroes; records beyond capacity are counted, not
 * stored).  Tiles with status 0 cost one status read, so the call can be
 * issued unconditionally after every verify (no host sync). */
ABFT_API int abft_locate_correct(const abft_mat_t *mat, const abft_tiles_t *tiles, int32_t which,
                        const abft_tol_t *tol, const abft_report_t *report,
                        abft_fix_t *fixes, int32_t max_fixes, int32_t *n_fixes,
                        abft_stream_t stream);

/* a2 + a3 fused — abft_check.  abft_verify followed by abft_locate_correct
 * on the same range, arguments and outcomes as the two calls in sequence
 * (status, counts, corrections and fix records equal), in ONE launch: the
 * CTA that finishes a tile's verify and finds it flagged runs the locate /
 * classify / correct rounds of that tile itself (a check of Alg. 2,
 * without a separate locate launch).  Where the locate tables do not fit the
 * pass kernel's shared memory (fp64 nb=1024) the library issues the two
 * launches instead.  Errors as abft_verify / abft_locate_correct. */
ABFT_API int abft_check(const abft_mat_t *mat, const abft_tiles_t *tiles, int32_t which,
                const abft_tol_t *tol, const abft_report_t *report,
                abft_fix_t *fixes, int32_t max_fixes, int32_t *n_fixes, abft_stream_t stream);

/* Fault injection (paper §X.A): element[offset] ^= xor_mask on the
 * device (fp32 uses the low 32 bits of the mask). */
ABFT_API int abft_inject(void *ptr, int32_t dtype, int64_t offset, uint64_t xor_mask, abft_stream_t stream);

/* Sizes (elements) of the checksum and magnitude arrays for an m x n matrix
 * with tile nb at minimal leading dimensions (space overhead 4/nb, L531,
 * plus 2/nb for magnitudes).  Host pointers; any may be NULL. */
ABFT_API int abft_sizes(int64_t m, int64_t n, int64_t nb, int64_t *colchk_elems, int64_t *rowchk_elems,
               int64_t *colmag_elems, int64_t *rowmag_elems);

/* ------------------------------------------------ update rules (a4-a6) -- */

/* a5 — abft_update_trsm (PU, L139-L143, Table II).
 * side 'R': X = B * op(T)^-1  =>  chk (nvec x nb) <- chk * op(T)^-1 and, when
 *           mag != NULL, mag (nmag x nb) <- mag * |op(T)^-1| (c-6).
 * side 'L': X = op(T)^-1 * B  =>  chk (nb x nvec) <- op(T)^-1 * chk and
 *           mag (nb x nmag) <- |op(T)^-1| * mag.
 * uplo 'L'/'U', trans 'N'/'T', diag 'N'/'U' describe T (nb x nb, ldt) as in
 * BLAS trsm.  Column checksums of a column panel are stacked as 2 rows per
 * tile, so nvec = 2*(#tiles); nmag = #tiles. */
ABFT_API int abft_update_trsm(int32_t dtype, char side, char uplo, char trans, char diag, int64_t nb,
                     const void *T, int64_t ldt, void *chk, int64_t ldchk, int64_t nvec,
                     void *mag, int64_t ldmag, int64_t nmag, abft_stream_t stream);

/* a6 — abft_update_gemm (TMU, L124-L131, L189, L191-L222).
 * which COL: Cchk (M2 x N) += alpha * op(Xchk) (M2 x K) * op(Y) (K x N)
 *            Cmag (M2/2 x N) += |alpha| * op(Xmag) (M2/2 x K) * |op(Y)|
 * which ROW: Cchk (N x M2) += alpha * op(Y) (N x K) * op(Xchk) (K x M2)
 *            Cmag (N x M2/2) += |alpha| * |op(Y)| * op(Xmag) (K x M2/2)
 * transX / transY 'N'/'T' select op().  Cholesky's TMU c(A_ij) -= c(L_ik)
 * L_jk^T is which=COL, transX='N', transY='T' (Y = the panel L21); its
 * r(A_ij) -= L_ik c(L_jk)^T is which=ROW, transX='T' (Xchk = the panel's
 * column checksums, i.e. "transposing the column checksum of the column
 * panel", L189), transY='N'.  LU: c(A) -= c(L) U, r(A) -= L r(U) (c-13).
 * Mags nullable (both or neither); |op(Y)| is materialised in library
 * scratch. */
ABFT_API int abft_update_gemm(int32_t dtype, int32_t which, char transX, char transY, double alpha,
                     const void *Xchk, int64_t ldx, const void *Y, int64_t ldy,
                     void *Cchk, int64_t ldcc, int64_t M2, int64_t N, int64_t K,
                     const void *Xmag, int64_t ldxm, void *Cmag, int64_t ldcm,
                     abft_stream_t stream);

/* a4 — abft_panel_potrf (PD of Cholesky, Table II, c-12).  `diag` is ONE
 * nb x nb tile (m = n = nb) whose colchk holds c_sym(A_kk) (SYM_LOWER view)
 * and colmag its magnitudes.  Computes L_kk = chol(A_kk) in place (lower;
 * cuSOLVER on the device), L_kk^-1 (into Linv, device nb x nb with leading
 * dimension ldw, when non-NULL — the driver reuses it for the PU), then
 * c(L_kk) = c_sym(A_kk) * L_kk^-T and m_c(L_kk) = m_c * |L_kk^-T|.  colchk
 * may be NULL (plain PD).  LAPACK info (0, or k > 0 if the leading minor k is
 * not positive definite) goes to *info (device int32). */
ABFT_API int abft_panel_potrf(const abft_mat_t *diag, void *Linv, int64_t ldw, int32_t *info,
                              abft_stream_t stream);

/* a4 — abft_panel_getrf (PD of LU with partial pivoting for iteration k of
 * the square matrix `mat`; [13] via L135-L145, c-13, c-14).  In order:
 * cuSOLVER dgetrf of the column panel A[k*nb:, k*nb:(k+1)*nb] (pivots to
 * ipiv[0..nb), 1-based global, LAPACK convention); when mat carries
 * checksums: the pre-swap row check (c-14b) of every trailing row the pivots
 * move (row checksums of tile columns > k; flagged tiles are classified and
 * corrected by abft_locate_correct with `tol`, `rep`, `fixes`); the row swaps
 * of all columns outside the panel (LAPACK laswp) with the column-checksum
 * deltas of c-14 (panel columns from the pre-PD copy, L430), row checksums
 * and magnitudes moved with their rows; then L_kk^-1 -> Linv, U_kk^-1 -> Uinv
 * (nb x nb, ld nb, device) and c(L_I) = c(P~_I) U_kk^-1 (I >= k),
 * r(U_kk) = L_kk^-1 r(P~_kk), magnitudes by the absolute inverses (c-6).
 * mat->colchk == NULL gives the plain PD (getrf + swaps + inverses).
 * LAPACK info (U(i,i) == 0) goes to *info (device int32). */
ABFT_API int abft_panel_getrf(const abft_mat_t *mat, int32_t k, int64_t *ipiv, const abft_tol_t *tol,
                              const abft_report_t *rep, abft_fix_t *fixes, int32_t max_fixes,
                              int32_t *n_fixes, void *Linv, void *Uinv, int32_t *info,
                              abft_stream_t stream);

/* a4 — abft_panel_geqrf (PD of Householder QR for iteration k; Table III,
 * Alg. 1, c-15).  cuSOLVER dgeqrf of the column panel (LAPACK
 * storage: R on and above the diagonal, v(2:) below, tau[0..nb)), the unit
 * lower trapezoidal V into V (device, (n-k*nb) x nb, ld n-k*nb), the
 * triangular factor T of the compact WY form (CTF, L238; not protected, c-16)
 * into T (nb x nb, ld nb); when mat carries checksums (panel_copy: device
 * (n-k*nb) x nb scratch for the pre-PD panel): c(V) per panel tile by the
 * Alg. 1 recurrences replayed on the checksum rows, r(R) = rows of Q^T r(P),
 * magnitudes by c-6.  *info (device int32) from dgeqrf. */
ABFT_API int abft_panel_geqrf(const abft_mat_t *mat, int32_t k, void *tau, void *V, void *T,
                              void *panel_copy, int32_t *info, abft_stream_t stream);

/* W = T^-1 for an nb x nb triangular T (uplo 'L'/'U', diag 'N'/'U'); the
 * other triangle of W is written as zero.  Helper of the a5 rule (the
 * magnitude propagation needs |T^-1| explicitly, c-6). */
ABFT_API int abft_tri_inverse(int32_t dtype, char uplo, char diag, int64_t nb, const void *T, int64_t ldt,
                              void *W, int64_t ldw, abft_stream_t stream);

/* a5 with a precomputed inverse W = T^-1 (as abft_update_trsm, without the
 * triangular solve): side 'R': chk (nvec x nb) <- chk * op(W),
 * mag (nmag x nb) <- mag * |op(W)|; side 'L': chk (nb x nvec) <- op(W) * chk,
 * mag (nb x nmag) <- |op(W)| * mag.  Skinny DGEMMs, results copied back. */
ABFT_API int abft_update_trsm_inv(int32_t dtype, char side, char trans, int64_t nb, const void *W,
                                  int64_t ldw, void *chk, int64_t ldchk, int64_t nvec, void *mag,
                                  int64_t ldmag, int64_t nmag, abft_stream_t stream);

/* a6 for the symmetric (Cholesky) TMU A22 -= L21 L21^T over ntk trailing tile
 * rows/columns (L189, c-12): with P = c(L21) L21^T (one 2ntk x ntk*nb DGEMM),
 *   c(A_IJ) -= P[2I.., cols of J]          for I >= J  (Cc: colchk block at
 *              tile row k+1, column (k+1)nb; leading dimension ldc)
 *   r(A_IJ) -= P[2J.., cols of I]^T        for I >= J  (Rr: rowchk block, ldr)
 * and, when mL != NULL, with Q = m_c(L21) |L21|^T: Cm += Q (lower tiles),
 * Rm += Q^T (c-6).  L21: ntk*nb x nb (ldl); cL: 2ntk x nb panel column
 * checksums (ld ldc, the colchk leading dimension); mL: ntk x nb (ldcm).
 * Rr == NULL (with Rm == NULL): column rule only (the single-side checking
 * schemes of ft_opts_t.scheme). */
ABFT_API int abft_update_syrk(int32_t dtype, int64_t nb, int64_t ntk, const void *L21, int64_t ldl,
                              const void *cL, int64_t ldc, const void *mL, int64_t ldcm, void *Cc,
                              void *Rr, int64_t ldr, void *Cm, void *Rm, int64_t ldrm, abft_stream_t stream);

/* ----------------------------------------------------- drivers (a7) -- */
typedef struct ft_ctx ft_ctx_t;

/* Fault-injection hooks of the drivers (paper §X.A).
 * point: where in Alg. 2 iteration `iter` the flip is applied (FT_AT_*).
 * kind:  FT_KIND_PERSIST (computation / DRAM / communication: the flipped
 *        value stays) or FT_KIND_ONCHIP (flipped before the op that follows
 *        `point` and restored right after it, before any check).
 * target: 0 = A, 1 = colchk, 2 = rowchk, 3 = the CTF T of ft_geqrf (nb x nb,
 *         local (gi, gj); points FT_AT_POST_PD / FT_AT_PRE_TMU of iterations
 *         k < n/nb - 1); (gi, gj) element of that array. */
enum {
  FT_AT_PRE_PD_CHECK = 0, FT_AT_PRE_PD = 1, FT_AT_POST_PD = 2, FT_AT_PRE_PU_CHECK = 3,
  FT_AT_PRE_PU = 4, FT_AT_POST_PU = 5, FT_AT_PRE_TMU = 6, FT_AT_POST_TMU = 7,
  /* pd_location = FT_PD_HOST only (Alg. 2 lines 3 and 6): a flip in the host
   * copy right after the device-to-host transfer of iteration iter's panel,
   * or in the device panel right after the host-to-device transfer of the
   * factored panel (target must be 0 = A; first trip of the iteration only) */
  FT_AT_D2H = 8, FT_AT_H2D = 9
};
/* Where the panel decomposition runs (ft_opts_t.pd_location). */
enum { FT_PD_DEVICE = 0, FT_PD_HOST = 1 };
enum { FT_KIND_PERSIST = 0, FT_KIND_ONCHIP = 1 };
typedef struct {
  int32_t iter, point, kind, target;
  int64_t gi, gj;
  uint64_t xor_mask;
} ft_inject_t;

typedef struct {
  int64_t nb;            /* tile size (power of two, 32..1024) */
  int32_t abft;          /* 0: unprotected blocked driver (the overhead baseline) */
  int32_t tol_kind;      /* ABFT_TOL_* */
  double tol_scale;
  int32_t fig4a_repair;  /* 1: guarded Fig. 4a trailing repair after the panel re-check (c-25) */
  int32_t n_inject;      /* fault plan (host array) */
  const ft_inject_t *inject;
  abft_fix_t *fix_log;   /* optional device log of every fix (capacity fix_log_cap) */
  int32_t fix_log_cap;
  int32_t pu_gemm;       /* 1: PU as L21 = A21 * L_kk^-T (DGEMM with the PD's explicit inverse) in
                            both the protected and the unprotected driver; 0: cuBLAS DTRSM */
  int32_t refresh;       /* abft_tol_t.refresh for every check of the run (default 1) */
  int32_t restart;       /* 1: local restart (L430): copy the PD / PU input with its checksums after the
                            pre-op check; a 2D error left by the post-op check restores the copy and
                            redoes the op once (one 8-byte read-back per check; ft_potrf) */
  int32_t pd_location;   /* FT_PD_DEVICE (default): PD by cuSOLVER on the device.  FT_PD_HOST: Alg. 2
                            lines 3-7 as the paper runs them (L364-L372, L61): the panel (Cholesky:
                            A_kk; LU/QR: the m_k x nb column panel) goes to pinned host memory, is
                            factored there by the host LAPACK set with ft_ctx_set_host_lapack, and
                            comes back; with abft, both transfers carry a fresh column-checksum
                            guard (reading c-28): the host checks what it received (locate/correct,
                            else re-transfer), the device verifies + corrects the factored panel
                            (abft_verify / abft_locate_correct; uncorrectable -> re-send), then the
                            PD checksum rule and the post-PD check run on the device as usual.
                            The host waits for the device once per iteration. */
  int32_t fig4b;         /* 1 (default): Fig. 4b on-chip 1D detection (L359, f1) — when a pre-PD / pre-PU
                            check of iteration k corrected a 1D pattern (class 1D_ROW / 1D_COL: several
                            errors in one row / column of a block, the trace of an on-chip fault in the
                            previous TMU), the whole trailing matrix is checked right away (ft_potrf,
                            ft_getrf; ft_geqrf checks all of A2 before every TMU anyway).  Decided on the
                            device: without such a fix the check's kernels exit at once. */
  int32_t trailing_check_period; /* P > 0: check the whole trailing matrix after the TMU of every P-th
                            iteration (L359: "periodically check the correctness of trailing matrix
                            ... to avoid 2D propagation"); 0 (default): never */
  int32_t checksum_gemm; /* 1: every check of ft_potrf recomputes the checksums with abft_verify_gemm
                            (the prior-art GEMM-based recalculation, L442) instead of the fused pass;
                            no refresh, no Fig. 4b check.  For the paper's comparison "with / without
                            the optimized checksum kernel" (L653-L657).  Default 0. */
  int32_t scheme;        /* FT_SCHEME_* (ft_potrf only; ft_getrf / ft_geqrf return -7 for anything but
                            FT_SCHEME_NEW): the checking scheme, for the paper's comparison of
                            schemes (L35, L47, L542, Table VIII, Figs. 12-14; reading c-34) */
  int32_t timing;        /* 1: per-phase device time (CUDA events on the stream each phase runs on) into
                            ft_stats_t.ms_phase; costs two event records per timed span.  Default 0. */
  int32_t lookahead;     /* 1 = the TMU of iteration k updates tile column k+1 first (and re-checks the
                            panel(s), Fig. 4a), then iteration k+1's panel work runs on a second stream
                            next to the rest of the TMU (reading c-35): ft_potrf (FT_SCHEME_NEW or
                            abft = 0) its checks, PD and PU; ft_getrf its checks and the factorization
                            of the column panel (the swaps outside it and the PU follow the TMU).  Off
                            for an iteration whose fault hooks it would move.  Ignored by ft_geqrf.
                            Default 0 (bindings: 1). */
} ft_opts_t;

/* ft_opts_t.scheme (reading c-34).  NEW: the paper's scheme, Alg. 2 (full
 * checksums, pre-op checks of PD / PU inputs, post-op checks of their outputs,
 * the Fig. 4a heuristic TMU check).  FULL_POST: full checksums [13], every
 * op's output checked after it (L_kk, the panel, the whole trailing matrix
 * after each TMU).  SINGLE_POST: column checksums only [51, 52], the same
 * post-op checks on c.  SINGLE_PRE: column checksums only [11], every op's
 * input checked before it (A_kk, the panel, panel + trailing matrix before
 * each TMU).  Single-side schemes neither maintain nor check row checksums.
 * Local restart (restart=1) applies where a post-op check exists. */
enum { FT_SCHEME_NEW = 0, FT_SCHEME_FULL_POST = 1, FT_SCHEME_SINGLE_POST = 2, FT_SCHEME_SINGLE_PRE = 3 };

/* Host-side statistics, filled after the driver's final synchronisation. */
typedef struct {
  int32_t counts[ABFT_NCOUNTS]; /* summed over every check of the run */
  int32_t n_fixes;              /* total fix records (may exceed fix_log_cap) */
  int32_t repairs_applied;      /* Fig. 4a trailing repairs (c-25) */
  int32_t repairs_skipped;      /* guarded-out repairs (|E| too large) */
  int32_t uncorrectable;        /* tiles left 2D (-> ABFT_E_UNCORRECTABLE) */
  int32_t n_checks;             /* verify calls issued */
  double ms_total;
  int32_t restarts;             /* local restarts performed (f1) */
  /* FT_PD_HOST transfer guard (reading c-28) */
  int32_t xfer_d2h_flagged;     /* host check: columns whose guard residual was flagged */
  int32_t xfer_d2h_fixed;       /* host check: elements corrected */
  int32_t xfer_retransfers;     /* device-to-host transfers repeated */
  int32_t xfer_h2d_flagged;     /* device check: flagged columns */
  int32_t xfer_h2d_fixed;       /* device check: elements corrected (also in the fix log) */
  int32_t xfer_resends;         /* host-to-device transfers repeated */
  int32_t xfer_uncorrectable;   /* transfers still wrong after 2 repeats (-> uncorrectable) */
  double ms_host_pd;            /* wall time of the host round trips (transfers + host PD) */
  /* ft_geqrf CTF check (row f2, L263; reading c-29) */
  int32_t ctf_flagged;          /* checks whose E = T^T V^T V T - T - T^T exceeded the bound */
  int32_t ctf_recomputed;       /* T recomputed from V after a flagged check */
  /* outcomes by class, from the fix log of the run */
  int32_t detected;             /* tiles a check flagged (= counts[ABFT_CNT_TILES_FLAGGED]) */
  int32_t corrected_0d;         /* data elements fixed as 0D errors (L330) */
  int32_t corrected_1d;         /* data elements fixed as part of a 1D pattern (1D_ROW, 1D_COL, SYM_CROSS) */
  int32_t checksum_repaired;    /* checksum entries re-encoded (CHK_CORRUPT, STALE_R, STALE_C) */
  int32_t comm_errors;          /* transfer-guard corrections and repeats (FT_PD_HOST, Alg. 2 lines 3-7) */
  /* opts->timing: device ms per phase (FT_PH_*), summed over the run; the
     phases of the look-ahead side stream overlap the main stream's */
  double ms_phase[8];
} ft_stats_t;
/* ft_stats_t.ms_phase indices */
enum { FT_PH_PD = 0, FT_PH_PU = 1, FT_PH_TMU = 2, FT_PH_RULES = 3, FT_PH_CHECKS = 4, FT_PH_RESTART = 5,
       FT_PH_ENCODE = 6, FT_PH_OTHER = 7, FT_NPHASE = 8 };

/* A driver context on `device`; the ft_* drivers are ordered on `stream`
 * (any stream, the legacy default one included): internally they run on a
 * private non-blocking stream of the context that waits for `stream` at entry
 * and that `stream` waits for at exit (so the optional device-decided restart
 * below can capture its redo into a CUDA graph).  Owned by the caller; free
 * with ft_ctx_destroy. */
ABFT_API int ft_ctx_create(ft_ctx_t **ctx, int32_t device, abft_stream_t stream);
ABFT_API int ft_ctx_destroy(ft_ctx_t *ctx);

/* Host LAPACK for pd_location = FT_PD_HOST: `path` is a shared library with
 * the LP64 (int32) Fortran LAPACK symbols dpotrf_/spotrf_, dgetrf_/sgetrf_,
 * dgeqrf_/sgeqrf_, plain or with the "scipy_" prefix (the OpenBLAS bundled with
 * SciPy).  Host pointer; the library is dlopen'ed and kept until
 * ft_ctx_destroy.  Returns ABFT_E_UNSUPPORTED when it cannot be loaded or a
 * symbol is missing. */
ABFT_API int ft_ctx_set_host_lapack(ft_ctx_t *ctx, const char *path);

/* ft_potrf — fault-tolerant lower Cholesky A = L L^T of the n x n SPD matrix
 * dA (device, lda >= n, n % nb == 0), right-looking blocked, Alg. 2 order
 * (L364-L379): per iteration k — check A_kk (SYM_LOWER, both) -> PD + c-12
 * -> check L_kk (LOWER, c) -> check panel A_ik (both) -> PU + a5 -> check
 * L_ik (c) -> TMU (DSYRK on tensor cores) + a6 -> heuristic re-check of L_ik
 * (Fig. 4a) with the guarded trailing repair (c-25).  Checksums are
 * allocated inside ctx.  Synchronises the host once at the end, plus, when
 * opts->restart, one wait per iteration for the post-PD local-restart
 * decision (f1, L430); the post-PU restart is decided on the device (its
 * redo is queued as gated kernels that run only after a 2D error, DESIGN.md
 * §2.10).  Returns ABFT_E_UNCORRECTABLE if a 2D error remained after the
 * restart (or without it).  *info (host) follows LAPACK potrf. */
ABFT_API int ft_potrf(ft_ctx_t *ctx, int32_t dtype, int64_t n, void *dA, int64_t lda,
             const ft_opts_t *opts, ft_stats_t *stats, int64_t *info);

/* ft_getrf — fault-tolerant LU with partial pivoting, PA = LU, of the square
 * n x n matrix dA (device, lda >= n, n % nb == 0), right-looking blocked,
 * full checksums on the trailing matrix ([13], L135-L145), Alg. 2 order per
 * iteration k: check the column panel (c+r) -> abft_panel_getrf (pre-swap row
 * check, swaps, c(L), r(U_kk)) -> check L (UNIT_LOWER, c) and U_kk (UPPER, r)
 * -> check the row panel (c+r) -> PU U12 = L_kk^-1 A12 + r(U12) -> check U12
 * (r) -> TMU DGEMM + c/r rules -> re-check both panels (Fig. 4a) with the
 * guarded repair (c-25).  ipiv: device int64[n], 1-based global pivots.
 * Returns ABFT_E_UNCORRECTABLE if a 2D error remained.  *info (host) follows
 * LAPACK getrf. */
ABFT_API int ft_getrf(ft_ctx_t *ctx, int32_t dtype, int64_t n, void *dA, int64_t lda, int64_t *ipiv,
                      const ft_opts_t *opts, ft_stats_t *stats, int64_t *info);

/* ft_geqrf — fault-tolerant Householder QR A = QR of the square n x n dA
 * (device, lda >= n, n % nb == 0) with full checksums (Table III): per
 * iteration k — check the column panel (c+r) -> abft_panel_geqrf -> check V
 * (UNIT_LOWER, c) and R_kk (UPPER, r) -> TMU A2 <- Q^T A2 (three DGEMMs) with
 * c(A2) -= c(V) W, r(A2) -= V T^T V^T r(A2), preceded by the check of A2
 * (c+r, c-25q) and the CTF check of T (f2, L263: E = T^T V^T V T - T - T^T
 * against the c-29 bound, recompute T from V when flagged; one host
 * read-back per iteration) -> re-check V (a V correction
 * after the TMU consumed it is outcome R) and R12 (r).  Output as LAPACK
 * dgeqrf (R and V in dA, tau: device array of n).  Returns
 * ABFT_E_UNCORRECTABLE if a 2D / consumed error remained. */
ABFT_API int ft_geqrf(ft_ctx_t *ctx, int32_t dtype, int64_t n, void *dA, int64_t lda, void *tau,
                      const ft_opts_t *opts, ft_stats_t *stats, int64_t *info);

#ifdef __cplusplus
}
#endif
#endif /* ABFT_H */
