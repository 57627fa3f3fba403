// ft_getrf.cu — LU with partial pivoting: PD checksum rules with pivot swaps
// (a4), left TRSM rule (a5), LU TMU rule (a6) and the fault-tolerant driver in
// Alg. 2 order (a7).
//
// Paper: full-checksum LU of [13] (L135-L145, §III.C): full checksums on the
// trailing matrix, c on the column panel, r on the row panel; Alg. 2
// (L364-L379); heuristic TMU check Fig. 4a (L359).  Readings: c-13 (LU rules),
// c-14 (pivot swap deltas from the pre-PD panel copy, L430), c-14b (pre-swap
// row check of every trailing row a swap moves), c-25 (Fig. 4a repair).
#include "ft_driver.cuh"

namespace abft {

// 1-based local pivots of the panel (cuSOLVER) -> 1-based global (LAPACK).
__global__ void lu_pivots_kernel(const int32_t* piv_local, int64_t* ipiv_global, int nb, int64_t r0) {
  for (int j = threadIdx.x; j < nb; j += blockDim.x) ipiv_global[j] = r0 + piv_local[j];
}

// The panel's pivot sequence as a permutation of the rows it moves: S (sorted
// distinct moved rows), src[s] = slot in S of the row whose value ends at
// S[s] after all nb swaps, tb[T - k] = first slot in tile row T (T = k..nt).
// One CTA of 1024 threads: bitonic sort in shared memory, then the nb swaps
// replayed on slot contents by one thread (row -> slot found in parallel).
__global__ void __launch_bounds__(1024) lu_perm_kernel(const int32_t* piv_local, int nb, int64_t r0, int nt, int k,
                                                       int64_t* S, int32_t* src, int32_t* tb, int32_t* nrows) {
  __shared__ int64_t key[2048];
  __shared__ int32_t content[2048];
  __shared__ int cnt;
  const int tid = threadIdx.x;
  for (int s = tid; s < 2048; s += blockDim.x) key[s] = INT64_MAX;
  __syncthreads();
  // candidates (p and q of every swap with p != q), duplicates kept for now
  for (int s = tid; s < 2 * nb; s += blockDim.x) {
    const int j = s < nb ? s : s - nb;
    const int64_t p = r0 + j, q = r0 + piv_local[j] - 1;
    if (p != q) key[s] = s < nb ? p : q;
  }
  __syncthreads();
  for (int size = 2; size <= 2048; size <<= 1)  // bitonic sort ascending
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
      for (int i = tid; i < 2048; i += blockDim.x) {
        const int partner = i ^ stride;
        if (partner > i) {
          const bool up = (i & size) == 0;
          const int64_t a = key[i], b = key[partner];
          if ((a > b) == up) {
            key[i] = b;
            key[partner] = a;
          }
        }
      }
      __syncthreads();
    }
  // unique: keep key[i] if it differs from key[i-1] (block scan of the flags)
  __shared__ int32_t wsum[32];
  __shared__ int64_t ukey[2048];
  __shared__ int16_t slotp[1024], slotq[1024];
  {
    const int i0 = 2 * tid, i1 = 2 * tid + 1;  // 1024 threads x 2 entries
    const int f0 = key[i0] != INT64_MAX && (i0 == 0 || key[i0] != key[i0 - 1]);
    const int f1 = key[i1] != INT64_MAX && key[i1] != key[i1 - 1];
    int v = f0 + f1, incl = v;
    const int lane = tid & 31, wid = tid >> 5;
    for (int m = 1; m < 32; m <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, incl, m);
      if (lane >= m) incl += y;
    }
    if (lane == 31) wsum[wid] = incl;
    __syncthreads();
    if (wid == 0) {
      int w = wsum[lane], wi = w;
      for (int m = 1; m < 32; m <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, wi, m);
        if (lane >= m) wi += y;
      }
      wsum[lane] = wi - w;  // exclusive warp offsets
      if (lane == 31) cnt = wi;
    }
    __syncthreads();
    const int excl = wsum[wid] + incl - v;
    if (f0) ukey[excl] = key[i0];
    if (f1) ukey[excl + f0] = key[i1];
  }
  __syncthreads();
  const int nu = cnt;
  for (int i = tid; i < 2048; i += blockDim.x) {
    key[i] = i < nu ? ukey[i] : INT64_MAX;
    content[i] = i;
  }
  __syncthreads();
  // row -> slot for both rows of every swap (parallel binary searches)
  for (int j = tid; j < nb; j += blockDim.x) {
    const int64_t p = r0 + j, q = r0 + piv_local[j] - 1;
    int sp = -1, sq = -1;
    if (p != q) {
      int lo = 0, hi = nu - 1;
      while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (key[mid] < p) lo = mid + 1; else hi = mid;
      }
      sp = lo;
      lo = 0;
      hi = nu - 1;
      while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (key[mid] < q) lo = mid + 1; else hi = mid;
      }
      sq = lo;
    }
    slotp[j] = (int16_t)sp;
    slotq[j] = (int16_t)sq;
  }
  __syncthreads();
  if (tid == 0) {  // the nb swaps in LAPACK order on slot contents (serial)
    for (int j = 0; j < nb; ++j) {
      const int a2 = slotp[j];
      if (a2 < 0) continue;
      const int b2 = slotq[j];
      const int t = content[a2];
      content[a2] = content[b2];
      content[b2] = t;
    }
  }
  __syncthreads();
  const int n = cnt;
  for (int s2 = tid; s2 < n; s2 += blockDim.x) {
    S[s2] = key[s2];
    src[s2] = content[s2];
  }
  for (int T = k + tid; T <= nt; T += blockDim.x) {  // first slot with row >= T*nb
    const int64_t r = (int64_t)T * nb;
    int lo = 0, hi = n;
    while (lo < hi) {
      const int mid = (lo + hi) >> 1;
      if (key[mid] < r) lo = mid + 1; else hi = mid;
    }
    tb[T - k] = lo;
  }
  if (tid == 0) *nrows = n;
}

// Pre-swap row check: row r of every trailing tile (I = r/nb, J > k) against
// its row checksums; a flagged tile gets ST_ROW so locate_correct treats it.
// One CTA per (tile column J, 32 consecutive entries of the sorted moved-row
// list): lane = moved row, so a warp's loads of one column are coalesced
// wherever the moved rows are contiguous (the panel's own rows); the 8 warps
// split the tile's columns and their partial sums are added in warp order.
// (A warp per (row, tile column) with lanes over columns read one 32-byte
// sector per element: 107 us per call at n=20480, profiles r01_s3.)
template <typename T>
__global__ void __launch_bounds__(256) lu_row_check_kernel(const T* A, int64_t lda, const T* rowchk, int64_t ldr,
                                                           const T* rowmag, int64_t ldrm, int use_mag, double tau_fac,
                                                           int nb, int k, int nt, const int64_t* rows,
                                                           const int32_t* nrows, int32_t* status, int64_t ld_status,
                                                           int32_t* counts) {
  __shared__ T part[8][32][3];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int ncols = nt - k - 1;
  if (ncols <= 0) return;
  const int J = k + 1 + (int)(blockIdx.x % ncols);
  const int ri = (int)(blockIdx.x / ncols) * 32 + lane;
  const int n = *nrows;
  if ((int)(blockIdx.x / ncols) * 32 >= n) return;  // whole CTA past the list (uniform)
  T e = T(0), w = T(0), a = T(0);
  const int cpw = nb / 8, c0 = warp * cpw;
  int64_t r = 0;
  if (ri < n) {
    r = rows[ri];
    const T* p = A + r + ((int64_t)J * nb + c0) * lda;
#pragma unroll 8
    for (int c = 0; c < cpw; ++c) {
      const T x = p[(int64_t)c * lda];
      e = fadd(e, x);
      w = ffma(T(c0 + c + 1), x, w);
      a = fadd(a, fabs(x));
    }
  }
  part[warp][lane][0] = e;
  part[warp][lane][1] = w;
  part[warp][lane][2] = a;
  __syncthreads();
  if (warp || ri >= n) return;
  for (int q = 1; q < 8; ++q) {
    e = fadd(e, part[q][lane][0]);
    w = fadd(w, part[q][lane][1]);
    a = fadd(a, part[q][lane][2]);
  }
  const T de = rowchk[r + (int64_t)(2 * J) * ldr] - e;
  const T dw = rowchk[r + (int64_t)(2 * J + 1) * ldr] - w;
  const double m = use_mag ? (double)rowmag[r + (int64_t)J * ldrm] : (double)a;
  const double t = tau_fac * m;
  const bool bad = !isfinite((double)de) || !isfinite((double)dw) || fabs((double)de) > t ||
                   fabs((double)dw) > (double)nb * t;
  if (!bad) return;
  atomicAdd(&counts[ABFT_CNT_ROWS_FLAGGED], 1);
  const int old = atomicOr(&status[r / nb + (int64_t)J * ld_status], ABFT_ST_ROW);
  if (!(old & (ABFT_ST_COL | ABFT_ST_ROW))) atomicAdd(&counts[ABFT_CNT_TILES_FLAGGED], 1);
}

// Row interchanges of every column outside the panel (LAPACK laswp) with
// the c-14 column-checksum deltas, applied as the net permutation of the moved
// rows: one CTA per column gathers the moved values into shared memory, the
// thread of each tile row sums its deltas in slot order (deterministic), then
// the permuted values are written back.  (Warp per tile row, lanes strided
// over its slots, butterfly reduction: a fixed order, so deterministic.)  Panel columns only update their
// checksums, with values from the pre-PD copy (L430).  Equal to the sequential
// swap rule in exact arithmetic.
// mode: 0 = every column (grid n), 1 = the panel's columns only (grid nb),
// 2 = every column outside the panel (grid n - nb; the look-ahead applies
// these after the rest of the TMU, reading c-35).
template <typename T>
__global__ void __launch_bounds__(256) lu_perm_cols_kernel(T* A, int64_t lda, int nb, int k, int nt, const int64_t* S,
                                                           const int32_t* src, const int32_t* tb,
                                                           const int32_t* nrows, const T* pcopy, int64_t ldp,
                                                           T* colchk, int64_t ldc, T* colmag, int64_t ldcm, int mode) {
  __shared__ T xs[2048];
  const int64_t r0 = (int64_t)k * nb, r1 = r0 + nb;
  const int64_t c = mode == 1 ? r0 + blockIdx.x : (mode == 2 && blockIdx.x >= r0 ? blockIdx.x + nb : blockIdx.x);
  const bool panel = c >= r0 && c < r1;
  if (panel && (!colchk || !pcopy)) return;  // no pcopy: restart undo, the panel is restored from its copy
  const int n = *nrows;
  const T* col = panel ? pcopy + (c - r0) * ldp - r0 : A + c * lda;
  for (int s = threadIdx.x; s < n; s += blockDim.x) xs[s] = col[S[s]];
  __syncthreads();
  if (colchk) {  // one warp per tile row: lane-strided slots, butterfly sum
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
    for (int T0 = wid; T0 < nt - k; T0 += nw) {
      const int b = tb[T0], e = tb[T0 + 1];
      if (b == e) continue;
      const int64_t base = (int64_t)(k + T0) * nb;
      T de = T(0), dw = T(0), da = T(0);
      for (int s = b + lane; s < e; s += 32) {
        const T xn = xs[src[s]], xo = xs[s];
        const T d = xn - xo;
        de += d;
        dw += T(S[s] - base + 1) * d;
        da += fabs(xn) - fabs(xo);
      }
      for (int m = 16; m >= 1; m >>= 1) {
        de += shfl_xor(de, m);
        dw += shfl_xor(dw, m);
        da += shfl_xor(da, m);
      }
      if (lane == 0) {
        const int64_t P = k + T0;
        colchk[2 * P + c * ldc] += de;
        colchk[2 * P + 1 + c * ldc] += dw;
        if (colmag) colmag[P + c * ldcm] += da;
      }
    }
  }
  if (panel) return;  // getrf already permuted the panel data
  T* colw = A + c * lda;
  for (int s = threadIdx.x; s < n; s += blockDim.x) colw[S[s]] = xs[src[s]];
}

// Row checksums (and row magnitudes) move with their rows (tile columns >= k).
template <typename T>
__global__ void __launch_bounds__(256) lu_perm_rowchk_kernel(T* rowchk, int64_t ldr, T* rowmag, int64_t ldrm, int J0,
                                                             const int64_t* S, const int32_t* src,
                                                             const int32_t* nrows) {
  __shared__ T vs[2048];
  const int J = J0 + blockIdx.x;
  const int n = *nrows;
  for (int a = 0; a < 3; ++a) {
    T* arr = a < 2 ? rowchk + (int64_t)(2 * J + a) * ldr : (rowmag ? rowmag + (int64_t)J * ldrm : nullptr);
    if (!arr) break;
    for (int s = threadIdx.x; s < n; s += blockDim.x) vs[s] = arr[S[s]];
    __syncthreads();
    for (int s = threadIdx.x; s < n; s += blockDim.x) arr[S[s]] = vs[src[s]];
    __syncthreads();
  }
}

// Fig. 4a repair for LU (c-25): a correction E of L21[p, q] or U12[q, c] found
// by the post-TMU panel re-check is pushed into the trailing matrix the TMU
// built from the bad value.  Single CTA, fixes in log order.
struct LuRepairArgs {
  void* A;
  int64_t lda, n, nb;
  int k;
  void *colchk, *rowchk, *colmag, *rowmag;
  int64_t ldc, ldr, ldcm, ldrm;
  const abft_fix_t* fixes;
  int cap;
  const int32_t* n_fixes;
  const int32_t* mark;
  int32_t* rep_counts;
  int32_t* counts;
  int64_t c0, c1;  // trailing columns to repair (look-ahead, reading c-35); [0, n) = all
};

template <typename T>
__global__ void lu_fig4a_repair_kernel(LuRepairArgs r) {
  const int n0 = *r.mark, n1 = min(*r.n_fixes, r.cap);
  T* A = reinterpret_cast<T*>(r.A);
  T* colchk = reinterpret_cast<T*>(r.colchk);
  T* rowchk = reinterpret_cast<T*>(r.rowchk);
  T* colmag = reinterpret_cast<T*>(r.colmag);
  T* rowmag = reinterpret_cast<T*>(r.rowmag);
  const int64_t nb = r.nb, nt = r.n / nb, k = r.k, r0 = k * nb, r1 = r0 + nb;
  __shared__ double s_max;
  __shared__ int s_skip;
  for (int f = n0; f < n1; ++f) {
    const abft_fix_t fx = r.fixes[f];
    if (fx.kind != ABFT_FIX_DATA) continue;
    const bool inL = fx.gj >= r0 && fx.gj < r1 && fx.gi >= r1;
    const bool inU = fx.gi >= r0 && fx.gi < r1 && fx.gj >= r1;
    if (!inL && !inU) continue;
    const double eps = fx.after - fx.before;
    double mx = 0.0;
    if (inL)
      for (int64_t a = r1 + threadIdx.x; a < r.n; a += blockDim.x) mx = fmax(mx, fabs((double)A[a + fx.gj * r.lda]));
    else
      for (int64_t c = r1 + threadIdx.x; c < r.n; c += blockDim.x) mx = fmax(mx, fabs((double)A[fx.gi + c * r.lda]));
    for (int m = 16; m >= 1; m >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, m));
    if (threadIdx.x == 0) s_max = 0.0;
    __syncthreads();
    if ((threadIdx.x & 31) == 0) atomicMax((unsigned long long*)&s_max, __double_as_longlong(mx));
    __syncthreads();
    if (threadIdx.x == 0) s_skip = !(isfinite(eps) && fabs(eps) <= 1024.0 * s_max);
    __syncthreads();
    if (s_skip) {
      if (threadIdx.x == 0) {
        atomicAdd(&r.rep_counts[1], 1);
        atomicAdd(&r.counts[ABFT_CNT_UNCORRECTABLE], 1);
      }
      __syncthreads();
      continue;
    }
    const T e = (T)eps, ae = fabs(e);
    if (inL) {  // row p of the trailing matrix: A[p, c] -= E U[q, c]; r(A_iJ)[p] -= E r(U_J)[q]
      const int64_t p = fx.gi, q = fx.gj - r0;
      const int64_t b0 = r1 > r.c0 ? r1 : r.c0, b1 = r.n < r.c1 ? r.n : r.c1;
      for (int64_t c = b0 + threadIdx.x; c < b1; c += blockDim.x) A[p + c * r.lda] -= e * A[r0 + q + c * r.lda];
      for (int64_t J = k + 1 + threadIdx.x; J < nt; J += blockDim.x) {
        if (J * nb < r.c0 || J * nb >= r.c1) continue;
        rowchk[p + 2 * J * r.ldr] -= e * rowchk[r0 + q + 2 * J * r.ldr];
        rowchk[p + (2 * J + 1) * r.ldr] -= e * rowchk[r0 + q + (2 * J + 1) * r.ldr];
        if (rowmag) rowmag[p + J * r.ldrm] += ae * rowmag[r0 + q + J * r.ldrm];
      }
    } else {  // column c: A[a, c] -= L[a, q] E; c(A_Ij)[:, c] -= E c(L_I)[:, q]
      const int64_t q = fx.gi - r0, c = fx.gj;
      const bool cin = c >= r.c0 && c < r.c1;
      for (int64_t a = r1 + threadIdx.x; cin && a < r.n; a += blockDim.x)
        A[a + c * r.lda] -= A[a + (r0 + q) * r.lda] * e;
      for (int64_t I = k + 1 + threadIdx.x; cin && I < nt; I += blockDim.x) {
        colchk[2 * I + c * r.ldc] -= e * colchk[2 * I + (r0 + q) * r.ldc];
        colchk[2 * I + 1 + c * r.ldc] -= e * colchk[2 * I + 1 + (r0 + q) * r.ldc];
        if (colmag) colmag[I + c * r.ldcm] += ae * colmag[I + (r0 + q) * r.ldcm];
      }
    }
    if (threadIdx.x == 0) atomicAdd(&r.rep_counts[0], 1);
    __syncthreads();
  }
}

// Inverse of the (S, src) permutation: sinv[src[s]] = s.
__global__ void lu_invert_perm_kernel(const int32_t* src, const int32_t* nrows, int32_t* sinv) {
  const int n = *nrows;
  for (int s = threadIdx.x; s < n; s += blockDim.x) sinv[src[s]] = s;
}

}  // namespace abft

// ------------------------------------------------------------ panel getrf --
// The permutation of one panel's pivots (lu_perm_kernel's output), read by
// the swap kernels and by the restart undo: local pivots | moved rows S |
// src | tile bounds | count.  In the caller's buffer when given (the driver:
// look-ahead splits the PD over two streams), else in stream scratch.
namespace abft {
struct LuPerm {
  int32_t* piv_local;
  int64_t* rows;
  int32_t* src;
  int32_t* tb;
  int32_t* nrows;
};
inline size_t lu_perm_bytes(int64_t nb, int64_t nt) {
  return (size_t)nb * 4 + 256 + (size_t)2 * nb * 8 + (size_t)2 * nb * 4 + ((size_t)nt + 2) * 4 + 4 + 256;
}
inline LuPerm lu_perm_at(void* buf, int64_t nb, int64_t nt) {
  char* b = (char*)buf;
  LuPerm P;
  P.rows = (int64_t*)b;                                   // 8-byte aligned first
  P.piv_local = (int32_t*)(b + (size_t)2 * nb * 8);
  P.src = P.piv_local + nb;
  P.nrows = P.src + 2 * nb;
  P.tb = P.nrows + 1;
  (void)nt;
  return P;
}
}  // namespace abft

// part 0: the whole PD (Alg. 2 order).  Look-ahead (reading c-35) splits it:
// part 1 = copy, factorization, pivots, the swaps' checksum deltas inside
// the panel, row checksums of tile column k moving with their rows, the
// diagonal inverses and the c(L), r(U_kk) rules; part 2 = the c-14b row check
// of the trailing rows a swap moves, the swaps of every column outside the
// panel (with their deltas) and the row checksums of tile columns > k.
// host != nullptr: the factorization is the FT_PD_HOST round trip (Alg. 2
// lines 3-7, ft_host.cu) instead of cuSOLVER.
static int panel_getrf_impl(const abft_mat_t* mat, int32_t k, int64_t* ipiv, const abft_tol_t* tol,
                            const abft_report_t* rep, abft_fix_t* fixes, int32_t max_fixes, int32_t* n_fixes,
                            void* Linv, void* Uinv, int32_t* info, abft_stream_t stream, abft::Driver* host,
                            int part = 0, void* perm_buf = nullptr);

extern "C" int abft_panel_getrf(const abft_mat_t* mat, int32_t k, int64_t* ipiv, const abft_tol_t* tol,
                                const abft_report_t* rep, abft_fix_t* fixes, int32_t max_fixes, int32_t* n_fixes,
                                void* Linv, void* Uinv, int32_t* info, abft_stream_t stream) {
  return panel_getrf_impl(mat, k, ipiv, tol, rep, fixes, max_fixes, n_fixes, Linv, Uinv, info, stream, nullptr);
}

static int panel_getrf_impl(const abft_mat_t* mat, int32_t k, int64_t* ipiv, const abft_tol_t* tol,
                            const abft_report_t* rep, abft_fix_t* fixes, int32_t max_fixes, int32_t* n_fixes,
                            void* Linv, void* Uinv, int32_t* info, abft_stream_t stream, abft::Driver* host,
                            int part, void* perm_buf) {
  using namespace abft;
  if (!mat || mat->m != mat->n || mat->nb < 32 || mat->nb > 1024 || (mat->nb & (mat->nb - 1)) ||
      mat->n % mat->nb || !mat->A || mat->lda < mat->m)
    return -1;
  const int64_t nb = mat->nb, n = mat->n, nt = n / nb;
  if (k < 0 || k >= nt) return -2;
  if (!ipiv) return -3;
  const bool ft = mat->colchk != nullptr;
  if (ft && (!mat->rowchk || !tol || !rep || !rep->status || !rep->counts || !n_fixes)) return -4;
  if (!Linv) return -9;
  if (!Uinv) return -10;
  if (!info) return -11;
  cudaStream_t s = (cudaStream_t)stream;
  const size_t es = mat->dtype == ABFT_F64 ? 8 : 4;
  const int64_t r0 = k * nb, mk = n - r0;
  char* A = (char*)mat->A;
  char* panel = A + (r0 + r0 * mat->lda) * es;
  if (!perm_buf) FT_TRY(scratch(s, 24, lu_perm_bytes(nb, nt), &perm_buf));
  const LuPerm P = lu_perm_at(perm_buf, nb, nt);
  auto perm_cols = [&](int mode) -> int {
    const unsigned grid = (unsigned)(mode == 0 ? n : (mode == 1 ? nb : n - nb));
    if (grid == 0) return 0;
    // scratch slot 10 holds the pre-PD panel copy (part 0 / 1 only read it)
    void* cp = nullptr;
    if (mode != 2 && ft) FT_TRY(scratch(s, 10, (size_t)mk * nb * es, &cp));
    if (mat->dtype == ABFT_F64)
      lu_perm_cols_kernel<double><<<grid, 256, 0, s>>>((double*)A, mat->lda, (int)nb, k, (int)nt, P.rows, P.src, P.tb,
                                                       P.nrows, (const double*)cp, mk, (double*)mat->colchk, mat->ldc,
                                                       (double*)mat->colmag, mat->ldcm, mode);
    else
      lu_perm_cols_kernel<float><<<grid, 256, 0, s>>>((float*)A, mat->lda, (int)nb, k, (int)nt, P.rows, P.src, P.tb,
                                                      P.nrows, (const float*)cp, mk, (float*)mat->colchk, mat->ldc,
                                                      (float*)mat->colmag, mat->ldcm, mode);
    ABFT_CUDA_TRY(cudaGetLastError());
    return 0;
  };
  auto perm_rowchk = [&](int J0, int J1) -> int {
    if (!ft || J1 <= J0) return 0;
    if (mat->dtype == ABFT_F64)
      lu_perm_rowchk_kernel<double><<<(unsigned)(J1 - J0), 256, 0, s>>>((double*)mat->rowchk, mat->ldr,
                                                                       (double*)mat->rowmag, mat->ldrm, J0, P.rows,
                                                                       P.src, P.nrows);
    else
      lu_perm_rowchk_kernel<float><<<(unsigned)(J1 - J0), 256, 0, s>>>((float*)mat->rowchk, mat->ldr,
                                                                      (float*)mat->rowmag, mat->ldrm, J0, P.rows,
                                                                      P.src, P.nrows);
    ABFT_CUDA_TRY(cudaGetLastError());
    return 0;
  };
  // c-14b: verify every trailing row a swap will move, fix before swapping
  auto row_check = [&]() -> int {
    if (!ft || k >= nt - 1) return 0;
    const int ncols = (int)(nt - k - 1);
    const int64_t items = (2 * nb + 31) / 32 * ncols;  // CTAs: (32-row chunk of <= 2nb moved rows, tile column)
    const bool use_mag = tol->kind == ABFT_TOL_MAGNITUDE && mat->rowmag;
    const double tf = mat->dtype == ABFT_F64 ? tau_factor<double>((int)nb, tol->scale)
                                             : tau_factor<float>((int)nb, tol->scale);
    if (mat->dtype == ABFT_F64)
      lu_row_check_kernel<double><<<(unsigned)items, 256, 0, s>>>(
          (const double*)A, mat->lda, (const double*)mat->rowchk, mat->ldr, (const double*)mat->rowmag, mat->ldrm,
          use_mag, tf, (int)nb, k, (int)nt, P.rows, P.nrows, rep->status, rep->ld_status, rep->counts);
    else
      lu_row_check_kernel<float><<<(unsigned)items, 256, 0, s>>>(
          (const float*)A, mat->lda, (const float*)mat->rowchk, mat->ldr, (const float*)mat->rowmag, mat->ldrm,
          use_mag, tf, (int)nb, k, (int)nt, P.rows, P.nrows, rep->status, rep->ld_status, rep->counts);
    ABFT_CUDA_TRY(cudaGetLastError());
    abft_tiles_t tr{(int)k, (int)nt, (int)k + 1, (int)nt, 0, ABFT_GENERAL};
    return abft_locate_correct(mat, &tr, ABFT_BOTH, tol, rep, fixes, max_fixes, n_fixes, stream);
  };
  if (part == 2) {  // look-ahead, after the rest of the TMU: outside the panel
    FT_TRY(row_check());
    FT_TRY(perm_cols(2));
    return perm_rowchk((int)k + 1, (int)nt);
  }
  // pre-PD panel copy (scratch slot 10) | getrf work (slot 12)
  int lwork = 0;
  if (!host) {
    std::unique_lock<std::mutex> lk;
    cusolverDnHandle_t h = solver_handle(s, lk);
    cusolverStatus_t st = mat->dtype == ABFT_F64
                              ? cusolverDnDgetrf_bufferSize(h, (int)mk, (int)nb, (double*)panel, (int)mat->lda, &lwork)
                              : cusolverDnSgetrf_bufferSize(h, (int)mk, (int)nb, (float*)panel, (int)mat->lda, &lwork);
    if (st != CUSOLVER_STATUS_SUCCESS) return ABFT_E_CUSOLVER;
  }
  if (ft) {
    void* cp = nullptr;
    FT_TRY(scratch(s, 10, (size_t)mk * nb * es, &cp));
    FT_TRY(abft::copy2d(cp, mk * es, panel, mat->lda * es, mk * es, nb, s));
  }
  if (host) {
    FT_TRY(host_panel_pd(*host, k, HOST_GETRF, r0, r0, mk, P.piv_local, nullptr, info));
  } else {
    void* work = nullptr;
    FT_TRY(scratch(s, 25, (size_t)(lwork + 1) * es, &work));
    std::unique_lock<std::mutex> lk;
    cusolverDnHandle_t h = solver_handle(s, lk);
    cusolverStatus_t st =
        mat->dtype == ABFT_F64
            ? cusolverDnDgetrf(h, (int)mk, (int)nb, (double*)panel, (int)mat->lda, (double*)work, P.piv_local, info)
            : cusolverDnSgetrf(h, (int)mk, (int)nb, (float*)panel, (int)mat->lda, (float*)work, P.piv_local, info);
    if (st != CUSOLVER_STATUS_SUCCESS) return ABFT_E_CUSOLVER;
  }
  lu_pivots_kernel<<<1, 256, 0, s>>>(P.piv_local, ipiv, (int)nb, r0);
  lu_perm_kernel<<<1, 1024, 0, s>>>(P.piv_local, (int)nb, r0, (int)nt, k, P.rows, P.src, P.tb, P.nrows);
  if (part == 0) {
    FT_TRY(row_check());
    // swaps: data outside the panel + c deltas (panel: from the pre-PD copy)
    FT_TRY(perm_cols(0));
    FT_TRY(perm_rowchk((int)k, (int)nt));
  } else {  // part 1: inside the panel only
    FT_TRY(perm_cols(1));
    FT_TRY(perm_rowchk((int)k, (int)k + 1));
  }
  // inverses of the diagonal factors (reused by the PU) and the c-13 PD rules
  FT_TRY(abft_tri_inverse(mat->dtype, 'L', 'U', nb, panel, mat->lda, Linv, nb, stream));
  FT_TRY(abft_tri_inverse(mat->dtype, 'U', 'N', nb, panel, mat->lda, Uinv, nb, stream));
  if (!ft) return 0;
  // c(L_I) = c(P~_I) U_kk^-1 for I >= k ; m_c <- m_c |U_kk^-1|
  FT_TRY(abft_update_trsm_inv(mat->dtype, 'R', 'N', nb, Uinv, nb, (char*)mat->colchk + (2 * k + r0 * mat->ldc) * es,
                              mat->ldc, 2 * (nt - k),
                              mat->colmag ? (char*)mat->colmag + (k + r0 * mat->ldcm) * es : nullptr, mat->ldcm,
                              nt - k, stream));
  // r(U_kk) = L_kk^-1 r(P~_kk) ; m_r <- |L_kk^-1| m_r
  FT_TRY(abft_update_trsm_inv(mat->dtype, 'L', 'N', nb, Linv, nb, (char*)mat->rowchk + (r0 + 2 * k * mat->ldr) * es,
                              mat->ldr, 2, mat->rowmag ? (char*)mat->rowmag + (r0 + k * mat->ldrm) * es : nullptr,
                              mat->ldrm, 1, stream));
  return 0;
}

// f1 (L430): take back the row swaps a part-0 panel_getrf_impl(k) applied
// outside its panel (permutation in perm_buf, or the stream scratch the PD
// used), with the column-checksum deltas and the row checksums moving back.
// The panel and its checksums are restored by the caller.
static int panel_getrf_undo(const abft_mat_t* mat, int k, cudaStream_t s, void* perm_buf) {
  using namespace abft;
  const int64_t nb = mat->nb, n = mat->n, nt = n / nb;
  if (!perm_buf) FT_TRY(scratch(s, 24, lu_perm_bytes(nb, nt), &perm_buf));
  const LuPerm P = lu_perm_at(perm_buf, nb, nt);
  void* si = nullptr;
  FT_TRY(scratch(s, 11, (size_t)2 * nb * 4, &si));
  int32_t* sinv = (int32_t*)si;
  lu_invert_perm_kernel<<<1, 1024, 0, s>>>(P.src, P.nrows, sinv);
  if (mat->dtype == ABFT_F64) {
    lu_perm_cols_kernel<double><<<(unsigned)n, 256, 0, s>>>((double*)mat->A, mat->lda, (int)nb, k, (int)nt, P.rows,
                                                            sinv, P.tb, P.nrows, nullptr, 0, (double*)mat->colchk,
                                                            mat->ldc, (double*)mat->colmag, mat->ldcm, 0);
    lu_perm_rowchk_kernel<double><<<(unsigned)(nt - k), 256, 0, s>>>((double*)mat->rowchk, mat->ldr,
                                                                    (double*)mat->rowmag, mat->ldrm, k, P.rows, sinv,
                                                                    P.nrows);
  } else {
    lu_perm_cols_kernel<float><<<(unsigned)n, 256, 0, s>>>((float*)mat->A, mat->lda, (int)nb, k, (int)nt, P.rows,
                                                           sinv, P.tb, P.nrows, nullptr, 0, (float*)mat->colchk,
                                                           mat->ldc, (float*)mat->colmag, mat->ldcm, 0);
    lu_perm_rowchk_kernel<float><<<(unsigned)(nt - k), 256, 0, s>>>((float*)mat->rowchk, mat->ldr,
                                                                   (float*)mat->rowmag, mat->ldrm, k, P.rows, sinv,
                                                                   P.nrows);
  }
  ABFT_CUDA_TRY(cudaGetLastError());
  return 0;
}

// ----------------------------------------------------------------- driver --
extern "C" int ft_getrf(ft_ctx_t* c, int32_t dtype, int64_t n, void* dA, int64_t lda, int64_t* ipiv,
                        const ft_opts_t* o, ft_stats_t* stats, int64_t* info_out) {
  using namespace abft;
  if (!c) return -1;
  if (dtype != ABFT_F32 && dtype != ABFT_F64) return -2;
  if (!o) return -7;
  const int64_t nb = o->nb;
  if (n < 0 || nb < 32 || nb > 1024 || (nb & (nb - 1)) || n % nb) return -3;
  if (!dA) return -4;
  if (lda < std::max<int64_t>(1, n)) return -5;
  if (!ipiv) return -6;
  if (o->n_inject < 0 || (o->n_inject > 0 && !o->inject)) return -7;
  if (o->scheme != FT_SCHEME_NEW || o->checksum_gemm) return -7;  // scheme / GEMM-check comparisons: ft_potrf only
  ABFT_CUDA_TRY(cudaSetDevice(c->device));
  Driver d;
  FT_TRY(d.setup(c, dtype, n, nb, dA, lda, o, /*lu=*/true));
  const int64_t nt = d.nt;
  const bool ft = o->abft != 0;
  std::unique_lock<std::mutex> lk;
  auto t0 = std::chrono::steady_clock::now();
  // the panel's permutation lives in a context buffer shared by both streams
  // (the look-ahead factors the panel on the side stream and applies the
  // swaps outside it on the main one)
  FT_TRY(grow_buffer(c->aux, c->aux_bytes, lu_perm_bytes(nb, nt)));
  void* perm = c->aux;
  const bool la_on = o->lookahead != 0;
  if (la_on) FT_TRY(d.side_setup());
  // the same predicate as oracle/drivers.py::lu_lookahead_ok
  auto la_at = [&](int k) -> bool {
    if (k + 1 >= nt) return false;
    if (ft && o->trailing_check_period > 0 && (k + 1) % o->trailing_check_period == 0) return false;
    const int64_t c0 = (int64_t)(k + 1) * nb, c1 = c0 + nb;
    for (int t = 0; t < o->n_inject; ++t) {
      const ft_inject_t& f = o->inject[t];
      if (f.iter == k && (f.point == FT_AT_PRE_TMU || f.point == FT_AT_POST_TMU)) return false;
      const bool pd_point = f.point == FT_AT_PRE_PD_CHECK || f.point == FT_AT_PRE_PD || f.point == FT_AT_POST_PD ||
                            f.point == FT_AT_D2H || f.point == FT_AT_H2D;
      if (f.iter == k + 1 && pd_point) {
        bool inside;
        if (f.target == 0 || f.target == 1)
          inside = f.gj >= c0 && f.gj < c1;
        else if (f.target == 2)
          inside = f.gj == 2 * (k + 1) || f.gj == 2 * (k + 1) + 1;
        else
          inside = false;
        if (!inside) return false;
      }
    }
    return true;
  };
  if (ft) {
    PhaseScope ps(d, FT_PH_ENCODE);
    abft_tiles_t all{0, (int)nt, 0, (int)nt, 0, ABFT_GENERAL};
    FT_TRY(abft_encode(&d.M, &all, ABFT_BOTH, (abft_stream_t)d.s));
  }
  const bool rs = ft && o->restart;

  // ---- Alg. 2 lines 3-7 of iteration k on d.s: check the column panel, PD,
  // check L and U_kk, local restart.  split: the look-ahead's part 1 (the
  // swaps outside the panel follow as pd_outside(k) on the main stream).
  auto chain_pd = [&](int k, bool split) -> int {
    cudaStream_t s = d.s;
    const abft_stream_t as = (abft_stream_t)s;
    const int64_t r0 = k * nb;
    if (ft) FT_TRY(d.begin_iteration());
    // Alg. 2 lines 3-4: check the column panel to be decomposed (c + r)
    // Local restart (f1, L430): the column panel with its checksums is copied
    // after its pre-op check (the panel by the check's own pass); layout in
    // rsv: panel | c | m_c | r | m_r
    const int64_t mk = n - r0;
    const int ntk = (int)(nt - k);
    char* rb = (char*)c->rsv;
    char* cp_a = rb;
    char* cp_c = cp_a + (size_t)mk * nb * d.es;
    char* cp_m = cp_c + (size_t)2 * ntk * nb * d.es;
    char* cp_r = cp_m + (size_t)ntk * nb * d.es;
    char* cp_rm = cp_r + (size_t)mk * 2 * d.es;
    FT_TRY(d.inject_at(k, FT_AT_PRE_PD_CHECK));
    if (ft) FT_TRY(d.check(k, (int)nt, k, k + 1, ABFT_GENERAL, ABFT_BOTH, false, nullptr, rs ? cp_a : nullptr, mk));
    if (rs) {
      PhaseScope ps(d, FT_PH_RESTART);
      FT_TRY(d.copies({{cp_c, 2 * ntk, d.colchk_at(2 * k, r0), d.M.ldc, 2 * ntk, nb},
                       {cp_m, ntk, d.colmag_at(k, r0), d.M.ldcm, ntk, nb},
                       {cp_r, mk, d.rowchk_at(r0, 2 * k), d.M.ldr, mk, 2},
                       {cp_rm, mk, d.rowmag_at(r0, k), d.M.ldrm, mk, 1}}));
    }
    // line 5: PD with pivoting, swap rule, c(L), r(U_kk)
    auto do_pd = [&]() -> int {
      PhaseScope ps(d, FT_PH_PD);
      FT_TRY(panel_getrf_impl(&d.M, k, ipiv + r0, ft ? &d.tol : nullptr, ft ? &d.R : nullptr, c->fixlog,
                              c->fixcap, d.nfix, c->linv, c->uinv, d.info, as,
                              o->pd_location == FT_PD_HOST ? &d : nullptr, split ? 1 : 0, perm));
      if (ft && !split && k < nt - 1) ++d.n_checks;  // the pre-swap row check (c-14b)
      accum_info_kernel<<<1, 1, 0, s>>>(d.info, d.info_total, r0);
      return 0;
    };
    auto post_pd_checks = [&]() -> int {
      FT_TRY(d.check(k, (int)nt, k, k + 1, ABFT_UNIT_LOWER, ABFT_COL));
      return d.check(k, k + 1, k, k + 1, ABFT_UPPER, ABFT_ROW);
    };
    FT_TRY(d.inject_at(k, FT_AT_PRE_PD));
    FT_TRY(do_pd());
    FT_TRY(d.restore_onchip());
    FT_TRY(d.inject_at(k, FT_AT_POST_PD));
    // line 7: check the decomposed panel: L (UNIT_LOWER on the diagonal, c) and U_kk (r)
    if (ft) {
      if (rs) FT_TRY(d.snap_uncorrectable());
      FT_TRY(post_pd_checks());
      auto pd_redo = [&]() -> int {  // 2D after the PD: undo its swaps, restore the copy, redo
        PhaseScope ps(d, FT_PH_RESTART);
        if (!split) FT_TRY(panel_getrf_undo(&d.M, k, s, perm));  // split: nothing outside the panel moved yet
        FT_TRY(d.copies({{d.a_at(r0, r0), lda, cp_a, mk, mk, nb},
                         {d.colchk_at(2 * k, r0), d.M.ldc, cp_c, 2 * ntk, 2 * ntk, nb},
                         {d.colmag_at(k, r0), d.M.ldcm, cp_m, ntk, ntk, nb},
                         {d.rowchk_at(r0, 2 * k), d.M.ldr, cp_r, mk, mk, 2},
                         {d.rowmag_at(r0, k), d.M.ldrm, cp_rm, mk, mk, 1}}));
        return 0;
      };
      // (The PD redo stays a host decision: cuSOLVER's getrf cannot read a
      // device gate; the PU redo below is device-decided.)
      int delta = 0;
      if (rs) FT_TRY(d.uncorrectable_added(&delta));
      if (delta > 0) {
        FT_TRY(d.take_back_uncorrectable(delta));
        FT_TRY(pd_redo());
        FT_TRY(do_pd());
        FT_TRY(post_pd_checks());
      }
    }
    return 0;
  };
  // ---- the look-ahead's part 2 of PD k (main stream, after the TMU that
  // shared its columns): c-14b row check, swaps outside the panel
  auto pd_outside = [&](int k) -> int {
    PhaseScope ps(d, FT_PH_PD);
    FT_TRY(panel_getrf_impl(&d.M, k, ipiv + k * nb, ft ? &d.tol : nullptr, ft ? &d.R : nullptr, c->fixlog, c->fixcap,
                            d.nfix, c->linv, c->uinv, d.info, (abft_stream_t)d.s, nullptr, 2, perm));
    if (ft && k < nt - 1) ++d.n_checks;  // the pre-swap row check (c-14b)
    return 0;
  };
  // ---- Alg. 2 lines 8-10: check the row panel, PU, check U12 (main stream)
  auto chain_pu = [&](int k) -> int {
    cudaStream_t s = d.s;
    const abft_stream_t as = (abft_stream_t)s;
    const int64_t r0 = k * nb, r1 = r0 + nb, nk = n - r1;
    const int m2 = (int)(2 * (nt - k - 1));
    char* rb = (char*)c->rsv;
    // line 8: check the row panel to be updated (c + r)
    // local restart copy of the row panel: A12 (by the check's own pass) |
    // r(A12) | m_r(A12)
    char* pu_a = rb;
    char* pu_r = pu_a + (size_t)nb * nk * d.es;
    char* pu_rm = pu_r + (size_t)nb * m2 * d.es;
    FT_TRY(d.inject_at(k, FT_AT_PRE_PU_CHECK));
    if (ft) FT_TRY(d.check(k, k + 1, k + 1, (int)nt, ABFT_GENERAL, ABFT_BOTH, false, nullptr, rs ? pu_a : nullptr, nb));
    if (rs) {
      PhaseScope ps(d, FT_PH_RESTART);
      FT_TRY(d.copies({{pu_r, nb, d.rowchk_at(r0, 2 * (k + 1)), d.M.ldr, nb, m2},
                       {pu_rm, nb, d.rowmag_at(r0, k + 1), d.M.ldrm, nb, m2 / 2}}));
    }
    // Fig. 4b (L359): a 1D pattern fixed in this iteration -> check the trailing matrix
    if (ft) FT_TRY(d.fig4b_check(k + 1, (int)nt, k + 1, (int)nt, ABFT_GENERAL, ABFT_BOTH, false));
    // line 9: PU  U12 = L_kk^-1 A12 (DGEMM with the PD's inverse) + r rule
    FT_TRY(d.inject_at(k, FT_AT_PRE_PU));
    const bool refresh = d.diag_touched_before_pu(k);
    if (refresh) FT_TRY(abft_tri_inverse(dtype, 'L', 'U', nb, d.a_at(r0, r0), lda, c->linv, nb, as));
    auto pu_data = [&]() -> int {
      PhaseScope ps(d, FT_PH_PU);
      // not in place: from the local-restart copy of A12 straight into A12 when
      // there is one (no fault plan: copy == A12), else via scratch + copy back
      const bool from_copy = rs && o->n_inject == 0;
      const void* src = from_copy ? (const void*)pu_a : d.a_at(r0, r1);
      const int lds = from_copy ? (int)nb : (int)lda;
      void* dst = from_copy ? d.a_at(r0, r1) : c->putmp;
      const int ldd = from_copy ? (int)lda : (int)nb;
      cublasHandle_t h = blas_handle(s, lk);
      cublasStatus_t st;
      if (dtype == ABFT_F64) {
        const double one = 1.0, zero = 0.0;
        st = cublasDgemm(h, CUBLAS_OP_N, CUBLAS_OP_N, (int)nb, (int)nk, (int)nb, &one, (const double*)c->linv,
                         (int)nb, (const double*)src, lds, &zero, (double*)dst, ldd);
      } else {
        const float one = 1.0f, zero = 0.0f;
        st = cublasSgemm(h, CUBLAS_OP_N, CUBLAS_OP_N, (int)nb, (int)nk, (int)nb, &one, (const float*)c->linv, (int)nb,
                         (const float*)src, lds, &zero, (float*)dst, ldd);
      }
      lk.unlock();
      if (st != CUBLAS_STATUS_SUCCESS) return ABFT_E_CUBLAS;
      if (from_copy) return 0;
      return abft::copy2d(d.a_at(r0, r1), lda * d.es, c->putmp, nb * d.es, nb * d.es, nk, s);
    };
    auto pu_chk = [&]() -> int {  // r(U_kJ) = L_kk^-1 r(A_kJ), m_r <- |L_kk^-1| m_r  (c-13)
      PhaseScope ps(d, FT_PH_RULES);
      return abft_update_trsm_inv(dtype, 'L', 'N', nb, c->linv, nb, d.rowchk_at(r0, 2 * (k + 1)), d.M.ldr, m2,
                                  d.rowmag_at(r0, k + 1), d.M.ldrm, m2 / 2, as);
    };
    FT_TRY(pu_data());
    FT_TRY(d.restore_onchip());
    if (refresh) FT_TRY(abft_tri_inverse(dtype, 'L', 'U', nb, d.a_at(r0, r0), lda, c->linv, nb, as));
    if (ft) FT_TRY(pu_chk());
    FT_TRY(d.inject_at(k, FT_AT_POST_PU));
    // line 10: check the updated row panel (r); 2D -> local restart of the PU (L430, L434)
    if (ft) {
      if (rs) FT_TRY(d.snap_uncorrectable());
      FT_TRY(d.check(k, k + 1, k + 1, (int)nt, ABFT_GENERAL, ABFT_ROW));
      // 2D after the PU: local restart from the pre-PU copy (L430), decided on
      // the device (Driver::gated_restart): U12 = L_kk^-1 A12, its row
      // checksums and magnitudes as gated GEMMs from the copy, then re-check.
      auto pu_redo = [&](const int32_t* g) -> int {
        {
          PhaseScope ps(d, FT_PH_RESTART);
          // data, checksum and magnitude products as one gated launch
          const GatedGemm gg[3] = {{nb, nk, nb, c->linv, nb, pu_a, nb, d.a_at(r0, r1), lda, 0, 0, 0, 0},
                                   {nb, m2, nb, c->linv, nb, pu_r, nb, d.rowchk_at(r0, 2 * (k + 1)), d.M.ldr, 0, 0, 0, 0},
                                   {nb, m2 / 2, nb, c->linv, nb, pu_rm, nb, d.rowmag_at(r0, k + 1), d.M.ldrm, 0, 0, 1,
                                    0}};
          FT_TRY(gemm_gated_multi(dtype, gg, 3, g, s));
        }
        return d.check(k, k + 1, k + 1, (int)nt, ABFT_GENERAL, ABFT_ROW);
      };
      if (rs) FT_TRY(d.gated_restart(1, pu_redo));
    }
    return 0;
  };
  // ---- TMU data on trailing columns [c0, c1): A[r1:, c0:c1] -= L21 U12[:, c0-r1 ..]
  auto tmu_data = [&](int k, int64_t c0, int64_t c1) -> int {
    const int64_t r0 = k * nb, r1 = r0 + nb, rows = n - r1, w = c1 - c0;
    if (w <= 0 || rows <= 0) return 0;
    PhaseScope ps(d, FT_PH_TMU);
    cublasHandle_t h = blas_handle(d.s, lk);
    cublasStatus_t st;
    if (dtype == ABFT_F64) {
      const double m1 = -1.0, one = 1.0;
      st = cublasDgemm(h, CUBLAS_OP_N, CUBLAS_OP_N, (int)rows, (int)w, (int)nb, &m1, (const double*)d.a_at(r1, r0),
                       (int)lda, (const double*)d.a_at(r0, c0), (int)lda, &one, (double*)d.a_at(r1, c0), (int)lda);
    } else {
      const float m1 = -1.0f, one = 1.0f;
      st = cublasSgemm(h, CUBLAS_OP_N, CUBLAS_OP_N, (int)rows, (int)w, (int)nb, &m1, (const float*)d.a_at(r1, r0),
                       (int)lda, (const float*)d.a_at(r0, c0), (int)lda, &one, (float*)d.a_at(r1, c0), (int)lda);
    }
    lk.unlock();
    return st == CUBLAS_STATUS_SUCCESS ? 0 : ABFT_E_CUBLAS;
  };
  // ---- TMU checksum rules (c-13) for trailing tile columns [c0, c1)
  auto tmu_chk = [&](int k, int64_t c0, int64_t c1) -> int {
    const int64_t r0 = k * nb, r1 = r0 + nb;
    const int J0 = (int)(c0 / nb), J1 = (int)(c1 / nb);
    const int m2 = (int)(2 * (nt - k - 1));
    if (J1 <= J0) return 0;
    PhaseScope ps(d, FT_PH_RULES);
    const abft_stream_t as = (abft_stream_t)d.s;
    // c(A_IJ) -= c(L_Ik) U_kJ
    FT_TRY(abft_update_gemm(dtype, ABFT_COL, 'N', 'N', -1.0, d.colchk_at(2 * (k + 1), r0), d.M.ldc, d.a_at(r0, c0),
                            lda, d.colchk_at(2 * (k + 1), c0), d.M.ldc, m2, c1 - c0, nb, d.colmag_at(k + 1, r0),
                            d.M.ldcm, d.colmag_at(k + 1, c0), d.M.ldcm, as));
    // r(A_IJ) -= L_Ik r(U_kJ)
    if (J1 - J0 == 1)  // one tile column (look-ahead's first part): one pass over L21, no |L21| copy
      return panel_row_rule(dtype, n - r1, nb, d.a_at(r1, r0), lda, d.rowchk_at(r0, 2 * J0),
                            d.rowchk_at(r0, 2 * J0 + 1), 1, d.rowmag_at(r0, J0), 1, d.rowchk_at(r1, 2 * J0),
                            d.rowchk_at(r1, 2 * J0 + 1), d.rowmag_at(r1, J0), d.s);
    return abft_update_gemm(dtype, ABFT_ROW, 'N', 'N', -1.0, d.rowchk_at(r0, 2 * J0), d.M.ldr, d.a_at(r1, r0), lda,
                            d.rowchk_at(r1, 2 * J0), d.M.ldr, 2 * (J1 - J0), n - r1, nb, d.rowmag_at(r0, J0),
                            d.M.ldrm, d.rowmag_at(r1, J0), d.M.ldrm, as);
  };
  // ---- line 13: heuristic re-check of both panels (Fig. 4a) + guarded repair
  // restricted to the trailing columns [c0, c1) that consumed the panels
  auto recheck = [&](int k, int64_t c0, int64_t c1) -> int {
    ABFT_CUDA_TRY(cudaMemcpyAsync(d.mark, d.nfix, sizeof(int32_t), cudaMemcpyDeviceToDevice, d.s));
    FT_TRY(d.check(k + 1, (int)nt, k, k + 1, ABFT_GENERAL, ABFT_COL));
    FT_TRY(d.check(k, k + 1, k + 1, (int)nt, ABFT_GENERAL, ABFT_ROW));
    if (!o->fig4a_repair) return 0;
    PhaseScope ps(d, FT_PH_OTHER);
    LuRepairArgs ra{};
    ra.A = dA;
    ra.lda = lda;
    ra.n = n;
    ra.nb = nb;
    ra.k = k;
    ra.colchk = d.M.colchk;
    ra.rowchk = d.M.rowchk;
    ra.colmag = d.M.colmag;
    ra.rowmag = d.M.rowmag;
    ra.ldc = d.M.ldc;
    ra.ldr = d.M.ldr;
    ra.ldcm = d.M.ldcm;
    ra.ldrm = d.M.ldrm;
    ra.fixes = c->fixlog;
    ra.cap = c->fixcap;
    ra.n_fixes = d.nfix;
    ra.mark = d.mark;
    ra.rep_counts = d.rep;
    ra.counts = d.counts;
    ra.c0 = c0;
    ra.c1 = c1;
    if (dtype == ABFT_F64)
      lu_fig4a_repair_kernel<double><<<1, 256, 0, d.s>>>(ra);
    else
      lu_fig4a_repair_kernel<float><<<1, 256, 0, d.s>>>(ra);
    ABFT_CUDA_TRY(cudaGetLastError());
    return 0;
  };

  bool chained = false;  // PD k already factored by the look-ahead (part 1)
  for (int k = 0; k < nt; ++k) {
    d.iter_event();
    const int64_t r1 = (int64_t)(k + 1) * nb, r2 = r1 + nb;
    if (!chained)
      FT_TRY(chain_pd(k, false));
    else
      FT_TRY(pd_outside(k));
    chained = false;
    if (k == nt - 1) break;
    FT_TRY(chain_pu(k));
    // line 12: TMU  A22 -= L21 U12 (DGEMM on tensor cores) + c-13 rules
    FT_TRY(d.inject_at(k, FT_AT_PRE_TMU));
    if (la_on && la_at(k)) {
      // look-ahead (c-35): tile column k+1 first, the re-checks, then the
      // rest while the side stream factors panel k+1 (part 1; enqueued after
      // the rest, so its host wait overlaps the DGEMM)
      FT_TRY(tmu_data(k, r1, r2));
      FT_TRY(d.restore_onchip());
      if (ft) {
        FT_TRY(tmu_chk(k, r1, r2));
        FT_TRY(recheck(k, r1, r2));
      }
      ABFT_CUDA_TRY(cudaEventRecord(c->ev_col, d.s));
      // the rest's checksum rules on a stream of its own next to the DGEMM
      // (they read the re-checked panels L21, U12 and their checksums and
      // write the checksums of tile columns >= k+2, which neither the DGEMM
      // nor the side chain's panel k+1 touches), joined before the re-check;
      // runs with a fault plan keep Alg. 2's sequential order
      static const bool rule_seq = getenv("ABFT_RULE_STREAM") && atoi(getenv("ABFT_RULE_STREAM")) == 0;
      const bool par = ft && !rule_seq && o->n_inject == 0;
      if (par) {
        FT_TRY(d.rule_setup());
        ABFT_CUDA_TRY(cudaStreamWaitEvent(c->rule, c->ev_col, 0));
        cudaStream_t keep = d.s;
        d.s = c->rule;
        const int rc = tmu_chk(k, r2, n);
        d.s = keep;
        FT_TRY(rc);
        ABFT_CUDA_TRY(cudaEventRecord(c->ev_rule, c->rule));
      }
      FT_TRY(tmu_data(k, r2, n));
      if (ft) {
        if (!par) FT_TRY(tmu_chk(k, r2, n));
        FT_TRY(d.inject_at(k, FT_AT_POST_TMU));
        if (par) ABFT_CUDA_TRY(cudaStreamWaitEvent(d.s, c->ev_rule, 0));
        FT_TRY(recheck(k, r2, n));
      }
      ABFT_CUDA_TRY(cudaStreamWaitEvent(c->side, c->ev_col, 0));
      d.on_side(true);
      const int rc = chain_pd(k + 1, true);
      if (rc == 0) ABFT_CUDA_TRY(cudaEventRecord(c->ev_side, d.s));
      d.on_side(false);
      if (rc) return rc;
      ABFT_CUDA_TRY(cudaStreamWaitEvent(d.s, c->ev_side, 0));
      chained = true;
      continue;
    }
    FT_TRY(tmu_data(k, r1, n));
    FT_TRY(d.restore_onchip());
    if (ft) FT_TRY(tmu_chk(k, r1, n));
    FT_TRY(d.inject_at(k, FT_AT_POST_TMU));
    if (ft) {
      FT_TRY(recheck(k, 0, n));
      FT_TRY(d.periodic_check(k, k + 1, (int)nt, k + 1, (int)nt, ABFT_GENERAL, false));  // L359
    }
  }
  d.iter_event();
  return d.finish(t0, stats, info_out);
}
