// ft_potrf.cu — PD checksum rule for Cholesky (a4) and the fault-tolerant
// Cholesky driver in the paper's reordered checking scheme (a7).
//
// Paper: Table II / §IV.A (L152-L189) full-checksum Cholesky; Alg. 2
// (L364-L379) checking order; heuristic TMU checking Fig. 4a (L357-L359);
// PD on the CPU in MAGMA (L61) — here the PD runs on the device (cuSOLVER),
// DESIGN.md §7 explains why.  Readings: c-12 (Cholesky rules), c-24 (views
// before/after PD), c-25 (guarded Fig. 4a trailing repair), c-8 (fault hooks).
#include <cublas_v2.h>
#include <cusolverDn.h>

#include <chrono>
#include <mutex>
#include <vector>

#include "abft_common.cuh"

namespace abft {
cublasHandle_t blas_handle(cudaStream_t s, std::unique_lock<std::mutex>& lk);
cusolverDnHandle_t solver_handle(cudaStream_t s, std::unique_lock<std::mutex>& lk);
int scratch(cudaStream_t s, int slot, size_t bytes, void** out);
}  // namespace abft

#define FT_TRY(expr)          \
  do {                        \
    int _rc = (expr);         \
    if (_rc) return _rc;      \
  } while (0)

// ------------------------------------------------------------ panel potrf --
namespace abft {
template <typename T>
static int potrf_tile(const abft_mat_t* d, int32_t* info, cudaStream_t s) {
  std::unique_lock<std::mutex> lk;
  cusolverDnHandle_t h = solver_handle(s, lk);
  int lwork = 0;
  cusolverStatus_t st;
  if (sizeof(T) == 8)
    st = cusolverDnDpotrf_bufferSize(h, CUBLAS_FILL_MODE_LOWER, (int)d->nb, (double*)d->A, (int)d->lda, &lwork);
  else
    st = cusolverDnSpotrf_bufferSize(h, CUBLAS_FILL_MODE_LOWER, (int)d->nb, (float*)d->A, (int)d->lda, &lwork);
  if (st != CUSOLVER_STATUS_SUCCESS) return ABFT_E_CUSOLVER;
  void* w = nullptr;
  FT_TRY(scratch(s, 4, (size_t)(lwork + 1) * sizeof(T), &w));
  if (sizeof(T) == 8)
    st = cusolverDnDpotrf(h, CUBLAS_FILL_MODE_LOWER, (int)d->nb, (double*)d->A, (int)d->lda, (double*)w, lwork, info);
  else
    st = cusolverDnSpotrf(h, CUBLAS_FILL_MODE_LOWER, (int)d->nb, (float*)d->A, (int)d->lda, (float*)w, lwork, info);
  if (st != CUSOLVER_STATUS_SUCCESS) return ABFT_E_CUSOLVER;
  return 0;
}
}  // namespace abft

extern "C" int abft_panel_potrf(const abft_mat_t* d, void* Linv, int64_t ldw, int32_t* info, abft_stream_t stream) {
  if (!d || d->m != d->nb || d->n != d->nb || !d->A || d->lda < d->nb) return -1;
  if (Linv && ldw < d->nb) return -3;
  if (!info) return -4;
  if (d->dtype != ABFT_F32 && d->dtype != ABFT_F64) return -1;
  cudaStream_t s = (cudaStream_t)stream;
  int rc = d->dtype == ABFT_F64 ? abft::potrf_tile<double>(d, info, s) : abft::potrf_tile<float>(d, info, s);
  if (rc) return rc;
  if (!d->colchk && !Linv) return 0;
  // L_kk^-1 once (reused by the caller for the PU when Linv is given)
  void* W = Linv;
  int64_t ldW = ldw;
  if (!W) {
    FT_TRY(abft::scratch(s, 8, (size_t)d->nb * d->nb * (d->dtype == ABFT_F64 ? 8 : 4), &W));
    ldW = d->nb;
  }
  FT_TRY(abft_tri_inverse(d->dtype, 'L', 'N', d->nb, d->A, d->lda, W, ldW, stream));
  if (!d->colchk) return 0;
  // c(L_kk) = c_sym(A_kk) L_kk^-T ; m_c(L_kk) = m_c |L_kk^-T|   (c-12, c-6)
  return abft_update_trsm_inv(d->dtype, 'R', 'T', d->nb, W, ldW, d->colchk, d->ldc, 2, d->colmag, d->ldcm,
                              d->colmag ? 1 : 0, stream);
}

// --------------------------------------------------------- Fig. 4a repair --
namespace abft {
struct RepairArgs {
  void* A;
  int64_t lda, n, nb;
  int k;
  void *colchk, *rowchk, *colmag, *rowmag;
  int64_t ldc, ldr, ldcm, ldrm;
  const abft_fix_t* fixes;
  int cap;
  const int32_t* n_fixes;
  const int32_t* mark;
  int32_t* rep_counts;  // [0] applied, [1] skipped
  int32_t* counts;      // report counts: a skipped repair is uncorrectable (R)
};

template <typename T>
__global__ void fig4a_repair_kernel(RepairArgs r) {
  const int n0 = *r.mark, n1 = min(*r.n_fixes, r.cap);
  T* A = reinterpret_cast<T*>(r.A);
  T* colchk = reinterpret_cast<T*>(r.colchk);
  T* rowchk = reinterpret_cast<T*>(r.rowchk);
  T* colmag = reinterpret_cast<T*>(r.colmag);
  T* rowmag = reinterpret_cast<T*>(r.rowmag);
  const int64_t nb = r.nb, nt = r.n / nb, k = r.k;
  const int64_t row0 = (k + 1) * nb;  // first trailing row
  __shared__ double s_max;
  __shared__ int s_skip;
  for (int f = n0; f < n1; ++f) {
    abft_fix_t fx = r.fixes[f];
    if (fx.kind != ABFT_FIX_DATA) continue;
    const int64_t p = fx.gi, q = fx.gj;
    if (q < k * nb || q >= (k + 1) * nb || p < row0) continue;  // not a panel element of this iteration
    const double eps = fx.after - fx.before;                    // E = L_true - L_bad
    // guard (c-25): |E| <= 2^10 max|L_panel(:, q)| and finite
    double mx = 0.0;
    for (int64_t a = row0 + threadIdx.x; a < r.n; a += blockDim.x) mx = fmax(mx, fabs((double)A[a + q * r.lda]));
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
      continue;
    }
    const T e = (T)eps;
    const T ae = fabs(e);
    const int64_t i = p / nb, pl = p % nb, ql = q - k * nb;
    // data: row p left of the diagonal, column p below it, and (p, p)
    for (int64_t b = row0 + threadIdx.x; b < p; b += blockDim.x) A[p + b * r.lda] -= e * A[b + q * r.lda];
    for (int64_t a = p + 1 + threadIdx.x; a < r.n; a += blockDim.x) A[a + p * r.lda] -= e * A[a + q * r.lda];
    if (threadIdx.x == 0) A[p + p * r.lda] -= 2 * e * A[p + q * r.lda] - e * e;
    // column checksums of tile column i: c(A_Ii)[:, pl] -= E * c(L_I)[:, ql], I >= i
    for (int64_t I = i + threadIdx.x; I < nt; I += blockDim.x) {
      T* dst = colchk + 2 * I + (i * nb + pl) * r.ldc;
      const T* src = colchk + 2 * I + (k * nb + ql) * r.ldc;
      dst[0] -= e * src[0];
      dst[1] -= e * src[1];
      if (colmag) colmag[I + (i * nb + pl) * r.ldcm] += ae * colmag[I + (k * nb + ql) * r.ldcm];
    }
    // row checksums of tile row i: r(A_iJ)[pl, :] -= E * c(L_J)[:, ql]^T, k < J <= i
    for (int64_t J = k + 1 + threadIdx.x; J <= i; J += blockDim.x) {
      T* dst = rowchk + p + (2 * J) * r.ldr;
      const T* src = colchk + 2 * J + (k * nb + ql) * r.ldc;
      dst[0] -= e * src[0];
      dst[r.ldr] -= e * src[1];
      if (rowmag && colmag) rowmag[p + J * r.ldrm] += ae * colmag[J + (k * nb + ql) * r.ldcm];
    }
    if (threadIdx.x == 0) atomicAdd(&r.rep_counts[0], 1);
    __syncthreads();
  }
}

// LAPACK info of the whole factorization: first failing tile's local minor
// offset by the tile origin.
__global__ void accum_info_kernel(int32_t* tile_info, int32_t* total, int64_t offset) {
  if (*tile_info != 0 && *total == 0) *total = (int32_t)(*tile_info + offset);
  *tile_info = 0;
}
}  // namespace abft

// ----------------------------------------------------------------- driver --
struct ft_ctx {
  int device = 0;
  cudaStream_t stream = nullptr;
  void* state = nullptr;  // colchk | rowchk | colmag | rowmag
  size_t state_bytes = 0;
  int32_t* ints = nullptr;  // status | counts[8] | n_fixes | mark | info | rep[2]
  size_t ints_n = 0;
  abft_fix_t* fixlog = nullptr;
  int fixcap = 0;
  void* linv = nullptr;  // nb x nb inverse of the current L_kk
  size_t linv_bytes = 0;
  void* putmp = nullptr;  // n x nb panel scratch for the GEMM-based PU
  size_t putmp_bytes = 0;
};

extern "C" int ft_ctx_create(ft_ctx_t** ctx, int32_t device, abft_stream_t stream) {
  if (!ctx) return -1;
  ABFT_CUDA_TRY(cudaSetDevice(device));
  ft_ctx* c = new ft_ctx();
  c->device = device;
  c->stream = (cudaStream_t)stream;
  c->fixcap = 1 << 16;
  if (cudaMalloc(&c->fixlog, sizeof(abft_fix_t) * c->fixcap) != cudaSuccess) {
    delete c;
    return ABFT_E_NOMEM;
  }
  *ctx = c;
  return 0;
}

extern "C" int ft_ctx_destroy(ft_ctx_t* c) {
  if (!c) return -1;
  cudaSetDevice(c->device);
  if (c->state) cudaFree(c->state);
  if (c->ints) cudaFree(c->ints);
  if (c->fixlog) cudaFree(c->fixlog);
  if (c->linv) cudaFree(c->linv);
  if (c->putmp) cudaFree(c->putmp);
  delete c;
  return 0;
}

namespace {

struct Driver {
  ft_ctx* c;
  cudaStream_t s;
  int32_t dtype;
  int64_t n, nb, nt, lda;
  size_t es;
  void* A;
  const ft_opts_t* o;
  abft_mat_t M{};
  abft_report_t R{};
  abft_tol_t tol{};
  int32_t *status, *counts, *nfix, *mark, *info, *rep;
  std::vector<ft_inject_t> onchip_pending;
  int n_checks = 0;

  char* elem(int target, int64_t gi, int64_t gj) {
    if (target == 1) return (char*)M.colchk + (gi + gj * M.ldc) * es;
    if (target == 2) return (char*)M.rowchk + (gi + gj * M.ldr) * es;
    return (char*)A + (gi + gj * lda) * es;
  }
  // Elements the op after `point` overwrites: an on-chip flip there cannot be
  // changed back, so it stays (reading c-8).
  bool in_update_region(int point, int k, int64_t gi, int64_t gj) const {
    const int64_t r0 = k * nb, r1 = (k + 1) * nb;
    if (point == FT_AT_PRE_PD) return gi >= r0 && gi < r1 && gj >= r0 && gj < r1;
    if (point == FT_AT_PRE_PU) return gi >= r1 && gj >= r0 && gj < r1;
    if (point == FT_AT_PRE_TMU) return gi >= r1 && gj >= r1;
    return false;
  }
  int inject_at(int k, int point) {
    for (int t = 0; t < o->n_inject; ++t) {
      const ft_inject_t& f = o->inject[t];
      if (f.iter != k || f.point != point) continue;
      FT_TRY(abft_inject(elem(f.target, f.gi, f.gj), dtype, 0, f.xor_mask, (abft_stream_t)s));
      bool op_point = point == FT_AT_PRE_PD || point == FT_AT_PRE_PU || point == FT_AT_PRE_TMU;
      if (f.kind == FT_KIND_ONCHIP && op_point && f.target == 0 && !in_update_region(point, k, f.gi, f.gj))
        onchip_pending.push_back(f);
    }
    return 0;
  }
  // Fault-injection runs only: does the plan touch L_kk between the PD (which
  // produced the inverse the GEMM-based PU reads) and the PU?  Then the PU
  // must see the flipped L_kk, as an in-place TRSM would (reading c-8).
  bool lkk_touched_before_pu(int k) const {
    for (int t = 0; t < o->n_inject; ++t) {
      const ft_inject_t& f = o->inject[t];
      if (f.iter != k || f.target != 0) continue;
      if (f.point != FT_AT_PRE_PU_CHECK && f.point != FT_AT_PRE_PU) continue;
      if (f.gi >= k * nb && f.gi < (k + 1) * nb && f.gj >= k * nb && f.gj < (k + 1) * nb) return true;
    }
    return false;
  }
  int restore_onchip() {  // after the op: undo on-chip flips (the stored value was never wrong)
    for (auto& f : onchip_pending) FT_TRY(abft_inject(elem(f.target, f.gi, f.gj), dtype, 0, f.xor_mask, (abft_stream_t)s));
    onchip_pending.clear();
    return 0;
  }
  int check(int I0, int I1, int J0, int J1, int view, int which, bool lower_only = false) {
    abft_tiles_t t{I0, I1, J0, J1, lower_only ? 1 : 0, view};
    FT_TRY(abft_verify(&M, &t, which, &tol, &R, (abft_stream_t)s));
    FT_TRY(abft_locate_correct(&M, &t, which, &tol, &R, c->fixlog, c->fixcap, nfix, (abft_stream_t)s));
    ++n_checks;
    return 0;
  }
  void* colchk_at(int64_t r, int64_t col) { return (char*)M.colchk + (r + col * M.ldc) * es; }
  void* colmag_at(int64_t r, int64_t col) { return (char*)M.colmag + (r + col * M.ldcm) * es; }
  void* rowchk_at(int64_t r, int64_t col) { return (char*)M.rowchk + (r + col * M.ldr) * es; }
  void* rowmag_at(int64_t r, int64_t col) { return (char*)M.rowmag + (r + col * M.ldrm) * es; }
  void* a_at(int64_t r, int64_t col) { return (char*)A + (r + col * lda) * es; }
};

}  // namespace

extern "C" int ft_potrf(ft_ctx_t* c, int32_t dtype, int64_t n, void* dA, int64_t lda, const ft_opts_t* o,
                        ft_stats_t* stats, int64_t* info_out) {
  using namespace abft;
  if (!c) return -1;
  if (dtype != ABFT_F32 && dtype != ABFT_F64) return -2;
  if (!o) return -6;
  const int64_t nb = o->nb;
  if (n < 0 || nb < 32 || nb > 1024 || (nb & (nb - 1)) || n % nb) return -3;
  if (!dA) return -4;
  if (lda < std::max<int64_t>(1, n)) return -5;
  if (o->n_inject < 0 || (o->n_inject > 0 && !o->inject)) return -6;
  ABFT_CUDA_TRY(cudaSetDevice(c->device));
  Driver d;
  d.c = c;
  d.s = c->stream;
  d.dtype = dtype;
  d.n = n;
  d.nb = nb;
  d.nt = n / nb;
  d.lda = lda;
  d.es = dtype == ABFT_F64 ? 8 : 4;
  d.A = dA;
  d.o = o;
  const int64_t nt = d.nt;
  const bool ft = o->abft != 0;
  cudaStream_t s = d.s;
  // ---- state buffers (grown, never shrunk) ----
  size_t need = ft ? (size_t)(2 * nt * n + n * 2 * nt + nt * n + n * nt) * d.es : 0;
  if (c->state_bytes < need) {
    if (c->state) cudaFree(c->state);
    c->state = nullptr;
    c->state_bytes = 0;
    if (cudaMalloc(&c->state, need) != cudaSuccess) return ABFT_E_NOMEM;
    c->state_bytes = need;
  }
  size_t ints_need = (size_t)nt * nt + 8 + 1 + 1 + 1 + 2 + 4;
  if (c->ints_n < ints_need) {
    if (c->ints) cudaFree(c->ints);
    if (cudaMalloc(&c->ints, ints_need * sizeof(int32_t)) != cudaSuccess) return ABFT_E_NOMEM;
    c->ints_n = ints_need;
  }
  auto grow = [](void*& p, size_t& have, size_t need) -> int {
    if (have >= need) return 0;
    if (p) cudaFree(p);
    p = nullptr;
    have = 0;
    if (cudaMalloc(&p, need) != cudaSuccess) return ABFT_E_NOMEM;
    have = need;
    return 0;
  };
  FT_TRY(grow(c->linv, c->linv_bytes, (size_t)nb * nb * d.es));
  if (o->pu_gemm) FT_TRY(grow(c->putmp, c->putmp_bytes, (size_t)n * nb * d.es));
  d.status = c->ints;
  d.counts = d.status + nt * nt;
  d.nfix = d.counts + 8;
  d.mark = d.nfix + 1;
  d.info = d.mark + 1;
  d.rep = d.info + 1;
  ABFT_CUDA_TRY(cudaMemsetAsync(c->ints, 0, ints_need * sizeof(int32_t), s));
  char* st = (char*)c->state;
  d.M.dtype = dtype;
  d.M.m = n;
  d.M.n = n;
  d.M.nb = nb;
  d.M.A = dA;
  d.M.lda = lda;
  if (ft) {
    d.M.colchk = st;
    d.M.ldc = 2 * nt;
    st += 2 * nt * n * d.es;
    d.M.rowchk = st;
    d.M.ldr = n;
    st += n * 2 * nt * d.es;
    d.M.colmag = st;
    d.M.ldcm = nt;
    st += nt * n * d.es;
    d.M.rowmag = st;
    d.M.ldrm = n;
  }
  d.R.status = d.status;
  d.R.ld_status = nt;
  d.R.counts = d.counts;
  d.tol.kind = o->tol_kind;
  d.tol.scale = o->tol_scale > 0 ? o->tol_scale : 1.0;

  std::unique_lock<std::mutex> lk;
  auto t0 = std::chrono::steady_clock::now();
  const abft_stream_t as = (abft_stream_t)s;

  if (ft) {
    abft_tiles_t all{0, (int)nt, 0, (int)nt, 1, ABFT_SYM_LOWER};
    FT_TRY(abft_encode(&d.M, &all, ABFT_BOTH, as));
  }
  for (int k = 0; k < nt; ++k) {
    const int64_t r1 = (k + 1) * nb;  // first row/col after the panel
    const int64_t nk = n - r1;        // trailing size
    const int m2 = (int)(2 * (nt - k - 1));
    // Alg. 2 lines 3-4: check the panel to be decomposed (diag tile, SYM view, both)
    FT_TRY(d.inject_at(k, FT_AT_PRE_PD_CHECK));
    if (ft) FT_TRY(d.check(k, k + 1, k, k + 1, ABFT_SYM_LOWER, ABFT_BOTH));
    // line 5: PD (+ checksum rule c-12)
    FT_TRY(d.inject_at(k, FT_AT_PRE_PD));
    {
      abft_mat_t D{};
      D.dtype = dtype;
      D.m = D.n = D.nb = nb;
      D.A = d.a_at(k * nb, k * nb);
      D.lda = lda;
      if (ft) {
        D.colchk = d.colchk_at(2 * k, k * nb);
        D.ldc = d.M.ldc;
        D.colmag = d.colmag_at(k, k * nb);
        D.ldcm = d.M.ldcm;
      }
      const bool need_inv = ft || o->pu_gemm;
      FT_TRY(abft_panel_potrf(&D, need_inv ? c->linv : nullptr, nb, d.info, as));
      accum_info_kernel<<<1, 1, 0, s>>>(d.info, d.rep + 2, (int64_t)k * nb);
    }
    FT_TRY(d.restore_onchip());
    FT_TRY(d.inject_at(k, FT_AT_POST_PD));
    // line 7: check the decomposed panel (LOWER view, c only; c-24)
    if (ft) FT_TRY(d.check(k, k + 1, k, k + 1, ABFT_LOWER, ABFT_COL));
    if (k == nt - 1) break;
    // line 8: check the panel to be updated (both checksums)
    FT_TRY(d.inject_at(k, FT_AT_PRE_PU_CHECK));
    if (ft) FT_TRY(d.check(k + 1, (int)nt, k, k + 1, ABFT_GENERAL, ABFT_BOTH));
    // line 9: PU  L_ik = A_ik L_kk^-T  (+ c(L_ik) = c(A_ik) L_kk^-T, c-12)
    FT_TRY(d.inject_at(k, FT_AT_PRE_PU));
    const bool refresh_inv = o->pu_gemm && d.lkk_touched_before_pu(k);
    if (refresh_inv) FT_TRY(abft_tri_inverse(dtype, 'L', 'N', nb, d.a_at(k * nb, k * nb), lda, c->linv, nb, as));
    {
      cublasHandle_t h = blas_handle(s, lk);
      if (o->pu_gemm) {
        // L21 = A21 L_kk^-T as a DGEMM with the explicit inverse (tensor cores),
        // written to scratch and copied back
        if (dtype == ABFT_F64) {
          const double one = 1.0, zero = 0.0;
          if (cublasDgemm(h, CUBLAS_OP_N, CUBLAS_OP_T, (int)nk, (int)nb, (int)nb, &one, (const double*)d.a_at(r1, k * nb),
                          (int)lda, (const double*)c->linv, (int)nb, &zero, (double*)c->putmp, (int)nk) !=
              CUBLAS_STATUS_SUCCESS)
            return ABFT_E_CUBLAS;
        } else {
          const float one = 1.0f, zero = 0.0f;
          if (cublasSgemm(h, CUBLAS_OP_N, CUBLAS_OP_T, (int)nk, (int)nb, (int)nb, &one, (const float*)d.a_at(r1, k * nb),
                          (int)lda, (const float*)c->linv, (int)nb, &zero, (float*)c->putmp, (int)nk) !=
              CUBLAS_STATUS_SUCCESS)
            return ABFT_E_CUBLAS;
        }
        lk.unlock();
        ABFT_CUDA_TRY(cudaMemcpy2DAsync(d.a_at(r1, k * nb), lda * d.es, c->putmp, nk * d.es, nk * d.es, nb,
                                        cudaMemcpyDeviceToDevice, s));
      } else if (dtype == ABFT_F64) {
        const double one = 1.0;
        if (cublasDtrsm(h, CUBLAS_SIDE_RIGHT, CUBLAS_FILL_MODE_LOWER, CUBLAS_OP_T, CUBLAS_DIAG_NON_UNIT, (int)nk,
                        (int)nb, &one, (const double*)d.a_at(k * nb, k * nb), (int)lda, (double*)d.a_at(r1, k * nb),
                        (int)lda) != CUBLAS_STATUS_SUCCESS)
          return ABFT_E_CUBLAS;
      } else {
        const float one = 1.0f;
        if (cublasStrsm(h, CUBLAS_SIDE_RIGHT, CUBLAS_FILL_MODE_LOWER, CUBLAS_OP_T, CUBLAS_DIAG_NON_UNIT, (int)nk,
                        (int)nb, &one, (const float*)d.a_at(k * nb, k * nb), (int)lda, (float*)d.a_at(r1, k * nb),
                        (int)lda) != CUBLAS_STATUS_SUCCESS)
          return ABFT_E_CUBLAS;
      }
      if (lk.owns_lock()) lk.unlock();
    }
    FT_TRY(d.restore_onchip());  // on-chip flips hit the data step only (c-8)
    if (refresh_inv) FT_TRY(abft_tri_inverse(dtype, 'L', 'N', nb, d.a_at(k * nb, k * nb), lda, c->linv, nb, as));
    if (ft)  // c(L_ik) = c(A_ik) L_kk^-T, m_c <- m_c |L_kk^-T| with the PD's inverse (c-12, c-6)
      FT_TRY(abft_update_trsm_inv(dtype, 'R', 'T', nb, c->linv, nb, d.colchk_at(2 * (k + 1), k * nb), d.M.ldc, m2,
                                  d.colmag_at(k + 1, k * nb), d.M.ldcm, m2 / 2, as));
    FT_TRY(d.inject_at(k, FT_AT_POST_PU));
    // line 10: check the updated panel (c only; 1D_ROW fixable, 2D -> restart, L434)
    if (ft) FT_TRY(d.check(k + 1, (int)nt, k, k + 1, ABFT_GENERAL, ABFT_COL));
    // line 12: TMU  A22 -= L21 L21^T (DSYRK on tensor cores) + checksum rules c-12
    FT_TRY(d.inject_at(k, FT_AT_PRE_TMU));
    {
      cublasHandle_t h = blas_handle(s, lk);
      if (dtype == ABFT_F64) {
        const double m1 = -1.0, one = 1.0;
        if (cublasDsyrk(h, CUBLAS_FILL_MODE_LOWER, CUBLAS_OP_N, (int)nk, (int)nb, &m1, (const double*)d.a_at(r1, k * nb),
                        (int)lda, &one, (double*)d.a_at(r1, r1), (int)lda) != CUBLAS_STATUS_SUCCESS)
          return ABFT_E_CUBLAS;
      } else {
        const float m1 = -1.0f, one = 1.0f;
        if (cublasSsyrk(h, CUBLAS_FILL_MODE_LOWER, CUBLAS_OP_N, (int)nk, (int)nb, &m1, (const float*)d.a_at(r1, k * nb),
                        (int)lda, &one, (float*)d.a_at(r1, r1), (int)lda) != CUBLAS_STATUS_SUCCESS)
          return ABFT_E_CUBLAS;
      }
      lk.unlock();
    }
    FT_TRY(d.restore_onchip());  // on-chip flips hit the data step only (c-8)
    if (ft) {
      // c(A_ij) -= c(L_ik) L_jk^T and r(A_ij) -= L_ik c(L_jk)^T from one product (c-12, L189)
      FT_TRY(abft_update_syrk(dtype, nb, nt - k - 1, d.a_at(r1, k * nb), lda, d.colchk_at(2 * (k + 1), k * nb), d.M.ldc,
                              d.colmag_at(k + 1, k * nb), d.M.ldcm, d.colchk_at(2 * (k + 1), r1),
                              d.rowchk_at(r1, 2 * (k + 1)), d.M.ldr, d.colmag_at(k + 1, r1), d.rowmag_at(r1, k + 1),
                              d.M.ldrm, as));
    }
    FT_TRY(d.inject_at(k, FT_AT_POST_TMU));
    // line 13: heuristic panel re-check for the TMU (Fig. 4a) + guarded repair (c-25)
    if (ft) {
      ABFT_CUDA_TRY(cudaMemcpyAsync(d.mark, d.nfix, sizeof(int32_t), cudaMemcpyDeviceToDevice, s));
      FT_TRY(d.check(k + 1, (int)nt, k, k + 1, ABFT_GENERAL, ABFT_COL));
      if (o->fig4a_repair) {
        RepairArgs ra{};
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
        if (dtype == ABFT_F64)
          fig4a_repair_kernel<double><<<1, 256, 0, s>>>(ra);
        else
          fig4a_repair_kernel<float><<<1, 256, 0, s>>>(ra);
        ABFT_CUDA_TRY(cudaGetLastError());
      }
    }
  }
  // ---- the single host synchronisation: stats ----
  int32_t host_ints[8 + 1 + 1 + 1 + 2 + 1];
  ABFT_CUDA_TRY(cudaMemcpyAsync(host_ints, d.counts, sizeof(host_ints), cudaMemcpyDeviceToHost, s));
  if (o->fix_log && o->fix_log_cap > 0)
    ABFT_CUDA_TRY(cudaMemcpyAsync(o->fix_log, c->fixlog, sizeof(abft_fix_t) * std::min(o->fix_log_cap, c->fixcap),
                                  cudaMemcpyDeviceToDevice, s));
  ABFT_CUDA_TRY(cudaStreamSynchronize(s));
  auto t1 = std::chrono::steady_clock::now();
  if (info_out) *info_out = host_ints[13];
  if (stats) {
    for (int i = 0; i < 8; ++i) stats->counts[i] = host_ints[i];
    stats->n_fixes = host_ints[8];
    stats->repairs_applied = host_ints[11];
    stats->repairs_skipped = host_ints[12];
    stats->uncorrectable = host_ints[ABFT_CNT_UNCORRECTABLE];
    stats->n_checks = d.n_checks;
    stats->ms_total = std::chrono::duration<double, std::milli>(t1 - t0).count();
  }
  return host_ints[ABFT_CNT_UNCORRECTABLE] ? ABFT_E_UNCORRECTABLE : 0;
}
