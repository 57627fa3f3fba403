// ft_potrf.cu — PD checksum rule for Cholesky (a4) and the fault-tolerant
// Cholesky driver in the paper's reordered checking scheme (a7).
//
// Paper: Table II / §IV.A (L152-L189) full-checksum Cholesky; Alg. 2
// (L364-L379) checking order; heuristic TMU checking Fig. 4a (L357-L359);
// PD on the CPU in MAGMA (L61) — here the PD runs on the device (cuSOLVER),
// DESIGN.md §7 explains why.  Readings: c-12 (Cholesky rules), c-24 (views
// before/after PD), c-25 (guarded Fig. 4a trailing repair), c-8 (fault hooks).
#include <dlfcn.h>

#include <initializer_list>
#include <tuple>

#include "ft_driver.cuh"

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

namespace abft {
// The device part of the PD after the factorization (c-12): L_kk^-1 and the
// checksum rule.  Shared by abft_panel_potrf and the FT_PD_HOST driver path.
int panel_potrf_rules(const abft_mat_t* d, void* Linv, int64_t ldw, abft_stream_t stream);
}  // namespace abft

extern "C" int abft_panel_potrf(const abft_mat_t* d, void* Linv, int64_t ldw, int32_t* info, abft_stream_t stream) {
  if (!d || d->m != d->nb || d->n != d->nb || !d->A || d->lda < d->nb) return -1;
  if (Linv && ldw < d->nb) return -3;
  if (!info) return -4;
  if (d->dtype != ABFT_F32 && d->dtype != ABFT_F64) return -1;
  cudaStream_t s = (cudaStream_t)stream;
  int rc = d->dtype == ABFT_F64 ? abft::potrf_tile<double>(d, info, s) : abft::potrf_tile<float>(d, info, s);
  if (rc) return rc;
  return abft::panel_potrf_rules(d, Linv, ldw, stream);
}

int abft::panel_potrf_rules(const abft_mat_t* d, void* Linv, int64_t ldw, abft_stream_t stream) {
  cudaStream_t s = (cudaStream_t)stream;
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
  int64_t c0, c1;       // trailing columns to repair (look-ahead, reading c-35); [0, n) = all
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
    // data: row p left of the diagonal, column p below it, and (p, p) —
    // restricted to the columns [c0, c1) whose update consumed the bad value
    const bool pin = p >= r.c0 && p < r.c1;
    const int64_t b0 = row0 > r.c0 ? row0 : r.c0, b1 = p < r.c1 ? p : r.c1;
    for (int64_t b = b0 + threadIdx.x; b < b1; b += blockDim.x) A[p + b * r.lda] -= e * A[b + q * r.lda];
    if (pin) {
      for (int64_t a = p + 1 + threadIdx.x; a < r.n; a += blockDim.x) A[a + p * r.lda] -= e * A[a + q * r.lda];
      if (threadIdx.x == 0) A[p + p * r.lda] -= 2 * e * A[p + q * r.lda] - e * e;
    }
    // column checksums of tile column i: c(A_Ii)[:, pl] -= E * c(L_I)[:, ql], I >= i
    for (int64_t I = i + threadIdx.x; pin && I < nt; I += blockDim.x) {
      T* dst = colchk + 2 * I + (i * nb + pl) * r.ldc;
      const T* src = colchk + 2 * I + (k * nb + ql) * r.ldc;
      dst[0] -= e * src[0];
      dst[1] -= e * src[1];
      if (colmag) colmag[I + (i * nb + pl) * r.ldcm] += ae * colmag[I + (k * nb + ql) * r.ldcm];
    }
    // row checksums of tile row i: r(A_iJ)[pl, :] -= E * c(L_J)[:, ql]^T, k < J <= i
    for (int64_t J = k + 1 + threadIdx.x; J <= i; J += blockDim.x) {
      if (J * nb < r.c0 || J * nb >= r.c1) continue;
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

}  // namespace abft

// ----------------------------------------------------------------- driver --
namespace abft {
__global__ void add_i32_kernel(int32_t* p, int32_t v) { *p += v; }
}  // namespace abft

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
  if (cudaHostAlloc((void**)&c->hpin, 16 * sizeof(int32_t), cudaHostAllocMapped) != cudaSuccess ||
      cudaHostGetDevicePointer((void**)&c->hpin_dev, c->hpin, 0) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev, cudaEventDisableTiming) != cudaSuccess) {
    cudaFree(c->fixlog);
    if (c->hpin) cudaFreeHost(c->hpin);
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
  if (c->uinv) cudaFree(c->uinv);
  if (c->putmp) cudaFree(c->putmp);
  if (c->aux) cudaFree(c->aux);
  if (c->rsv) cudaFree(c->rsv);
  if (c->hpin) cudaFreeHost(c->hpin);
  if (c->ev) cudaEventDestroy(c->ev);
  if (c->join) cudaEventDestroy(c->join);
  for (cudaEvent_t e : c->evpool) cudaEventDestroy(e);
  if (c->ev_col) cudaEventDestroy(c->ev_col);
  if (c->ev_side) cudaEventDestroy(c->ev_side);
  if (c->ev_rule) cudaEventDestroy(c->ev_rule);
  if (c->rule) {
    cudaStreamSynchronize(c->rule);
    abft::release_stream_handles(c->rule);
    abft::release_stream_pools(c->rule);
    cudaStreamDestroy(c->rule);
  }
  if (c->putmp2) cudaFree(c->putmp2);
  if (c->side) {
    cudaStreamSynchronize(c->side);
    abft::release_stream_handles(c->side);
    abft::release_stream_pools(c->side);
    cudaStreamDestroy(c->side);
  }
  if (c->drv) {
    // the library keeps cuBLAS / cuSOLVER handles, scratch and pass pools per
    // stream: release the private stream's before the stream goes away
    cudaStreamSynchronize(c->drv);
    abft::release_stream_handles(c->drv);
    abft::release_stream_pools(c->drv);
    cudaStreamDestroy(c->drv);
  }
  if (c->hstage) cudaFreeHost(c->hstage);
  if (c->dguard) cudaFree(c->dguard);
  for (cudaEvent_t e : c->hchunk)
    if (e) cudaEventDestroy(e);
  if (c->lapack) dlclose(c->lapack);
  delete c;
  return 0;
}

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
  if (o->scheme < FT_SCHEME_NEW || o->scheme > FT_SCHEME_SINGLE_PRE) return -6;
  // checking scheme (reading c-34): which checks run, and on which checksums
  const int scheme = o->scheme;
  const bool s_new = scheme == FT_SCHEME_NEW;
  const bool single = scheme == FT_SCHEME_SINGLE_POST || scheme == FT_SCHEME_SINGLE_PRE;
  const bool pre_checks = s_new || scheme == FT_SCHEME_SINGLE_PRE;  // PD / PU inputs
  const bool post_checks = scheme != FT_SCHEME_SINGLE_PRE;          // PD / PU outputs
  const int W = single ? ABFT_COL : ABFT_BOTH;
  ABFT_CUDA_TRY(cudaSetDevice(c->device));
  Driver d;
  FT_TRY(d.setup(c, dtype, n, nb, dA, lda, o, /*lu=*/false));
  const int64_t nt = d.nt;
  const bool ft = o->abft != 0;
  std::unique_lock<std::mutex> lk;
  auto t0 = std::chrono::steady_clock::now();
  // Look-ahead (reading c-35): the next panel's PD / PU on the side stream
  // next to the rest of the TMU; the new scheme (or the unprotected driver).
  const bool la_on = o->lookahead && (!ft || s_new);
  if (la_on) FT_TRY(d.side_setup());
  // the same predicate as oracle/drivers.py::lookahead_ok: the split must not
  // move a fault hook relative to Alg. 2 (c-8)
  auto la_at = [&](int k) -> bool {
    if (k + 1 >= nt) return false;
    // the periodic trailing check of iteration k covers tile column k+1 too
    if (ft && o->trailing_check_period > 0 && (k + 1) % o->trailing_check_period == 0) return false;
    const int64_t c0 = (int64_t)(k + 1) * nb, c1 = c0 + nb;
    for (int t = 0; t < o->n_inject; ++t) {
      const ft_inject_t& f = o->inject[t];
      if (f.iter == k && (f.point == FT_AT_PRE_TMU || f.point == FT_AT_POST_TMU)) return false;
      if (f.iter == k + 1 && (f.point <= FT_AT_POST_PU || f.point == FT_AT_D2H || f.point == FT_AT_H2D)) {
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
    abft_tiles_t all{0, (int)nt, 0, (int)nt, 1, ABFT_SYM_LOWER};
    FT_TRY(abft_encode(&d.M, &all, W, (abft_stream_t)d.s));
  }
  // Local restart (f1, L430): the PD input tile and the PU input panel are
  // copied (with their checksums) right after their pre-op checks; a 2D
  // error left by the post-op check restores the copy and redoes the op.
  const bool rs = ft && o->restart && post_checks;

  // ---- Alg. 2 lines 3-10 of iteration k: PD and PU with their checks, on d.s
  // (the main stream, or the side stream under look-ahead).  fig4b_here: the
  // Fig. 4b trailing check before the PU (under look-ahead the main stream
  // runs it after the side stream joins: it reads only the trailing matrix).
  auto chain = [&](int k, bool fig4b_here) -> int {
    cudaStream_t s = d.s;
    const abft_stream_t as = (abft_stream_t)s;
    const int64_t r0 = (int64_t)k * nb;
    const int64_t r1 = r0 + nb;   // first row/col after the panel
    const int64_t nk = n - r1;    // trailing size
    const int m2 = (int)(2 * (nt - k - 1));
    if (ft) FT_TRY(d.begin_iteration());
    char* rbuf = (char*)c->rsv;
    auto copy2d = [&](void* dst, int64_t ldd, const void* src, int64_t lds, int64_t rows, int64_t cols) -> int {
      if (rows <= 0 || cols <= 0) return 0;
      FT_TRY(abft::copy2d(dst, ldd * d.es, src, lds * d.es, rows * d.es, cols, s));
      return 0;
    };
    // pd copy: A_kk (nb x nb) | c(A_kk) (2 x nb) | m_c (1 x nb);  pu copy: A21 | c(A21) | m_c(A21)
    char* pd_a = rbuf;
    char* pd_c = pd_a + (size_t)nb * nb * d.es;
    char* pd_m = pd_c + (size_t)2 * nb * d.es;
    char* pu_a = pd_m + (size_t)nb * d.es;
    char* pu_c = pu_a + (size_t)nk * nb * d.es;
    char* pu_m = pu_c + (size_t)m2 * nb * d.es;
    // several restart copies as one launch: (dst, ldd, src, lds, rows, cols) in elements
    auto copies = [&](std::initializer_list<std::tuple<void*, int64_t, const void*, int64_t, int64_t, int64_t>> l) {
      Copy2D cs[4];
      int n = 0;
      for (const auto& t : l)
        cs[n++] = Copy2D{std::get<0>(t), (size_t)std::get<1>(t) * d.es, std::get<2>(t), (size_t)std::get<3>(t) * d.es,
                         (size_t)std::get<4>(t) * d.es, (size_t)std::get<5>(t)};
      return copy2d_multi(cs, n, s);
    };
    // PD restart decision: snapshot the uncorrectable count before the check,
    // read the difference back into pinned memory after it (one event)
    auto post_readback = [&]() -> int { return d.post_delta(0); };
    auto readback_delta = [&](int* delta) -> int { return d.wait_delta(0, delta); };
    // Alg. 2 lines 3-4: check the panel to be decomposed (diag tile, SYM view,
    // both); with local restart the check's pass also leaves the PD input's
    // copy (f1, L430) in pd_a
    FT_TRY(d.inject_at(k, FT_AT_PRE_PD_CHECK));
    const bool ck_pd = rs && pre_checks;
    if (ft && pre_checks)
      FT_TRY(d.check(k, k + 1, k, k + 1, ABFT_SYM_LOWER, W, false, nullptr, ck_pd ? pd_a : nullptr, nb));
    if (rs) {
      PhaseScope ps(d, FT_PH_RESTART);
      if (!ck_pd) FT_TRY(copy2d(pd_a, nb, d.a_at(r0, r0), lda, nb, nb));
      FT_TRY(copies({{pd_c, 2, d.colchk_at(2 * k, r0), d.M.ldc, 2, nb}, {pd_m, 1, d.colmag_at(k, r0), d.M.ldcm, 1, nb}}));
    }
    auto do_pd = [&]() -> int {
      PhaseScope ps(d, FT_PH_PD);
      abft_mat_t D{};
      D.dtype = dtype;
      D.m = D.n = D.nb = nb;
      D.A = d.a_at(r0, r0);
      D.lda = lda;
      if (ft && !(Driver::diag_skip() & 8)) {
        D.colchk = d.colchk_at(2 * k, r0);
        D.ldc = d.M.ldc;
        D.colmag = d.colmag_at(k, r0);
        D.ldcm = d.M.ldcm;
      }
      const bool need_inv = ft || o->pu_gemm;
      if (o->pd_location == FT_PD_HOST) {  // Alg. 2 lines 3-7 with the PD on the host (c-28)
        FT_TRY(host_panel_pd(d, k, HOST_POTRF, r0, r0, nb, nullptr, nullptr, d.info));
        FT_TRY(panel_potrf_rules(&D, need_inv ? c->linv : nullptr, nb, as));
      } else {
        FT_TRY(abft_panel_potrf(&D, need_inv ? c->linv : nullptr, nb, d.info, as));
      }
      accum_info_kernel<<<1, 1, 0, s>>>(d.info, d.info_total, r0);
      return 0;
    };
    // line 5: PD (+ checksum rule c-12)
    FT_TRY(d.inject_at(k, FT_AT_PRE_PD));
    FT_TRY(do_pd());
    FT_TRY(d.restore_onchip());
    FT_TRY(d.inject_at(k, FT_AT_POST_PD));
    // line 7: check the decomposed panel (LOWER view, c only; c-24)
    if (ft && post_checks) {
      if (rs) ABFT_CUDA_TRY(cudaMemcpyAsync(d.snap, d.counts + ABFT_CNT_UNCORRECTABLE, 4, cudaMemcpyDeviceToDevice, s));
      FT_TRY(d.check(k, k + 1, k, k + 1, ABFT_LOWER, ABFT_COL));
      if (rs) FT_TRY(post_readback());
    }
    // The PD restart decision is taken after the pre-PU check has been queued
    // (that check reads only the panel below A_kk), so the host waits while the
    // device works.  Not when the fault plan injects at the pre-PU-check point:
    // then the paper's order is kept exactly.
    const bool defer_pd = rs && k < nt - 1 && !d.has_inject(k, FT_AT_PRE_PU_CHECK);
    auto pd_restart = [&]() -> int {
      int delta = 0;
      FT_TRY(readback_delta(&delta));
      if (delta <= 0) return 0;
      ++d.restarts;
      add_i32_kernel<<<1, 1, 0, s>>>(d.counts + ABFT_CNT_UNCORRECTABLE, -delta);
      FT_TRY(copies({{d.a_at(r0, r0), lda, pd_a, nb, nb, nb},
                     {d.colchk_at(2 * k, r0), d.M.ldc, pd_c, 2, 2, nb},
                     {d.colmag_at(k, r0), d.M.ldcm, pd_m, 1, 1, nb}}));
      FT_TRY(do_pd());
      return d.check(k, k + 1, k, k + 1, ABFT_LOWER, ABFT_COL);
    };
    if (rs && !defer_pd) FT_TRY(pd_restart());
    if (k == nt - 1) return 0;
    // line 8: check the panel to be updated (both checksums)
    FT_TRY(d.inject_at(k, FT_AT_PRE_PU_CHECK));
    const bool ck_pu = rs && pre_checks;  // the check's pass leaves the PU input's copy in pu_a
    if (ft && pre_checks)
      FT_TRY(d.check(k + 1, (int)nt, k, k + 1, ABFT_GENERAL, W, false, nullptr, ck_pu ? pu_a : nullptr, nk));
    if (rs) {
      PhaseScope ps(d, FT_PH_RESTART);
      if (!ck_pu) FT_TRY(copy2d(pu_a, nk, d.a_at(r1, r0), lda, nk, nb));
      FT_TRY(copies({{pu_c, m2, d.colchk_at(2 * (k + 1), r0), d.M.ldc, m2, nb},
                     {pu_m, m2 / 2, d.colmag_at(k + 1, r0), d.M.ldcm, m2 / 2, nb}}));
    }
    if (defer_pd) FT_TRY(pd_restart());
    // Fig. 4b (L359): a 1D pattern fixed by this iteration's pre-PD / pre-PU
    // checks is the trace of an on-chip fault in the last TMU: check the
    // whole trailing matrix now (gated on the device)
    if (ft && s_new && fig4b_here)
      FT_TRY(d.fig4b_check(k + 1, (int)nt, k + 1, (int)nt, ABFT_SYM_LOWER, ABFT_BOTH, true));
    if (ft && s_new && !fig4b_here) FT_TRY(d.mark_fig4b_end());  // the deferred check's window ends here
    // line 9: PU  L_ik = A_ik L_kk^-T  (+ c(L_ik) = c(A_ik) L_kk^-T, c-12)
    auto pu_data = [&]() -> int {
      PhaseScope ps(d, FT_PH_PU);
      cublasHandle_t h = blas_handle(s, lk);
      if (o->pu_gemm) {
        // L21 = A21 L_kk^-T as a DGEMM with the explicit inverse (tensor cores).
        // The GEMM cannot run in place: it reads the local-restart copy of A21
        // when there is one (no fault plan: the copy equals A21) and writes
        // A21 directly, else it writes scratch that is copied back.
        const bool from_copy = rs && o->n_inject == 0;
        const void* src = from_copy ? (const void*)pu_a : d.a_at(r1, r0);
        const int lds = from_copy ? (int)nk : (int)lda;
        void* dst = from_copy ? d.a_at(r1, r0) : c->putmp;
        const int ldd = from_copy ? (int)lda : (int)nk;
        cublasStatus_t st;
        if (dtype == ABFT_F64) {
          const double one = 1.0, zero = 0.0;
          st = cublasDgemm(h, CUBLAS_OP_N, CUBLAS_OP_T, (int)nk, (int)nb, (int)nb, &one, (const double*)src, lds,
                           (const double*)c->linv, (int)nb, &zero, (double*)dst, ldd);
        } else {
          const float one = 1.0f, zero = 0.0f;
          st = cublasSgemm(h, CUBLAS_OP_N, CUBLAS_OP_T, (int)nk, (int)nb, (int)nb, &one, (const float*)src, lds,
                           (const float*)c->linv, (int)nb, &zero, (float*)dst, ldd);
        }
        lk.unlock();
        if (st != CUBLAS_STATUS_SUCCESS) return ABFT_E_CUBLAS;
        if (!from_copy) FT_TRY(abft::copy2d(d.a_at(r1, r0), lda * d.es, c->putmp, nk * d.es, nk * d.es, nb, s));
      } else {
        cublasStatus_t st;
        if (dtype == ABFT_F64) {
          const double one = 1.0;
          st = cublasDtrsm(h, CUBLAS_SIDE_RIGHT, CUBLAS_FILL_MODE_LOWER, CUBLAS_OP_T, CUBLAS_DIAG_NON_UNIT, (int)nk,
                           (int)nb, &one, (const double*)d.a_at(r0, r0), (int)lda, (double*)d.a_at(r1, r0), (int)lda);
        } else {
          const float one = 1.0f;
          st = cublasStrsm(h, CUBLAS_SIDE_RIGHT, CUBLAS_FILL_MODE_LOWER, CUBLAS_OP_T, CUBLAS_DIAG_NON_UNIT, (int)nk,
                           (int)nb, &one, (const float*)d.a_at(r0, r0), (int)lda, (float*)d.a_at(r1, r0), (int)lda);
        }
        lk.unlock();
        if (st != CUBLAS_STATUS_SUCCESS) return ABFT_E_CUBLAS;
      }
      return 0;
    };
    auto pu_chk = [&]() -> int {  // c(L_ik) = c(A_ik) L_kk^-T, m_c <- m_c |L_kk^-T| with the PD's inverse (c-12, c-6)
      PhaseScope ps(d, FT_PH_RULES);
      if (Driver::diag_skip() & 8) return 0;
      return abft_update_trsm_inv(dtype, 'R', 'T', nb, c->linv, nb, d.colchk_at(2 * (k + 1), r0), d.M.ldc, m2,
                                  d.colmag_at(k + 1, r0), d.M.ldcm, m2 / 2, as);
    };
    FT_TRY(d.inject_at(k, FT_AT_PRE_PU));
    const bool refresh_inv = o->pu_gemm && d.diag_touched_before_pu(k);
    if (refresh_inv) FT_TRY(abft_tri_inverse(dtype, 'L', 'N', nb, d.a_at(r0, r0), lda, c->linv, nb, as));
    FT_TRY(pu_data());
    FT_TRY(d.restore_onchip());  // on-chip flips hit the data step only (c-8)
    if (refresh_inv) FT_TRY(abft_tri_inverse(dtype, 'L', 'N', nb, d.a_at(r0, r0), lda, c->linv, nb, as));
    if (ft) FT_TRY(pu_chk());
    FT_TRY(d.inject_at(k, FT_AT_POST_PU));
    // line 10: check the updated panel (c only; 1D_ROW fixable, 2D -> restart, L434)
    if (ft && post_checks) {
      if (rs) ABFT_CUDA_TRY(cudaMemcpyAsync(d.snap, d.counts + ABFT_CNT_UNCORRECTABLE, 4, cudaMemcpyDeviceToDevice, s));
      FT_TRY(d.check(k + 1, (int)nt, k, k + 1, ABFT_GENERAL, ABFT_COL));
      // 2D after the PU: local restart from the pre-PU copy (L430), decided on
      // the device (Driver::gated_restart): restore-and-redo as one gated
      // GEMM per array, reading the copy and the PD's inverse, then re-check.
      auto pu_redo = [&](const int32_t* g) -> int {
        {
          PhaseScope ps(d, FT_PH_RESTART);
          // data, checksum and magnitude products as one gated launch
          const GatedGemm gg[3] = {{nk, nb, nb, pu_a, nk, c->linv, nb, d.a_at(r1, r0), lda, 0, 1, 0, 0},
                                   {m2, nb, nb, pu_c, m2, c->linv, nb, d.colchk_at(2 * (k + 1), r0), d.M.ldc, 0, 1, 0, 0},
                                   {m2 / 2, nb, nb, pu_m, m2 / 2, c->linv, nb, d.colmag_at(k + 1, r0), d.M.ldcm, 0, 1,
                                    0, 1}};
          FT_TRY(gemm_gated_multi(dtype, gg, 3, g, s));
        }
        return d.check(k + 1, (int)nt, k, k + 1, ABFT_GENERAL, ABFT_COL);
      };
      if (rs) FT_TRY(d.gated_restart(1, pu_redo));
    }
    return 0;
  };

  // ---- TMU data step on trailing columns [c0, c1) (tile aligned, c1 = n or
  // c0 + nb): the lower part of A[c0:n, c0:c1] -= L21 L21[c0-r1 .. c1-r1]^T
  auto tmu_data = [&](int k, int64_t c0, int64_t c1) -> int {
    const int64_t r0 = (int64_t)k * nb, w = c1 - c0, below = n - c1;
    if (w <= 0) return 0;
    PhaseScope ps(d, FT_PH_TMU);
    cublasHandle_t h = blas_handle(d.s, lk);
    cublasStatus_t st = CUBLAS_STATUS_SUCCESS;
    if (dtype == ABFT_F64) {
      const double m1 = -1.0, one = 1.0;
      st = cublasDsyrk(h, CUBLAS_FILL_MODE_LOWER, CUBLAS_OP_N, (int)w, (int)nb, &m1, (const double*)d.a_at(c0, r0),
                       (int)lda, &one, (double*)d.a_at(c0, c0), (int)lda);
      if (st == CUBLAS_STATUS_SUCCESS && below > 0)
        st = cublasDgemm(h, CUBLAS_OP_N, CUBLAS_OP_T, (int)below, (int)w, (int)nb, &m1, (const double*)d.a_at(c1, r0),
                         (int)lda, (const double*)d.a_at(c0, r0), (int)lda, &one, (double*)d.a_at(c1, c0), (int)lda);
    } else {
      const float m1 = -1.0f, one = 1.0f;
      st = cublasSsyrk(h, CUBLAS_FILL_MODE_LOWER, CUBLAS_OP_N, (int)w, (int)nb, &m1, (const float*)d.a_at(c0, r0),
                       (int)lda, &one, (float*)d.a_at(c0, c0), (int)lda);
      if (st == CUBLAS_STATUS_SUCCESS && below > 0)
        st = cublasSgemm(h, CUBLAS_OP_N, CUBLAS_OP_T, (int)below, (int)w, (int)nb, &m1, (const float*)d.a_at(c1, r0),
                         (int)lda, (const float*)d.a_at(c0, r0), (int)lda, &one, (float*)d.a_at(c1, c0), (int)lda);
    }
    lk.unlock();
    return st == CUBLAS_STATUS_SUCCESS ? 0 : ABFT_E_CUBLAS;
  };
  // ---- TMU checksum rules (c-12, L189) for trailing tile columns [c0, c1)
  auto tmu_chk = [&](int k, int64_t c0, int64_t c1) -> int {
    const int64_t r0 = (int64_t)k * nb;
    const abft_stream_t as = (abft_stream_t)d.s;
    const int J0 = (int)(c0 / nb), J1 = (int)(c1 / nb);
    if (J1 <= J0 || (Driver::diag_skip() & 4)) return 0;
    PhaseScope ps(d, FT_PH_RULES);
    if (c1 == n) {  // tile columns J0.. (to the end): the one-product rule of the sub-problem
      const int64_t ntk = nt - J0;
      return abft_update_syrk(dtype, nb, ntk, d.a_at(c0, r0), lda, d.colchk_at(2 * J0, r0), d.M.ldc,
                              d.colmag_at(J0, r0), d.M.ldcm, d.colchk_at(2 * J0, c0),
                              single ? nullptr : d.rowchk_at(c0, 2 * J0), d.M.ldr, d.colmag_at(J0, c0),
                              single ? nullptr : d.rowmag_at(c0, J0), d.M.ldrm, as);
    }
    // one tile column J0 (look-ahead's first part): every tile I >= J0 of it
    //   c(A_I,J0) -= c(L_Ik) L_J0,k^T,  m_c += m_c(L_Ik) |L_J0,k|^T
    //   r(A_I,J0) -= L_Ik c(L_J0,k)^T,  m_r += |L_Ik| m_c(L_J0,k)^T
    const int64_t m2 = 2 * (nt - J0);
    int rc = ABFT_E_UNSUPPORTED;
    if (dtype == ABFT_F64)  // the DMMA rule kernel restricted to this tile column (abft_rule_dmma.cu)
      rc = update_syrk_dmma(nb, nt - J0, (const double*)d.a_at(c0, r0), lda, (const double*)d.colchk_at(2 * J0, r0),
                            d.M.ldc, (const double*)d.colmag_at(J0, r0), d.M.ldcm, (double*)d.colchk_at(2 * J0, c0),
                            nullptr, d.M.ldr, (double*)d.colmag_at(J0, c0), nullptr, d.M.ldrm, d.s, 1);
    if (rc == ABFT_E_UNSUPPORTED)
      rc = abft_update_gemm(dtype, ABFT_COL, 'N', 'T', -1.0, d.colchk_at(2 * J0, r0), d.M.ldc, d.a_at(c0, r0), lda,
                            d.colchk_at(2 * J0, c0), d.M.ldc, m2, nb, nb, d.colmag_at(J0, r0), d.M.ldcm,
                            d.colmag_at(J0, c0), d.M.ldcm, as);
    FT_TRY(rc);
    if (single) return 0;
    return panel_row_rule(dtype, n - c0, nb, d.a_at(c0, r0), lda, d.colchk_at(2 * J0, r0), d.colchk_at(2 * J0 + 1, r0),
                          d.M.ldc, d.colmag_at(J0, r0), d.M.ldcm, d.rowchk_at(c0, 2 * J0),
                          d.rowchk_at(c0, 2 * J0 + 1), d.rowmag_at(c0, J0), d.s);
  };
  // ---- line 13: heuristic panel re-check for the TMU (Fig. 4a) + guarded
  // repair (c-25) restricted to the trailing columns [c0, c1) that consumed it
  auto recheck = [&](int k, int64_t c0, int64_t c1) -> int {
    ABFT_CUDA_TRY(cudaMemcpyAsync(d.mark, d.nfix, sizeof(int32_t), cudaMemcpyDeviceToDevice, d.s));
    FT_TRY(d.check(k + 1, (int)nt, k, k + 1, ABFT_GENERAL, ABFT_COL));
    if (!o->fig4a_repair || (Driver::diag_skip() & 1)) return 0;
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
    ra.c0 = c0;
    ra.c1 = c1;
    PhaseScope ps(d, FT_PH_OTHER);
    if (dtype == ABFT_F64)
      fig4a_repair_kernel<double><<<1, 256, 0, d.s>>>(ra);
    else
      fig4a_repair_kernel<float><<<1, 256, 0, d.s>>>(ra);
    ABFT_CUDA_TRY(cudaGetLastError());
    return 0;
  };

  bool chained = false;  // iteration k's PD / PU already ran as look-ahead
  for (int k = 0; k < nt; ++k) {
    d.iter_event();
    if (!chained) FT_TRY(chain(k, true));
    chained = false;
    if (k == nt - 1) break;
    const int64_t r1 = (int64_t)(k + 1) * nb, r2 = r1 + nb;
    // prior-operation scheme [11]: the TMU's inputs (panel, trailing matrix) before it
    if (ft && scheme == FT_SCHEME_SINGLE_PRE) {
      FT_TRY(d.check(k + 1, (int)nt, k, k + 1, ABFT_GENERAL, ABFT_COL));
      FT_TRY(d.check(k + 1, (int)nt, k + 1, (int)nt, ABFT_SYM_LOWER, ABFT_COL, true));
    }
    // line 12: TMU  A22 -= L21 L21^T (DSYRK on tensor cores) + checksum rules c-12
    FT_TRY(d.inject_at(k, FT_AT_PRE_TMU));
    if (la_on && la_at(k)) {
      // look-ahead (c-35): tile column k+1 first, its re-check, then the rest
      // of the TMU on the main stream while the side stream runs PD / PU of
      // iteration k+1 (enqueued after the rest: the side chain's host waits
      // then overlap the DSYRK)
      FT_TRY(tmu_data(k, r1, r2));
      FT_TRY(d.restore_onchip());
      if (ft) {
        FT_TRY(tmu_chk(k, r1, r2));
        FT_TRY(recheck(k, r1, r2));
      }
      ABFT_CUDA_TRY(cudaEventRecord(c->ev_col, d.s));
      // the rest's checksum rule on a stream of its own next to the DSYRK (it
      // reads only the re-checked panel L21 and its c / m_c, and writes the
      // checksums of tile columns >= k+2, which neither the DSYRK nor the side
      // chain touches), joined before the re-check whose repair may adjust
      // them: 310.8 -> 310.1 ms at n=30720.  Runs with a fault plan keep
      // Alg. 2's sequential order (the POST_TMU hook sits between the two).
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
        FT_TRY(d.periodic_check(k, k + 1, (int)nt, k + 1, (int)nt, ABFT_SYM_LOWER, true));
      }
      ABFT_CUDA_TRY(cudaStreamWaitEvent(c->side, c->ev_col, 0));
      d.on_side(true);
      const int rc = chain(k + 1, false);
      if (rc == 0) ABFT_CUDA_TRY(cudaEventRecord(c->ev_side, d.s));
      d.on_side(false);
      if (rc) return rc;
      ABFT_CUDA_TRY(cudaStreamWaitEvent(d.s, c->ev_side, 0));
      if (ft && k + 1 < nt - 1)  // Fig. 4b of iteration k+1 (reads the trailing matrix only)
        FT_TRY(d.fig4b_check(k + 2, (int)nt, k + 2, (int)nt, ABFT_SYM_LOWER, ABFT_BOTH, true, /*deferred=*/true));
      chained = true;
      continue;
    }
    // (Running the checksum rule and the panel re-check on a second stream
    // next to the DSYRK was measured: no gain at any stream priority — the
    // DSYRK keeps every SM busy — so everything stays on one stream.)
    FT_TRY(tmu_data(k, r1, n));
    FT_TRY(d.restore_onchip());  // on-chip flips hit the data step only (c-8)
    if (ft) FT_TRY(tmu_chk(k, r1, n));  // c(A_ij) -= c(L_ik) L_jk^T, r(A_ij) -= L_ik c(L_jk)^T from one product
    FT_TRY(d.inject_at(k, FT_AT_POST_TMU));
    // post-operation schemes [13], [51, 52]: the TMU's output, the whole trailing matrix
    if (ft && (scheme == FT_SCHEME_FULL_POST || scheme == FT_SCHEME_SINGLE_POST))
      FT_TRY(d.check(k + 1, (int)nt, k + 1, (int)nt, ABFT_SYM_LOWER, W, true));
    if (ft && s_new) {
      FT_TRY(recheck(k, 0, n));
      // periodic trailing-matrix check (L359)
      FT_TRY(d.periodic_check(k, k + 1, (int)nt, k + 1, (int)nt, ABFT_SYM_LOWER, true));
    }
  }
  d.iter_event();
  return d.finish(t0, stats, info_out);
}
