// ft_geqrf.cu — Householder QR with full checksums: the Alg. 1 panel (a4), the
// CTF, the QR TMU rules (a6) and the fault-tolerant driver (a7).
//
// Paper: Table III / §IV.B (L191-L237): full-checksum QR; Alg. 1 (L228-L235,
// garbled; reconstruction c-15) keeps the column checksums of the Householder
// vectors and the row checksums of R through the PD "with O(1) extra
// operation for each Householder vector"; the triangular factor T is not
// protected (L263, c-16).
//
// B200 design: the panel data is factored by cuSOLVER
// dgeqrf (LAPACK conventions: v(1) = 1, tau, beta = -sign(x1)||x||); the
// Alg. 1 checksum recurrences are then REPLAYED on the small checksum arrays
// with the same reflector quantities — for every checksum row rho
//   c_x = ck[rho, j] - W[rho, :j] R[:j, j]
//   v_ck = (c_x - beta_j W[rho, j]) / (x1 - beta_j),   x1 - beta_j = -tau_j beta_j
//   ck[rho, j+1:] -= v_ck z_j[j+1:],   z_j = tau_j v_j^T P^(j-1) = row j of T^T V^T P0
// which is algebraically Alg. 1 (the rows of Z = T^T V^T P0 are exactly the
// tau_j y_j of the interleaved algorithm), one warp per checksum row, instead
// of interleaving two checksum rows into a memory-bound unblocked panel
// factorization.  r(R) follows from r(P) by Q^T = I - V T^T V^T (GEMMs).
//
// CTF check (row f2, L263; reading c-29): before the TMU, with V as it is in
// memory, E = T^T (V^T V) T - T - T^T must vanish (orthogonality of
// I - V T V^T); a flagged T is recomputed from V and checked again.
#include "ft_driver.cuh"

namespace abft {

__global__ void add_i32_kernel_qr(int32_t* p, int32_t v) { *p += v; }

// Vbuf (mk x nb, ld mk) = unit lower trapezoidal V of the factored panel.
template <typename T>
__global__ void qr_build_v_kernel(T* V, int64_t mk, int nb, const T* panel, int64_t lda) {
  const int64_t total = mk * nb;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    const int64_t c = idx / mk, r = idx - c * mk;
    V[idx] = r > c ? panel[r + c * lda] : (r == c ? T(1) : T(0));
  }
}

// T^-1 = striu(V^T V) + diag(1/tau) ("UT transform"; tau = 0 -> T[j,j] = 0
// handled by setting the diagonal to 1 and zeroing row/column j of T after).
template <typename T>
__global__ void qr_tinv_kernel(T* Ti, const T* S, const T* tau, int nb) {
  const int64_t total = (int64_t)nb * nb;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    const int c = (int)(idx / nb), r = (int)(idx - (int64_t)c * nb);
    T v;
    if (r < c)
      v = S[idx];
    else if (r == c)
      v = tau[r] != T(0) ? T(1) / tau[r] : T(1);
    else
      v = T(0);
    Ti[idx] = v;
  }
}
template <typename T>
__global__ void qr_fix_zero_tau_kernel(T* Tm, const T* tau, int nb) {
  // a reflector with tau = 0 is the identity: its row and column of T vanish
  for (int j = blockIdx.x; j < nb; j += gridDim.x) {
    if (tau[j] != T(0)) continue;
    for (int i = threadIdx.x; i < nb; i += blockDim.x) {
      Tm[j + (int64_t)i * nb] = T(0);
      Tm[i + (int64_t)j * nb] = T(0);
    }
  }
}

// Alg. 1 checksum replay as a triangular solve.  Per checksum row x of the
// panel's colchk block (2 (nt-k) rows; tile row 0 = the diagonal tile, with
// weights w = 1 / (i+1), w = 0 elsewhere) Alg. 1 runs, for j = 0..nb-1,
//   y_j = (x_j - acc_j - beta_j w_j) / den_j,   x_c -= y_j Z[j,c]  (c > j)
// with den_j = -tau_j beta_j, beta_j = R[j,j], acc_j = sum_{i<j} w_i R[i,j]
// and Z = T^T V^T P0 (row j = tau_j v_j^T P^(j-1)).  That recurrence is the
// forward substitution of  y (D + striu(Z)) = b,  b_j = x_j - acc_j - beta_j w_j,
// so all rows are solved at once as  Y = B (D + striu(Z))^-1  (explicit
// triangular inverse + one DGEMM) instead of nb dependent steps per row.
// tau_j = 0 (identity reflector): y_j = w_j and step j changes nothing, i.e.
// row and column j of the off-diagonal part vanish and D_j = 1, b_j = w_j.
// Magnitudes (c-6): mv_j = (m_j + |beta_j| [I=0]) / |den_j|, m_c += mv_j |Z[j,c]|
//   <=>  mv (|D| - striu(|Z|)) = m + |beta| [I=0]  (an M-matrix, inverse >= 0).
template <typename T>
__global__ void qr_replay_mats_kernel(T* Tm, T* Mm, const T* ZT, const T* panel, int64_t lda, const T* tau, int nb) {
  const int64_t total = (int64_t)nb * nb;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    const int c = (int)(idx / nb), i = (int)(idx - (int64_t)c * nb);
    T t = T(0), m = T(0);
    if (i < c) {
      if (tau[i] != T(0) && tau[c] != T(0)) {
        const T z = ZT[c + (int64_t)i * nb];  // Z[i, c]
        t = z;
        m = -fabs(z);
      }
    } else if (i == c) {
      if (tau[c] != T(0)) {
        const T den = -tau[c] * panel[c + (int64_t)c * lda];
        t = den;
        m = fabs(den);
      } else {
        t = m = T(1);
      }
    }
    Tm[idx] = t;
    Mm[idx] = m;
  }
}

// right-hand sides in place: rows 0/1 (diagonal tile) get -acc_j - beta_j w_j;
// a tau_j = 0 column becomes w_j in every row (0 below the diagonal tile);
// magnitude row 0 gets +|beta_j|, a tau_j = 0 column becomes [I = 0].
template <typename T>
__global__ void qr_replay_rhs_kernel(T* ck, int64_t ldc, T* mck, int64_t ldcm, int nrows, const T* panel, int64_t lda,
                                     const T* tau, int nb) {
  const int j = blockIdx.x;
  T ae = T(0), aw = T(0);
  for (int i = threadIdx.x; i < j; i += blockDim.x) {
    const T r = panel[i + (int64_t)j * lda];
    ae = fadd(ae, r);
    aw = ffma(T(i + 1), r, aw);
  }
  __shared__ T se[32], sw[32];
  for (int m = 16; m >= 1; m >>= 1) {
    ae = fadd(ae, shfl_xor(ae, m));
    aw = fadd(aw, shfl_xor(aw, m));
  }
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  if (lane == 0) {
    se[wid] = ae;
    sw[wid] = aw;
  }
  __syncthreads();
  const T t = tau[j];
  const T beta = panel[j + (int64_t)j * lda];
  T* col = ck + (int64_t)j * ldc;
  T* mcol = mck ? mck + (int64_t)j * ldcm : nullptr;
  if (t == T(0)) {
    for (int r = threadIdx.x; r < nrows; r += blockDim.x) col[r] = r == 0 ? T(1) : (r == 1 ? T(j + 1) : T(0));
    if (mcol)
      for (int r = threadIdx.x; r < nrows / 2; r += blockDim.x) mcol[r] = r == 0 ? T(1) : T(0);
    return;
  }
  if (threadIdx.x == 0) {
    T e = T(0), w = T(0);
    for (int q = 0; q < (int)(blockDim.x >> 5); ++q) {
      e = fadd(e, se[q]);
      w = fadd(w, sw[q]);
    }
    col[0] = col[0] - e - beta;
    col[1] = col[1] - w - beta * T(j + 1);
    if (mcol) mcol[0] = mcol[0] + fabs(beta);
  }
}

// Post-TMU V re-check found a data fix inside panel k: the TMU consumed the bad
// V, which no additive repair removes for QR -> outcome R (reading c-25q).
__global__ void qr_consumed_fault_kernel(const abft_fix_t* fixes, int cap, const int32_t* n_fixes,
                                         const int32_t* mark, int64_t r0, int64_t r1, int32_t* rep,
                                         int32_t* counts) {
  const int n1 = min(*n_fixes, cap);
  int hit = 0;
  for (int f = *mark; f < n1; ++f)
    if (fixes[f].kind == ABFT_FIX_DATA && fixes[f].gj >= r0 && fixes[f].gj < r1) hit = 1;
  if (hit) {
    atomicAdd(&rep[1], 1);
    atomicAdd(&counts[ABFT_CNT_UNCORRECTABLE], 1);
  }
}

template <typename T>
static cublasStatus_t gemmT(cublasHandle_t h, cublasOperation_t a, cublasOperation_t b, int m, int n, int k, T al,
                            const T* A, int lda, const T* B, int ldb, T be, T* C, int ldc) {
  if (sizeof(T) == 8)
    return cublasDgemm(h, a, b, m, n, k, (const double*)&al, (const double*)A, lda, (const double*)B, ldb,
                       (const double*)&be, (double*)C, ldc);
  return cublasSgemm(h, a, b, m, n, k, (const float*)&al, (const float*)A, lda, (const float*)B, ldb,
                     (const float*)&be, (float*)C, ldc);
}

static unsigned blocks_of(int64_t work) {
  int64_t g = (work + 255) / 256;
  return (unsigned)(g < 1 ? 1 : (g > 148 * 16 ? 148 * 16 : g));
}

template <typename T>
int abs_copy(T* dst, const T* src, int64_t rows, int64_t cols, int64_t lds, cudaStream_t s);

// r(A2) -= V (T^T (V^T r(A2))) and m_r += |V| (|T|^T (|V|^T m_r))   (a6 for QR)
template <typename T>
static int qr_rows_rule(cublasHandle_t h, cudaStream_t s, int64_t mk, int nb, int64_t M2, const T* V, const T* Tm,
                        T* R, int64_t ldr, T* Rm, int64_t ldrm) {
  if (M2 <= 0) return 0;
  void* wv = nullptr;
  FT_TRY(scratch(s, 11, (size_t)nb * M2 * 2 * sizeof(T), &wv));
  T* t1 = reinterpret_cast<T*>(wv);
  T* t2 = t1 + (size_t)nb * M2;
  const T one = T(1), zero = T(0), mone = T(-1);
  if (gemmT<T>(h, CUBLAS_OP_T, CUBLAS_OP_N, nb, (int)M2, (int)mk, one, V, (int)mk, R, (int)ldr, zero, t1, nb) ||
      gemmT<T>(h, CUBLAS_OP_T, CUBLAS_OP_N, nb, (int)M2, nb, one, Tm, nb, t1, nb, zero, t2, nb) ||
      gemmT<T>(h, CUBLAS_OP_N, CUBLAS_OP_N, (int)mk, (int)M2, nb, mone, V, (int)mk, t2, nb, one, R, (int)ldr))
    return ABFT_E_CUBLAS;
  if (!Rm) return 0;
  const int64_t M = M2 / 2 > 0 ? M2 / 2 : 1;
  void* av = nullptr;
  FT_TRY(scratch(s, 12, ((size_t)mk * nb + (size_t)nb * nb) * sizeof(T), &av));
  T* aV = reinterpret_cast<T*>(av);
  T* aT = aV + (size_t)mk * nb;
  FT_TRY(abs_copy<T>(aV, V, mk, nb, mk, s));
  FT_TRY(abs_copy<T>(aT, Tm, nb, nb, nb, s));
  if (gemmT<T>(h, CUBLAS_OP_T, CUBLAS_OP_N, nb, (int)M, (int)mk, one, aV, (int)mk, Rm, (int)ldrm, zero, t1, nb) ||
      gemmT<T>(h, CUBLAS_OP_T, CUBLAS_OP_N, nb, (int)M, nb, one, aT, nb, t1, nb, zero, t2, nb) ||
      gemmT<T>(h, CUBLAS_OP_N, CUBLAS_OP_N, (int)mk, (int)M, nb, one, aV, (int)mk, t2, nb, one, Rm, (int)ldrm))
    return ABFT_E_CUBLAS;
  return 0;
}

template <typename T>
static int panel_geqrf_t(const abft_mat_t* mat, int k, T* tau, T* Vbuf, T* Tout, T* P0, int32_t* info,
                         cudaStream_t s, Driver* host = nullptr) {
  const int64_t nb = mat->nb, n = mat->n, nt = n / nb, r0 = k * nb, mk = n - r0;
  const bool ft = mat->colchk != nullptr;
  T* A = reinterpret_cast<T*>(mat->A);
  T* panel = A + r0 + r0 * mat->lda;
  if (ft)
    FT_TRY(abft::copy2d(P0, mk * sizeof(T), panel, mat->lda * sizeof(T), mk * sizeof(T), nb, s));
  if (host) {  // FT_PD_HOST: Alg. 2 lines 3-7 around the host dgeqrf (ft_host.cu)
    FT_TRY(host_panel_pd(*host, k, HOST_GEQRF, r0, r0, mk, nullptr, tau, info));
  } else {
    std::unique_lock<std::mutex> lk;
    cusolverDnHandle_t h = solver_handle(s, lk);
    int lwork = 0;
    cusolverStatus_t st = sizeof(T) == 8
                              ? cusolverDnDgeqrf_bufferSize(h, (int)mk, (int)nb, (double*)panel, (int)mat->lda, &lwork)
                              : cusolverDnSgeqrf_bufferSize(h, (int)mk, (int)nb, (float*)panel, (int)mat->lda, &lwork);
    if (st != CUSOLVER_STATUS_SUCCESS) return ABFT_E_CUSOLVER;
    void* w = nullptr;
    FT_TRY(scratch(s, 13, (size_t)(lwork + 1) * sizeof(T), &w));
    st = sizeof(T) == 8 ? cusolverDnDgeqrf(h, (int)mk, (int)nb, (double*)panel, (int)mat->lda, (double*)tau,
                                          (double*)w, lwork, info)
                        : cusolverDnSgeqrf(h, (int)mk, (int)nb, (float*)panel, (int)mat->lda, (float*)tau, (float*)w,
                                          lwork, info);
    if (st != CUSOLVER_STATUS_SUCCESS) return ABFT_E_CUSOLVER;
  }
  // V and the CTF: T = (striu(V^T V) + diag(1/tau))^-1
  qr_build_v_kernel<T><<<blocks_of(mk * nb), 256, 0, s>>>(Vbuf, mk, (int)nb, panel, mat->lda);
  void* sv = nullptr;
  FT_TRY(scratch(s, 14, (size_t)nb * nb * 3 * sizeof(T), &sv));
  T* S = reinterpret_cast<T*>(sv);
  T* Ti = S + (size_t)nb * nb;
  T* G = Ti + (size_t)nb * nb;
  {
    std::unique_lock<std::mutex> lk;
    cublasHandle_t h = blas_handle(s, lk);
    if (gemmT<T>(h, CUBLAS_OP_T, CUBLAS_OP_N, (int)nb, (int)nb, (int)mk, T(1), Vbuf, (int)mk, Vbuf, (int)mk, T(0), S,
                 (int)nb))
      return ABFT_E_CUBLAS;
  }
  qr_tinv_kernel<T><<<blocks_of(nb * nb), 256, 0, s>>>(Ti, S, tau, (int)nb);
  FT_TRY(abft_tri_inverse(mat->dtype, 'U', 'N', nb, Ti, nb, Tout, nb, (abft_stream_t)s));
  qr_fix_zero_tau_kernel<T><<<(unsigned)nb, 128, 0, s>>>(Tout, tau, (int)nb);
  ABFT_CUDA_TRY(cudaGetLastError());
  if (!ft) return 0;
  // Z = T^T (V^T P0): row j = tau_j v_j^T P^(j-1); stored transposed,
  // ZT = G^T T with G = V^T P0, so the replay reads row j of Z contiguously
  T* ZT = S;  // reuse
  {
    std::unique_lock<std::mutex> lk;
    cublasHandle_t h = blas_handle(s, lk);
    if (gemmT<T>(h, CUBLAS_OP_T, CUBLAS_OP_N, (int)nb, (int)nb, (int)mk, T(1), Vbuf, (int)mk, P0, (int)mk, T(0), G,
                 (int)nb) ||
        gemmT<T>(h, CUBLAS_OP_T, CUBLAS_OP_N, (int)nb, (int)nb, (int)nb, T(1), G, (int)nb, Tout, (int)nb, T(0), ZT,
                 (int)nb))
      return ABFT_E_CUBLAS;
  }
  const int nrows = (int)(2 * (nt - k));
  T* ck = reinterpret_cast<T*>(mat->colchk) + 2 * k + r0 * mat->ldc;
  T* mck = mat->colmag ? reinterpret_cast<T*>(mat->colmag) + k + r0 * mat->ldcm : nullptr;
  T* Tm = Ti;  // free again: D + striu(Z)
  T* Mm = G;   // |D| - striu(|Z|)
  void* wv = nullptr;
  FT_TRY(scratch(s, 16, (size_t)nb * nb * 2 * sizeof(T), &wv));
  T* W1 = reinterpret_cast<T*>(wv);
  T* W2 = W1 + (size_t)nb * nb;
  qr_replay_mats_kernel<T><<<blocks_of(nb * nb), 256, 0, s>>>(Tm, Mm, ZT, panel, mat->lda, tau, (int)nb);
  qr_replay_rhs_kernel<T><<<(unsigned)nb, 128, 0, s>>>(ck, mat->ldc, mck, mat->ldcm, nrows, panel, mat->lda, tau,
                                                        (int)nb);
  ABFT_CUDA_TRY(cudaGetLastError());
  FT_TRY(abft_tri_inverse(mat->dtype, 'U', 'N', nb, Tm, nb, W1, nb, (abft_stream_t)s));
  FT_TRY(abft_update_trsm_inv(mat->dtype, 'R', 'N', nb, W1, nb, ck, mat->ldc, nrows, nullptr, 0, 0,
                              (abft_stream_t)s));
  if (mck) {
    FT_TRY(abft_tri_inverse(mat->dtype, 'U', 'N', nb, Mm, nb, W2, nb, (abft_stream_t)s));
    FT_TRY(abft_update_trsm_inv(mat->dtype, 'R', 'N', nb, W2, nb, mck, mat->ldcm, nrows / 2, nullptr, 0, 0,
                                (abft_stream_t)s));
  }
  // r(R): r(P) <- Q^T r(P) for the panel's row checksums (m_k x 2)
  {
    std::unique_lock<std::mutex> lk;
    cublasHandle_t h = blas_handle(s, lk);
    T* R = reinterpret_cast<T*>(mat->rowchk) + r0 + 2 * k * mat->ldr;
    T* Rm = mat->rowmag ? reinterpret_cast<T*>(mat->rowmag) + r0 + k * mat->ldrm : nullptr;
    FT_TRY(qr_rows_rule<T>(h, s, mk, (int)nb, 2, Vbuf, Tout, R, mat->ldr, Rm, mat->ldrm));
  }
  return 0;
}

}  // namespace abft

extern "C" int abft_panel_geqrf(const abft_mat_t* mat, int32_t k, void* tau, void* V, void* T, void* panel_copy,
                                int32_t* info, abft_stream_t stream) {
  using namespace abft;
  if (!mat || mat->m != mat->n || mat->nb < 32 || mat->nb > 1024 || (mat->nb & (mat->nb - 1)) ||
      mat->n % mat->nb || !mat->A || mat->lda < mat->m)
    return -1;
  if (k < 0 || k >= mat->n / mat->nb) return -2;
  if (!tau) return -3;
  if (!V) return -4;
  if (!T) return -5;
  if (mat->colchk && (!mat->rowchk || !panel_copy)) return -6;
  if (!info) return -7;
  cudaStream_t s = (cudaStream_t)stream;
  return mat->dtype == ABFT_F64
             ? panel_geqrf_t<double>(mat, k, (double*)tau, (double*)V, (double*)T, (double*)panel_copy, info, s)
             : panel_geqrf_t<float>(mat, k, (float*)tau, (float*)V, (float*)T, (float*)panel_copy, info, s);
}

// ---------------------------------------------------------- CTF check (f2) --
namespace abft {
// a_i = sum_k |T_ki| sqrt(S_kk): |T|^T ||v|| (c-29 bound)
template <typename T>
__global__ void ctf_a_kernel(T* a, const T* Tm, const T* S, int nb) {
  const int i = blockIdx.x;
  double acc = 0.0;
  for (int k = threadIdx.x; k < nb; k += blockDim.x)
    acc += fabs((double)Tm[k + (int64_t)i * nb]) * sqrt(fabs((double)S[k + (int64_t)k * nb]));
  for (int m = 16; m >= 1; m >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, m);
  __shared__ double part[32];
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += part[w];
    a[i] = (T)t;
  }
}

// E = T^T S T (precomputed) ; flag (i, j) iff E_ij - T_ij - T_ji is non-finite
// or exceeds g4 (a_i a_j + |T_ij| + |T_ji|)
template <typename T>
__global__ void ctf_flag_kernel(const T* TST, const T* Tm, const T* a, int nb, double g4, int32_t* cnt) {
  const int64_t total = (int64_t)nb * nb;
  int bad = 0;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    const int j = (int)(idx / nb), i = (int)(idx - (int64_t)j * nb);
    const double tij = (double)Tm[idx], tji = (double)Tm[j + (int64_t)i * nb];
    const double e = (double)TST[idx] - tij - tji;
    const double b = g4 * ((double)a[i] * (double)a[j] + fabs(tij) + fabs(tji));
    if (!isfinite(e) || !isfinite(b) || !(fabs(e) <= b)) ++bad;
  }
  for (int m = 16; m >= 1; m >>= 1) bad += __shfl_xor_sync(0xffffffffu, bad, m);
  if ((threadIdx.x & 31) == 0 && bad) atomicAdd(cnt, bad);
}

// One CTF check of T (nb x nb) against the V in Vbuf (mk x nb): S = V^T V,
// TST = T^T (S T), flags -> *cnt (device).  S stays in `S` for a recompute.
template <typename T>
static int ctf_eval(cudaStream_t s, int64_t mk, int nb, const T* Vbuf, const T* Tm, T* S, T* W, T* TST, T* a,
                    double g4, int32_t* cnt) {
  {
    std::unique_lock<std::mutex> lk;
    cublasHandle_t h = blas_handle(s, lk);
    if (gemmT<T>(h, CUBLAS_OP_T, CUBLAS_OP_N, nb, nb, (int)mk, T(1), Vbuf, (int)mk, Vbuf, (int)mk, T(0), S, nb) ||
        gemmT<T>(h, CUBLAS_OP_N, CUBLAS_OP_N, nb, nb, nb, T(1), S, nb, Tm, nb, T(0), W, nb) ||
        gemmT<T>(h, CUBLAS_OP_T, CUBLAS_OP_N, nb, nb, nb, T(1), Tm, nb, W, nb, T(0), TST, nb))
      return ABFT_E_CUBLAS;
  }
  ABFT_CUDA_TRY(cudaMemsetAsync(cnt, 0, sizeof(int32_t), s));
  ctf_a_kernel<T><<<(unsigned)nb, 128, 0, s>>>(a, Tm, S, nb);
  ctf_flag_kernel<T><<<blocks_of((int64_t)nb * nb), 256, 0, s>>>(TST, Tm, a, nb, g4, cnt);
  ABFT_CUDA_TRY(cudaGetLastError());
  return 0;
}

// f2 for iteration k, in two halves so that its host read-back can share one
// wait with the PD restart decision: ctf_issue rebuilds V from memory,
// evaluates E and queues the flag count into hpin[1]; ctf_resolve (after the
// caller waited) recomputes T from V (the CTF of panel_geqrf_t:
// T = (striu(V^T V) + diag(1/tau))^-1) if flagged and checks again; a T still
// flagged is uncorrectable.
struct CtfWork {
  void* sv;
  double g4;
};

template <typename T>
static int ctf_issue(Driver& d, int64_t mk, T* Vbuf, T* Tm, CtfWork* w) {
  cudaStream_t s = d.s;
  const int nb = (int)d.nb;
  FT_TRY(scratch(s, 17, ((size_t)nb * nb * 4 + nb) * sizeof(T), &w->sv));
  T* S = reinterpret_cast<T*>(w->sv);
  T* W = S + (size_t)nb * nb;
  T* TST = W + (size_t)nb * nb;
  T* a = TST + (size_t)2 * nb * nb;
  const double m = (double)(mk + nb), u = Prec<T>::u;
  w->g4 = 4.0 * d.tol.scale * m * u / (1.0 - m * u);
  qr_build_v_kernel<T><<<blocks_of(mk * nb), 256, 0, s>>>(Vbuf, mk, nb, reinterpret_cast<T*>(d.a_at(d.n - mk, d.n - mk)),
                                                         d.lda);
  FT_TRY(ctf_eval<T>(s, mk, nb, Vbuf, Tm, S, W, TST, a, w->g4, d.ctf_cnt));
  return d.post_word(d.ctf_cnt, 1);
}

template <typename T>
static int ctf_resolve(Driver& d, int64_t mk, T* Vbuf, T* Tm, const T* tau, const CtfWork& w) {
  if (d.host_word(1) == 0) return 0;
  cudaStream_t s = d.s;
  const int nb = (int)d.nb;
  T* S = reinterpret_cast<T*>(w.sv);
  T* W = S + (size_t)nb * nb;
  T* TST = W + (size_t)nb * nb;
  T* Ti = TST + (size_t)nb * nb;
  T* a = Ti + (size_t)nb * nb;
  ++d.ctf_flagged;
  qr_tinv_kernel<T><<<blocks_of((int64_t)nb * nb), 256, 0, s>>>(Ti, S, tau, nb);
  FT_TRY(abft_tri_inverse(d.dtype, 'U', 'N', nb, Ti, nb, Tm, nb, (abft_stream_t)s));
  qr_fix_zero_tau_kernel<T><<<(unsigned)nb, 128, 0, s>>>(Tm, tau, nb);
  ++d.ctf_recomputed;
  FT_TRY(ctf_eval<T>(s, mk, nb, Vbuf, Tm, S, W, TST, a, w.g4, d.ctf_cnt));
  FT_TRY(d.post_word(d.ctf_cnt, 1));
  ABFT_CUDA_TRY(cudaEventSynchronize(d.c->ev));
  if (d.host_word(1) != 0) add_i32_kernel_qr<<<1, 1, 0, s>>>(d.counts + ABFT_CNT_UNCORRECTABLE, 1);
  return 0;
}
}  // namespace abft

// ----------------------------------------------------------------- driver --
namespace abft {
template <typename T>
static int geqrf_driver(Driver& d, ft_ctx* c, T* tau_all) {
  const int64_t nb = d.nb, n = d.n, nt = d.nt, lda = d.lda;
  const bool ft = d.o->abft != 0;
  cudaStream_t s = d.s;
  const abft_stream_t as = (abft_stream_t)s;
  T* Vbuf = reinterpret_cast<T*>(c->putmp);
  T* P0 = reinterpret_cast<T*>(c->aux);
  T* Tm = reinterpret_cast<T*>(c->linv);
  T* A = reinterpret_cast<T*>(d.A);
  void* wv = nullptr;
  FT_TRY(scratch(s, 15, (size_t)nb * n * 2 * sizeof(T), &wv));
  T* G = reinterpret_cast<T*>(wv);
  T* W = G + (size_t)nb * n;
  if (ft) {
    abft_tiles_t all{0, (int)nt, 0, (int)nt, 0, ABFT_GENERAL};
    FT_TRY(abft_encode(&d.M, &all, ABFT_BOTH, as));
  }
  for (int k = 0; k < nt; ++k) {
    d.iter_event();
    const int64_t r0 = k * nb, r1 = r0 + nb, mk = n - r0, nk = n - r1;
    // Alg. 2 lines 3-4: check the column panel to be decomposed (c + r)
    FT_TRY(d.inject_at(k, FT_AT_PRE_PD_CHECK));
    if (ft) FT_TRY(d.check(k, (int)nt, k, k + 1, ABFT_GENERAL, ABFT_BOTH));
    // Local restart (f1, L430): copy of the column panel with its checksums
    // (rsv: panel | c | m_c | r | m_r) after its pre-op check
    const bool rs = ft && d.o->restart;
    const int ntk = (int)(nt - k);
    char* cp_a = (char*)c->rsv;
    char* cp_c = cp_a + (size_t)mk * nb * d.es;
    char* cp_m = cp_c + (size_t)2 * ntk * nb * d.es;
    char* cp_r = cp_m + (size_t)ntk * nb * d.es;
    char* cp_rm = cp_r + (size_t)mk * 2 * d.es;
    if (rs) {
      FT_TRY(d.copy(cp_a, mk, d.a_at(r0, r0), lda, mk, nb));
      FT_TRY(d.copy(cp_c, 2 * ntk, d.colchk_at(2 * k, r0), d.M.ldc, 2 * ntk, nb));
      FT_TRY(d.copy(cp_m, ntk, d.colmag_at(k, r0), d.M.ldcm, ntk, nb));
      FT_TRY(d.copy(cp_r, mk, d.rowchk_at(r0, 2 * k), d.M.ldr, mk, 2));
      FT_TRY(d.copy(cp_rm, mk, d.rowmag_at(r0, k), d.M.ldrm, mk, 1));
    }
    // line 5: PD (Alg. 1: V with c(V), R_kk with r(R)) + CTF
    auto do_pd = [&]() -> int {
      if (d.o->pd_location == FT_PD_HOST)
        FT_TRY(panel_geqrf_t<T>(&d.M, k, tau_all + r0, Vbuf, Tm, P0, d.info, s, &d));
      else
        FT_TRY(abft_panel_geqrf(&d.M, k, tau_all + r0, Vbuf, Tm, P0, d.info, as));
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
    // line 7: check V (UNIT_LOWER on the diagonal, c) and R_kk (UPPER, r);
    // 2D -> restore the copy and redo the PD once.  The decision's read-back
    // shares one host wait with the CTF check's (the A2 check in between is
    // independent of the panel).
    auto restart_pd = [&]() -> int {
      FT_TRY(d.copy(d.a_at(r0, r0), lda, cp_a, mk, mk, nb));
      FT_TRY(d.copy(d.colchk_at(2 * k, r0), d.M.ldc, cp_c, 2 * ntk, 2 * ntk, nb));
      FT_TRY(d.copy(d.colmag_at(k, r0), d.M.ldcm, cp_m, ntk, ntk, nb));
      FT_TRY(d.copy(d.rowchk_at(r0, 2 * k), d.M.ldr, cp_r, mk, mk, 2));
      FT_TRY(d.copy(d.rowmag_at(r0, k), d.M.ldrm, cp_rm, mk, mk, 1));
      FT_TRY(do_pd());
      return post_pd_checks();
    };
    if (ft) {
      if (rs) FT_TRY(d.snap_uncorrectable());
      FT_TRY(post_pd_checks());
      if (rs) FT_TRY(d.post_delta(0));
    }
    if (k == nt - 1) {
      int delta = 0;
      if (rs) FT_TRY(d.wait_delta(0, &delta));
      if (delta > 0) {
        FT_TRY(d.take_back_uncorrectable(delta));
        FT_TRY(restart_pd());
      }
      break;
    }
    // QR's TMU reads all of A2 (W = T^T V^T A2): A2 is a reference part, so it
    // is checked before the TMU (Alg. 2 line 8 for QR, reading c-25q)
    if (ft) FT_TRY(d.check(k, (int)nt, k + 1, (int)nt, ABFT_GENERAL, ABFT_BOTH));
    // f2 (L263): T carries no checksum; verify the orthogonality of I - V T V^T
    if (ft) {
      CtfWork cw{};
      FT_TRY(ctf_issue<T>(d, mk, Vbuf, Tm, &cw));
      ABFT_CUDA_TRY(cudaEventSynchronize(c->ev));  // one wait: PD decision + CTF flags
      const int delta = rs ? d.host_word(0) : 0;
      if (delta > 0) {
        FT_TRY(d.take_back_uncorrectable(delta));
        FT_TRY(restart_pd());  // new V and T: check them again
        FT_TRY(ctf_issue<T>(d, mk, Vbuf, Tm, &cw));
        ABFT_CUDA_TRY(cudaEventSynchronize(c->ev));
      }
      FT_TRY(ctf_resolve<T>(d, mk, Vbuf, Tm, tau_all + r0, cw));
    }
    // line 12: TMU  A2 <- (I - V T V^T)^T A2 = A2 - V W,  W = T^T V^T A2
    FT_TRY(d.inject_at(k, FT_AT_PRE_TMU));
    const bool touched = d.o->n_inject > 0;  // V re-read from memory after hooks
    if (touched || ft) qr_build_v_kernel<T><<<blocks_of(mk * nb), 256, 0, s>>>(Vbuf, mk, (int)nb, A + r0 + r0 * lda, lda);
    {
      std::unique_lock<std::mutex> lk;
      cublasHandle_t h = blas_handle(s, lk);
      if (gemmT<T>(h, CUBLAS_OP_T, CUBLAS_OP_N, (int)nb, (int)nk, (int)mk, T(1), Vbuf, (int)mk, A + r0 + r1 * lda,
                   (int)lda, T(0), G, (int)nb) ||
          gemmT<T>(h, CUBLAS_OP_T, CUBLAS_OP_N, (int)nb, (int)nk, (int)nb, T(1), Tm, (int)nb, G, (int)nb, T(0), W,
                   (int)nb) ||
          gemmT<T>(h, CUBLAS_OP_N, CUBLAS_OP_N, (int)mk, (int)nk, (int)nb, T(-1), Vbuf, (int)mk, W, (int)nb, T(1),
                   A + r0 + r1 * lda, (int)lda))
        return ABFT_E_CUBLAS;
    }
    const bool had_onchip = !d.onchip_pending.empty();
    FT_TRY(d.restore_onchip());
    if (ft) {
      if (had_onchip)  // the checksum step re-reads V after the on-chip flip is gone
        qr_build_v_kernel<T><<<blocks_of(mk * nb), 256, 0, s>>>(Vbuf, mk, (int)nb, A + r0 + r0 * lda, lda);
      // c(A2) -= c(V) W ; m_c += m_c(V) |W|
      FT_TRY(abft_update_gemm(d.dtype, ABFT_COL, 'N', 'N', -1.0, d.colchk_at(2 * k, r0), d.M.ldc, W, nb,
                              d.colchk_at(2 * k, r1), d.M.ldc, 2 * (nt - k), nk, nb, d.colmag_at(k, r0), d.M.ldcm,
                              d.colmag_at(k, r1), d.M.ldcm, as));
      // r(A2) -= V (T^T V^T r(A2)) ; m_r += |V| (|T|^T |V|^T m_r)
      std::unique_lock<std::mutex> lk;
      cublasHandle_t h = blas_handle(s, lk);
      FT_TRY(qr_rows_rule<T>(h, s, mk, (int)nb, 2 * (nt - k - 1), Vbuf, Tm, (T*)d.rowchk_at(r0, 2 * (k + 1)),
                             d.M.ldr, (T*)d.rowmag_at(r0, k + 1), d.M.ldrm));
    }
    FT_TRY(d.inject_at(k, FT_AT_POST_TMU));
    // line 13: re-check V (Fig. 4a; a consumed V fault is R for QR) and R12 (r)
    if (ft) {
      ABFT_CUDA_TRY(cudaMemcpyAsync(d.mark, d.nfix, sizeof(int32_t), cudaMemcpyDeviceToDevice, s));
      FT_TRY(d.check(k, (int)nt, k, k + 1, ABFT_UNIT_LOWER, ABFT_COL));
      qr_consumed_fault_kernel<<<1, 1, 0, s>>>(c->fixlog, c->fixcap, d.nfix, d.mark, r0, r1, d.rep, d.counts);
      FT_TRY(d.check(k, k + 1, k + 1, (int)nt, ABFT_GENERAL, ABFT_ROW));
      FT_TRY(d.periodic_check(k, k + 1, (int)nt, k + 1, (int)nt, ABFT_GENERAL, false));  // L359
    }
  }
  return 0;
}
}  // namespace abft

extern "C" int ft_geqrf(ft_ctx_t* c, int32_t dtype, int64_t n, void* dA, int64_t lda, void* tau, const ft_opts_t* o,
                        ft_stats_t* stats, int64_t* info_out) {
  using namespace abft;
  if (!c) return -1;
  if (dtype != ABFT_F32 && dtype != ABFT_F64) return -2;
  if (!o) return -7;
  const int64_t nb = o->nb;
  if (n < 0 || nb < 32 || nb > 1024 || (nb & (nb - 1)) || n % nb) return -3;
  if (!dA) return -4;
  if (lda < std::max<int64_t>(1, n)) return -5;
  if (!tau) return -6;
  if (o->n_inject < 0 || (o->n_inject > 0 && !o->inject)) return -7;
  if (o->scheme != FT_SCHEME_NEW || o->checksum_gemm) return -7;  // scheme / GEMM-check comparisons: ft_potrf only
  ABFT_CUDA_TRY(cudaSetDevice(c->device));
  Driver d;
  FT_TRY(d.setup(c, dtype, n, nb, dA, lda, o, /*lu=*/true));
  d.qr = true;
  FT_TRY(grow_buffer(c->aux, c->aux_bytes, (size_t)n * nb * d.es));
  auto t0 = std::chrono::steady_clock::now();
  const int rc = dtype == ABFT_F64 ? geqrf_driver<double>(d, c, (double*)tau) : geqrf_driver<float>(d, c, (float*)tau);
  if (rc) return rc;
  d.iter_event();
  return d.finish(t0, stats, info_out);
}
