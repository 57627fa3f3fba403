// abft_update.cu — checksum maintenance through PD / PU / TMU (rows a4-a6).
//
// Paper: checksums are updated "as if the checksums are an extended part of
// the original input matrix ... applying the same operation" (L149, §IV);
// full checksums survive the TMU when one operand carries column and the
// other row checksums (L189, [31]); the checksum ops follow the original op
// with a smaller input (L475, §IX.A.2).  The skinny products (M2 = 2 rows per
// tile) are plain library GEMM/TRSM calls (cuBLAS, DMMA on B200 for fp64);
// the magnitude propagation of reading c-6 needs |op(Y)| and |T^-1|, which
// are produced by small elementwise kernels here.
#include <cublas_v2.h>
#include <cusolverDn.h>

#include <mutex>
#include <type_traits>
#include <unordered_map>
#include <vector>

#include "abft_common.cuh"

#define ABFT_CUBLAS_TRY(expr)                                                                    \
  do {                                                                                           \
    cublasStatus_t _s = (expr);                                                                  \
    if (_s != CUBLAS_STATUS_SUCCESS) {                                                           \
      fprintf(stderr, "[abft] cuBLAS status %d at %s:%d\n", (int)_s, __FILE__, __LINE__);        \
      return ABFT_E_CUBLAS;                                                                      \
    }                                                                                            \
  } while (0)
#define ABFT_CUSOLVER_TRY(expr)                                                                  \
  do {                                                                                           \
    cusolverStatus_t _s = (expr);                                                                \
    if (_s != CUSOLVER_STATUS_SUCCESS) {                                                         \
      fprintf(stderr, "[abft] cuSOLVER status %d at %s:%d\n", (int)_s, __FILE__, __LINE__);      \
      return ABFT_E_CUSOLVER;                                                                    \
    }                                                                                            \
  } while (0)

namespace abft {

// ------------------------------------------------------------- handles --
namespace {
struct Handles {
  cublasHandle_t blas = nullptr;
  cusolverDnHandle_t solver = nullptr;
  std::mutex mu;
};
std::mutex g_hmu;
// One cuBLAS / cuSOLVER handle pair per (device, stream): library calls issued
// on different streams at the same time (the drivers' side stream) must not
// share a handle's workspace.
std::unordered_map<uint64_t, Handles*>& handle_map() {
  static auto* m = new std::unordered_map<uint64_t, Handles*>();
  return *m;
}
uint64_t handle_key(cudaStream_t s) {
  int dev = 0;
  cudaGetDevice(&dev);
  return (reinterpret_cast<uint64_t>(s) << 8) ^ (uint64_t)dev;
}
Handles& handles_for(cudaStream_t s) {
  const uint64_t key = handle_key(s);
  std::lock_guard<std::mutex> g(g_hmu);
  auto& m = handle_map();
  auto it = m.find(key);
  if (it != m.end()) return *it->second;
  Handles* h = new Handles();
  cublasCreate(&h->blas);
  cusolverDnCreate(&h->solver);
  cublasSetStream(h->blas, s);
  cusolverDnSetStream(h->solver, s);
  m[key] = h;
  return *h;
}

// Scratch buffers private to the update ops (distinct from the pass pools).
struct Scratch {
  void* p = nullptr;
  size_t bytes = 0;
};
std::mutex g_smu;
constexpr int kScratchSlots = 32;  // slots in use: 1-23
std::unordered_map<uint64_t, Scratch>& scratch_map() {
  static auto* m = new std::unordered_map<uint64_t, Scratch>();
  return *m;
}
uint64_t scratch_key(cudaStream_t s, int slot) {
  int dev = 0;
  cudaGetDevice(&dev);
  return (reinterpret_cast<uint64_t>(s) << 12) ^ ((uint64_t)dev << 4) ^ (uint64_t)slot;
}
int scratch_get(cudaStream_t s, int slot, size_t bytes, void** out) {
  const uint64_t key = scratch_key(s, slot);
  std::lock_guard<std::mutex> g(g_smu);
  Scratch& sc = scratch_map()[key];
  if (sc.bytes < bytes) {
    if (sc.p) {
      ABFT_CUDA_TRY(cudaStreamSynchronize(s));
      ABFT_CUDA_TRY(cudaFree(sc.p));
    }
    size_t nb = bytes + bytes / 4 + 4096;
    if (cudaMalloc(&sc.p, nb) != cudaSuccess) {
      sc.p = nullptr;
      sc.bytes = 0;
      return ABFT_E_NOMEM;
    }
    sc.bytes = nb;
  }
  *out = sc.p;
  return 0;
}
}  // namespace

cublasHandle_t blas_handle(cudaStream_t s, std::unique_lock<std::mutex>& lk) {
  Handles& h = handles_for(s);
  lk = std::unique_lock<std::mutex>(h.mu);
  return h.blas;
}
cusolverDnHandle_t solver_handle(cudaStream_t s, std::unique_lock<std::mutex>& lk) {
  Handles& h = handles_for(s);
  lk = std::unique_lock<std::mutex>(h.mu);
  return h.solver;
}
int scratch(cudaStream_t s, int slot, size_t bytes, void** out) { return scratch_get(s, slot, bytes, out); }

void release_stream_handles(cudaStream_t s) {
  {
    std::lock_guard<std::mutex> g(g_hmu);
    auto& m = handle_map();
    auto it = m.find(handle_key(s));
    if (it != m.end()) {
      cublasDestroy(it->second->blas);
      cusolverDnDestroy(it->second->solver);
      delete it->second;
      m.erase(it);
    }
  }
  std::lock_guard<std::mutex> g(g_smu);
  auto& m = scratch_map();
  for (int slot = 0; slot < kScratchSlots; ++slot) {
    auto it = m.find(scratch_key(s, slot));
    if (it == m.end()) continue;
    if (it->second.p) cudaFree(it->second.p);
    m.erase(it);
  }
}

// ---------------------------------------------------- elementwise kernels --
// dst (rows x cols, ld = rows) = |src (ld = lds)|
template <typename T>
__global__ void abs_copy_kernel(T* __restrict__ dst, const T* __restrict__ src, int64_t rows, int64_t cols,
                                int64_t lds) {
  int64_t total = rows * cols;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    int64_t c = idx / rows, r = idx - c * rows;
    dst[idx] = fabs(src[r + c * lds]);
  }
}
template <typename T>
__global__ void identity_kernel(T* d, int n) {
  int64_t total = (int64_t)n * n;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    int64_t c = idx / n, r = idx - c * n;
    d[idx] = r == c ? T(1) : T(0);
  }
}
template <typename T>
__global__ void abs_inplace_kernel(T* d, int64_t total) {
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x)
    d[idx] = fabs(d[idx]);
}

static unsigned grid_for(int64_t total) {
  int64_t g = (total + 255) / 256;
  return (unsigned)(g < 148 * 16 ? (g < 1 ? 1 : g) : 148 * 16);
}

template <typename T>
int abs_copy(T* dst, const T* src, int64_t rows, int64_t cols, int64_t lds, cudaStream_t s) {
  if (rows * cols == 0) return 0;
  abs_copy_kernel<T><<<grid_for(rows * cols), 256, 0, s>>>(dst, src, rows, cols, lds);
  ABFT_CUDA_TRY(cudaGetLastError());
  return 0;
}
template int abs_copy<double>(double*, const double*, int64_t, int64_t, int64_t, cudaStream_t);
template int abs_copy<float>(float*, const float*, int64_t, int64_t, int64_t, cudaStream_t);

// ---------------------------------------------------- typed BLAS shims --
static cublasStatus_t gemm(cublasHandle_t h, cublasOperation_t ta, cublasOperation_t tb, int m, int n, int k,
                           const double* al, const double* A, int lda, const double* B, int ldb, const double* be,
                           double* C, int ldc) {
  return cublasDgemm(h, ta, tb, m, n, k, al, A, lda, B, ldb, be, C, ldc);
}
static cublasStatus_t gemm(cublasHandle_t h, cublasOperation_t ta, cublasOperation_t tb, int m, int n, int k,
                           const float* al, const float* A, int lda, const float* B, int ldb, const float* be,
                           float* C, int ldc) {
  return cublasSgemm(h, ta, tb, m, n, k, al, A, lda, B, ldb, be, C, ldc);
}

static cublasOperation_t op_of(char t) { return (t == 'T' || t == 't') ? CUBLAS_OP_T : CUBLAS_OP_N; }

// W = T^-1 (explicit triangular inverse; the other triangle of W is zero, a
// unit diagonal is materialised).  Recursive block inversion:
// the 64x64 diagonal blocks are inverted in shared memory by one CTA each
// (row-by-row substitution, threads over columns), then pairs of inverted
// blocks are merged level by level with two strided-batched DGEMMs,
//   lower: inv([A 0; B C]) = [A^-1 0; -C^-1 B A^-1  C^-1]
//   upper: inv([A B; 0 C]) = [A^-1  -A^-1 B C^-1; 0 C^-1].
constexpr int kInvBS = 64;

template <typename T>
__global__ void __launch_bounds__(256) tri_inv_base_kernel(const T* __restrict__ Tm, int ldt, T* __restrict__ W,
                                                           int ldw, int bs, int upper, int unit) {
  // X = L^-1 (Ls: the lower triangle, or U^T for upper); the load uses all
  // 256 threads, the substitution one thread per column
  extern __shared__ __align__(16) unsigned char inv_sm[];
  T(*Ls)[kInvBS + 1] = reinterpret_cast<T(*)[kInvBS + 1]>(inv_sm);
  T(*Xs)[kInvBS + 1] = Ls + kInvBS;
  const int b0 = blockIdx.x * bs;
  const int tid = threadIdx.x;
  for (int idx = tid; idx < bs * bs; idx += blockDim.x) {
    const int i = idx % bs, j = idx / bs;  // coalesced along i (column-major source)
    T v;
    if (upper)  // Ls = U^T (lower): Ls[j][i] = U[i][j] for i <= j
      v = Tm[(b0 + i) + (int64_t)(b0 + j) * ldt];
    else
      v = Tm[(b0 + i) + (int64_t)(b0 + j) * ldt];
    if (upper) {
      T u = (i <= j) ? v : T(0);
      if (unit && i == j) u = T(1);
      Ls[j][i] = u;
    } else {
      T l = (i >= j) ? v : T(0);
      if (unit && i == j) l = T(1);
      Ls[i][j] = l;
    }
    Xs[i][j] = (i == j) ? T(1) : T(0);
  }
  __syncthreads();
  // X = Ls^-1 blocked inside the CTA: the 16x16 diagonal blocks by forward
  // substitution (one thread per column), then the pairs merged level by
  // level, X21 = -X22 (L21 X11), as products over all 256 threads (three
  // barriers per level).  (A single forward substitution per column of the
  // 64x64 block was a 64-long dependent chain per thread: 51 us per 512x512
  // inverse, as was the column-oriented elimination before it.)
  T* Tmp = &Xs[0][0] + (size_t)kInvBS * (kInvBS + 1);  // [bs * 16] products of one level
  if (tid < bs) {
    const int b0l = tid & ~15, col = tid;
    Xs[col][col] = T(1) / Ls[col][col];
    for (int i = col + 1; i < b0l + 16 && i < bs; ++i) {
      T a0 = T(0), a1 = T(0);
      int k = col;
      for (; k + 1 < i; k += 2) {
        a0 = fma(Ls[i][k], Xs[k][col], a0);
        a1 = fma(Ls[i][k + 1], Xs[k + 1][col], a1);
      }
      if (k < i) a0 = fma(Ls[i][k], Xs[k][col], a0);
      Xs[i][col] = -(a0 + a1) / Ls[i][i];
    }
  }
  __syncthreads();
  for (int h = 16; h < bs; h *= 2) {
    const int hh = h * h, nout = (bs / (2 * h)) * hh;
    for (int idx = tid; idx < nout; idx += blockDim.x) {  // Tmp_p = L21_p X11_p
      const int pp = idx / hh, e = idx - pp * hh, r = e % h, c = e / h, o = 2 * h * pp;
      T acc = T(0);
      for (int t = c; t < h; ++t) acc = fma(Ls[o + h + r][o + t], Xs[o + t][o + c], acc);  // X11 lower
      Tmp[idx] = acc;
    }
    __syncthreads();
    for (int idx = tid; idx < nout; idx += blockDim.x) {  // X21_p = -X22_p Tmp_p
      const int pp = idx / hh, e = idx - pp * hh, r = e % h, c = e / h, o = 2 * h * pp;
      T acc = T(0);
      for (int t = 0; t <= r; ++t) acc = fma(Xs[o + h + r][o + h + t], Tmp[pp * hh + t + c * h], acc);  // X22 lower
      Xs[o + h + r][o + c] = -acc;
    }
    __syncthreads();
  }
  for (int idx = tid; idx < bs * bs; idx += blockDim.x) {
    const int i = idx % bs, jj = idx / bs;
    if (upper)  // W = X^T
      W[(b0 + i) + (int64_t)(b0 + jj) * ldw] = Xs[jj][i];
    else
      W[(b0 + i) + (int64_t)(b0 + jj) * ldw] = Xs[i][jj];
  }
}

static cublasStatus_t gemm_sb(cublasHandle_t h, cublasOperation_t ta, cublasOperation_t tb, int m, int n, int k,
                              const double* al, const double* A, int lda, long long sa, const double* B, int ldb,
                              long long sb, const double* be, double* C, int ldc, long long sc, int batch) {
  return cublasDgemmStridedBatched(h, ta, tb, m, n, k, al, A, lda, sa, B, ldb, sb, be, C, ldc, sc, batch);
}
static cublasStatus_t gemm_sb(cublasHandle_t h, cublasOperation_t ta, cublasOperation_t tb, int m, int n, int k,
                              const float* al, const float* A, int lda, long long sa, const float* B, int ldb,
                              long long sb, const float* be, float* C, int ldc, long long sc, int batch) {
  return cublasSgemmStridedBatched(h, ta, tb, m, n, k, al, A, lda, sa, B, ldb, sb, be, C, ldc, sc, batch);
}

template <typename T>
int tri_inverse_t(char uplo, char diag, int nb, const T* Tm, int ldt, T* W, int ldw, cudaStream_t s) {
  const bool upper = uplo == 'U' || uplo == 'u', unit = diag == 'U' || diag == 'u';
  const int bs = nb < kInvBS ? nb : kInvBS;
  if (nb % bs) return ABFT_E_UNSUPPORTED;
  ABFT_CUDA_TRY(cudaMemset2DAsync(W, (size_t)ldw * sizeof(T), 0, (size_t)nb * sizeof(T), nb, s));
  const size_t smem = (2 * kInvBS * (kInvBS + 1) + (size_t)kInvBS * 16) * sizeof(T);
  static bool attr = false;
  if (!attr) {
    ABFT_CUDA_TRY(cudaFuncSetAttribute(tri_inv_base_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    attr = true;
  }
  tri_inv_base_kernel<T><<<nb / bs, 256, smem, s>>>(Tm, ldt, W, ldw, bs, upper, unit);
  ABFT_CUDA_TRY(cudaGetLastError());
  if (bs == nb) return 0;
  void* tv = nullptr;
  int rc = scratch_get(s, 9, (size_t)nb * nb / 2 * sizeof(T), &tv);
  if (rc) return rc;
  T* tmp = reinterpret_cast<T*>(tv);
  std::unique_lock<std::mutex> lk;
  cublasHandle_t h = blas_handle(s, lk);
  const T one = T(1), zero = T(0), mone = T(-1);
  for (int sz = bs; sz < nb; sz *= 2) {
    const int batch = nb / (2 * sz);
    const long long sW = (long long)(2 * sz) * (1 + ldw), sT = (long long)(2 * sz) * (1 + ldt);
    const long long sTmp = (long long)sz * sz;
    const T* Ai = W;                                  // A^-1 at (0,0) of each pair
    const T* Ci = W + sz + (int64_t)sz * ldw;         // C^-1 at (s,s)
    if (!upper) {
      const T* B = Tm + sz;                           // B at (s,0) of T
      T* X = W + sz;                                  // result block (s,0) of W
      ABFT_CUBLAS_TRY(gemm_sb(h, CUBLAS_OP_N, CUBLAS_OP_N, sz, sz, sz, &one, B, ldt, sT, Ai, ldw, sW, &zero, tmp, sz,
                              sTmp, batch));
      ABFT_CUBLAS_TRY(gemm_sb(h, CUBLAS_OP_N, CUBLAS_OP_N, sz, sz, sz, &mone, Ci, ldw, sW, tmp, sz, sTmp, &zero, X, ldw,
                              sW, batch));
    } else {
      const T* B = Tm + (int64_t)sz * ldt;            // B at (0,s) of T
      T* X = W + (int64_t)sz * ldw;                   // result block (0,s) of W
      ABFT_CUBLAS_TRY(gemm_sb(h, CUBLAS_OP_N, CUBLAS_OP_N, sz, sz, sz, &one, Ai, ldw, sW, B, ldt, sT, &zero, tmp, sz,
                              sTmp, batch));
      ABFT_CUBLAS_TRY(gemm_sb(h, CUBLAS_OP_N, CUBLAS_OP_N, sz, sz, sz, &mone, tmp, sz, sTmp, Ci, ldw, sW, &zero, X, ldw,
                              sW, batch));
    }
  }
  return 0;
}

// out (rows x cols, ld ldo) <- tmp (ld rows): stream-ordered copy back
template <typename T>
static int copy_back(T* out, int64_t ldo, const T* tmp, int64_t rows, int64_t cols, cudaStream_t s) {
  return abft::copy2d(out, ldo * sizeof(T), tmp, rows * sizeof(T), rows * sizeof(T), cols, s);
}

// a5 with a precomputed inverse W = T^-1:
//   side R: chk (nvec x nb) <- chk * op(W);  mag (nmag x nb) <- mag * |op(W)|
//   side L: chk (nb x nvec) <- op(W) * chk;  mag (nb x nmag) <- |op(W)| * mag
int trsm_inv_rule(char side, char trans, int64_t nb, const double* W, int64_t ldw, double* chk, int64_t ldchk,
                  int64_t nvec, double* mag, int64_t ldmag, int64_t nmag, cudaStream_t s);  // abft_rule_small.cu

template <typename T>
int update_trsm_inv_t(char side, char trans, int64_t nb, const T* W, int64_t ldw, T* chk, int64_t ldchk, int64_t nvec,
                      T* mag, int64_t ldmag, int64_t nmag, cudaStream_t s) {
  // fp64: one clustered in-place DMMA launch (abft_rule_small.cu);
  // ABFT_RULE_CUBLAS=1 keeps the library route below (GEMM into scratch +
  // copy back per array), as fp32 and nb = 1024 do
  static const bool gemm_route = getenv("ABFT_RULE_CUBLAS") != nullptr;
  if constexpr (std::is_same<T, double>::value) {
    if (!gemm_route) {
      const int r = trsm_inv_rule(side, trans, nb, W, ldw, chk, ldchk, nvec, mag, ldmag, nmag, s);
      if (r != ABFT_E_UNSUPPORTED) return r;
    }
  }
  const bool left = side == 'L' || side == 'l';
  const cublasOperation_t oW = op_of(trans);
  const T one = T(1), zero = T(0);
  const int64_t nmax = nvec > nmag ? nvec : nmag;
  if (nmax <= 0) return 0;
  void* tv = nullptr;
  int rc = scratch_get(s, 2, (size_t)nb * nmax * sizeof(T), &tv);
  if (rc) return rc;
  T* tmp = reinterpret_cast<T*>(tv);
  std::unique_lock<std::mutex> lk;
  cublasHandle_t h = blas_handle(s, lk);
  if (nvec > 0) {
    if (!left) {
      ABFT_CUBLAS_TRY(gemm(h, CUBLAS_OP_N, oW, (int)nvec, (int)nb, (int)nb, &one, chk, (int)ldchk, W, (int)ldw, &zero,
                           tmp, (int)nvec));
      rc = copy_back<T>(chk, ldchk, tmp, nvec, nb, s);
    } else {
      ABFT_CUBLAS_TRY(gemm(h, oW, CUBLAS_OP_N, (int)nb, (int)nvec, (int)nb, &one, W, (int)ldw, chk, (int)ldchk, &zero,
                           tmp, (int)nb));
      rc = copy_back<T>(chk, ldchk, tmp, nb, nvec, s);
    }
    if (rc) return rc;
  }
  if (mag && nmag > 0) {
    void* av = nullptr;
    rc = scratch_get(s, 1, (size_t)nb * nb * sizeof(T), &av);
    if (rc) return rc;
    T* aW = reinterpret_cast<T*>(av);
    rc = abs_copy<T>(aW, W, nb, nb, ldw, s);
    if (rc) return rc;
    if (!left) {
      ABFT_CUBLAS_TRY(gemm(h, CUBLAS_OP_N, oW, (int)nmag, (int)nb, (int)nb, &one, mag, (int)ldmag, aW, (int)nb, &zero,
                           tmp, (int)nmag));
      rc = copy_back<T>(mag, ldmag, tmp, nmag, nb, s);
    } else {
      ABFT_CUBLAS_TRY(gemm(h, oW, CUBLAS_OP_N, (int)nb, (int)nmag, (int)nb, &one, aW, (int)nb, mag, (int)ldmag, &zero,
                           tmp, (int)nb));
      rc = copy_back<T>(mag, ldmag, tmp, nb, nmag, s);
    }
    if (rc) return rc;
  }
  return 0;
}

template <typename T>
int update_trsm_t(char side, char uplo, char trans, char diag, int64_t nb, const void* Tv, int64_t ldt, void* chkv,
                  int64_t ldchk, int64_t nvec, void* magv, int64_t ldmag, int64_t nmag, cudaStream_t s) {
  void* wv = nullptr;
  int rc = scratch_get(s, 5, (size_t)nb * nb * sizeof(T), &wv);
  if (rc) return rc;
  T* W = reinterpret_cast<T*>(wv);
  rc = tri_inverse_t<T>(uplo, diag, (int)nb, reinterpret_cast<const T*>(Tv), (int)ldt, W, (int)nb, s);
  if (rc) return rc;
  return update_trsm_inv_t<T>(side, trans, nb, W, nb, reinterpret_cast<T*>(chkv), ldchk, nvec,
                              reinterpret_cast<T*>(magv), ldmag, nmag, s);
}

// Cholesky TMU checksum rule from ONE product (c-12, L189).  P = c(L21) L21^T
// (M2 x nk) gives c(A_IJ) -= P[2I.., cols of J] for I >= J and, transposed,
// r(A_IJ) -= P[2J.., cols of I]^T for I >= J.  Magnitudes from
// Q = m_c(L21) |L21|^T likewise (c-6).
template <typename T>
__global__ void syrk_scatter_col_kernel(T* __restrict__ C, int64_t ldc, const T* __restrict__ P, int64_t M, int64_t nk,
                                        int nb, int rows_per_tile, T sign) {
  const int64_t total = M * nk;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    const int64_t x = idx / M, y = idx - x * M;
    if (y / rows_per_tile >= x / nb) C[y + x * ldc] += sign * P[idx];
  }
}
template <typename T>
__global__ void syrk_scatter_row_kernel(T* __restrict__ R, int64_t ldr, const T* __restrict__ P, int64_t M, int64_t nk,
                                        int nb, int rows_per_tile, T sign) {
  const int64_t total = M * nk;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    const int64_t y = idx / nk, x = idx - y * nk;
    if (x / nb >= y / rows_per_tile) R[x + y * ldr] += sign * P[y + x * M];
  }
}

// Both scatters from one read of P (nb % 32 == 0): a block owns a 32 x 32
// piece of P (32 columns x inside one tile column J = x / nb), stages it in
// shared memory, adds them to C with y as the fast index and to R, through
// the transpose, with x as the fast index — coalesced on both sides.  Same
// element operations as the two kernels above (bit-identical results).
template <typename T>
__global__ void __launch_bounds__(256) syrk_scatter_kernel(T* __restrict__ C, int64_t ldc, T* __restrict__ R,
                                                           int64_t ldr, const T* __restrict__ P, int64_t M,
                                                           int64_t nk, int nb, int rows_per_tile, T sign) {
  __shared__ T tile[32][33];
  const int64_t x0 = (int64_t)blockIdx.x * 32, y0 = (int64_t)blockIdx.y * 32;
  const int64_t J = x0 / nb;
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
#pragma unroll
  for (int j = ty; j < 32; j += 8) {
    const int64_t x = x0 + j, y = y0 + tx;
    const bool in = x < nk && y < M;
    const T v = in ? P[y + x * M] : T(0);
    tile[j][tx] = v;
    if (in && y / rows_per_tile >= J) C[y + x * ldc] += sign * v;
  }
  if (!R) return;
  __syncthreads();
#pragma unroll
  for (int i = ty; i < 32; i += 8) {
    const int64_t y = y0 + i, x = x0 + tx;
    if (x < nk && y < M && J >= y / rows_per_tile) R[x + y * ldr] += sign * tile[tx][i];
  }
}

template <typename T>
static void scatter_both(T* C, int64_t ldc, T* R, int64_t ldr, const T* P, int64_t M, int64_t nk, int64_t nb, int rpt,
                         T sign, cudaStream_t s) {
  if (nb % 32 == 0) {
    const dim3 grid((unsigned)((nk + 31) / 32), (unsigned)((M + 31) / 32));
    syrk_scatter_kernel<T><<<grid, 256, 0, s>>>(C, ldc, R, ldr, P, M, nk, (int)nb, rpt, sign);
    return;
  }
  syrk_scatter_col_kernel<T><<<grid_for(M * nk), 256, 0, s>>>(C, ldc, P, M, nk, (int)nb, rpt, sign);
  if (R) syrk_scatter_row_kernel<T><<<grid_for(M * nk), 256, 0, s>>>(R, ldr, P, M, nk, (int)nb, rpt, sign);
}

template <typename T>
int update_syrk_t(int64_t nb, int64_t ntk, const T* L21, int64_t ldl, const T* cL, int64_t ldc, const T* mL,
                  int64_t ldcm, T* Cc, T* Rr, int64_t ldr, T* Cm, T* Rm, int64_t ldrm, cudaStream_t s) {
  const int64_t nk = ntk * nb, M2 = 2 * ntk;
  if (nk == 0) return 0;
  if constexpr (sizeof(T) == 8) {
    // fp64: one fused DMMA kernel (abft_rule_dmma.cu); ABFT_RULE_CUBLAS=1 keeps
    // the GEMM route below (A/B measurements)
    static const bool gemm_route = getenv("ABFT_RULE_CUBLAS") != nullptr;
    if (!gemm_route) {
      const int r = update_syrk_dmma(nb, ntk, L21, ldl, cL, ldc, mL, ldcm, Cc, Rr, ldr, Cm, Rm, ldrm, s);
      if (r != ABFT_E_UNSUPPORTED) return r;
    }
  }
  void* pv = nullptr;
  int rc = scratch_get(s, 7, (size_t)M2 * nk * sizeof(T), &pv);
  if (rc) return rc;
  T* P = reinterpret_cast<T*>(pv);
  const T one = T(1), zero = T(0);
  {
    std::unique_lock<std::mutex> lk;
    cublasHandle_t h = blas_handle(s, lk);
    ABFT_CUBLAS_TRY(gemm(h, CUBLAS_OP_N, CUBLAS_OP_T, (int)M2, (int)nk, (int)nb, &one, cL, (int)ldc, L21, (int)ldl,
                         &zero, P, (int)M2));
  }
  scatter_both<T>(Cc, ldc, Rr, ldr, P, M2, nk, nb, 2, T(-1), s);
  ABFT_CUDA_TRY(cudaGetLastError());
  if (mL && Cm) {
    void* av = nullptr;
    rc = scratch_get(s, 3, (size_t)nk * nb * sizeof(T), &av);
    if (rc) return rc;
    T* aL = reinterpret_cast<T*>(av);
    rc = abs_copy<T>(aL, L21, nk, nb, ldl, s);
    if (rc) return rc;
    {
      std::unique_lock<std::mutex> lk;
      cublasHandle_t h = blas_handle(s, lk);
      ABFT_CUBLAS_TRY(gemm(h, CUBLAS_OP_N, CUBLAS_OP_T, (int)ntk, (int)nk, (int)nb, &one, mL, (int)ldcm, aL, (int)nk,
                           &zero, P, (int)ntk));
    }
    scatter_both<T>(Cm, ldcm, Rm, ldrm, P, ntk, nk, nb, 1, T(1), s);
    ABFT_CUDA_TRY(cudaGetLastError());
  }
  return 0;
}

template <typename T>
int update_gemm_t(int which, char transX, char transY, double alpha, const void* Xv, int64_t ldx, const void* Yv,
                  int64_t ldy, void* Cv, int64_t ldcc, int64_t M2, int64_t N, int64_t K, const void* Xmv,
                  int64_t ldxm, void* Cmv, int64_t ldcm, cudaStream_t s) {
  if (M2 == 0 || N == 0) return 0;
  // fp64: one DMMA launch (abft_rule_dmma.cu); ABFT_RULE_CUBLAS=1 keeps the
  // library route below (|op(Y)| copy + two GEMMs), as fp32 does
  static const bool gemm_route = getenv("ABFT_RULE_CUBLAS") != nullptr;
  if constexpr (std::is_same<T, double>::value) {
    if (!gemm_route) {
      const int r = update_gemm_dmma(which, transX, transY, alpha, (const double*)Xv, ldx, (const double*)Yv, ldy,
                                     (double*)Cv, ldcc, M2, N, K, (const double*)Xmv, ldxm, (double*)Cmv, ldcm, s);
      if (r != ABFT_E_UNSUPPORTED) return r;
    }
  }
  std::unique_lock<std::mutex> lk;
  cublasHandle_t h = blas_handle(s, lk);
  const T* X = reinterpret_cast<const T*>(Xv);
  const T* Y = reinterpret_cast<const T*>(Yv);
  T* C = reinterpret_cast<T*>(Cv);
  const T al = T(alpha), one = T(1);
  const cublasOperation_t oX = op_of(transX), oY = op_of(transY);
  if (which == ABFT_COL) {  // C (M2 x N) += al op(X)(M2 x K) op(Y)(K x N)
    ABFT_CUBLAS_TRY(gemm(h, oX, oY, (int)M2, (int)N, (int)K, &al, X, (int)ldx, Y, (int)ldy, &one, C, (int)ldcc));
  } else {  // C (N x M2) += al op(Y)(N x K) op(X)(K x M2)
    ABFT_CUBLAS_TRY(gemm(h, oY, oX, (int)N, (int)M2, (int)K, &al, Y, (int)ldy, X, (int)ldx, &one, C, (int)ldcc));
  }
  if (Xmv && Cmv) {
    // |op(Y)|: materialise the stored region of Y in scratch slot 3
    const bool yT = oY == CUBLAS_OP_T;
    int64_t yr, yc;  // stored shape of Y
    if (which == ABFT_COL) {
      yr = yT ? N : K;
      yc = yT ? K : N;
    } else {
      yr = yT ? K : N;
      yc = yT ? N : K;
    }
    void* av = nullptr;
    int rc = scratch_get(s, 3, (size_t)yr * yc * sizeof(T), &av);
    if (rc) return rc;
    T* aY = reinterpret_cast<T*>(av);
    rc = abs_copy<T>(aY, Y, yr, yc, ldy, s);
    if (rc) return rc;
    const T* Xm = reinterpret_cast<const T*>(Xmv);
    T* Cm = reinterpret_cast<T*>(Cmv);
    const T aal = T(alpha < 0 ? -alpha : alpha);
    const int64_t M = M2 / 2;
    if (which == ABFT_COL)
      ABFT_CUBLAS_TRY(gemm(h, oX, oY, (int)M, (int)N, (int)K, &aal, Xm, (int)ldxm, aY, (int)yr, &one, Cm, (int)ldcm));
    else
      ABFT_CUBLAS_TRY(gemm(h, oY, oX, (int)N, (int)M, (int)K, &aal, aY, (int)yr, Xm, (int)ldxm, &one, Cm, (int)ldcm));
  }
  return 0;
}

// Row checksums of one trailing tile column J0 after the Cholesky TMU
// (c-12, L189; the look-ahead's first part, reading c-35), every row x of the
// panel L (rows x nb):
//   r_e(x) -= sum_q L[x,q] c_e(L_J0)[q],  r_w(x) -= sum_q L[x,q] c_w(L_J0)[q],
//   m_r(x) += sum_q |L[x,q]| m_c(L_J0)[q]            (c-6)
// in ONE pass over L (the GEMM route needs |L| materialised first).  A block
// owns 32 rows; its 8 warps split the nb columns and their partials are
// added in warp order (deterministic).  Memory-latency bound at the panel
// sizes of late iterations: each lane keeps 16 column loads in flight (one
// load at a time ran 36 us per launch whatever the panel height, ncu r02a).
template <typename T>
__global__ void __launch_bounds__(256) panel_row_rule_kernel(int64_t rows, int nb, const T* __restrict__ L, int64_t ldl,
                                                             const T* __restrict__ ce, const T* __restrict__ cw,
                                                             int64_t ldc, const T* __restrict__ mc, int64_t ldcm,
                                                             T* __restrict__ re, T* __restrict__ rw,
                                                             T* __restrict__ rm) {
  // the tile column's checksum vectors, staged once per block
  __shared__ T sv[3][1024];
  __shared__ T part[8][3][32];
  for (int q = threadIdx.x; q < nb; q += blockDim.x) {
    sv[0][q] = ce[(int64_t)q * ldc];
    sv[1][q] = cw[(int64_t)q * ldc];
    sv[2][q] = mc ? mc[(int64_t)q * ldcm] : T(0);
  }
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t x = (int64_t)blockIdx.x * 32 + lane;
  const int qn = nb / 8, q0 = warp * qn;
  T se = T(0), sw = T(0), sm = T(0);
  if (x < rows) {
    // 16 independent column loads in flight per lane, then the same
    // sequential fma chain as one column at a time
    const T* Lx = L + x + (int64_t)q0 * ldl;
    for (int q = 0; q < qn; q += 16) {
      T l[16];
#pragma unroll
      for (int u = 0; u < 16; ++u) l[u] = q + u < qn ? __ldg(Lx + (int64_t)(q + u) * ldl) : T(0);
#pragma unroll
      for (int u = 0; u < 16; ++u) {
        if (q + u < qn) {
          se = fma(l[u], sv[0][q0 + q + u], se);
          sw = fma(l[u], sv[1][q0 + q + u], sw);
          sm = fma(fabs(l[u]), sv[2][q0 + q + u], sm);
        }
      }
    }
  }
  part[warp][0][lane] = se;
  part[warp][1][lane] = sw;
  part[warp][2][lane] = sm;
  __syncthreads();
  if (warp == 0 && x < rows) {
    T e = T(0), w = T(0), m = T(0);
#pragma unroll
    for (int g = 0; g < 8; ++g) {
      e += part[g][0][lane];
      w += part[g][1][lane];
      m += part[g][2][lane];
    }
    re[x] -= e;
    rw[x] -= w;
    if (rm) rm[x] += m;
  }
}

// The same rule with two rows per lane (16-B / 8-B vector loads: a warp
// reads 64 consecutive rows of a column, 512 B for fp64) and 8 loads in
// flight per lane; a block owns 64 rows.  The scalar version above ran the
// n=30720 first-iteration panel (124 MB) at 3.0 TB/s, latency-bound (ncu:
// 25 cycles per issued instruction, 43% occupancy).
template <typename T, typename V2>
__global__ void __launch_bounds__(256) panel_row_rule2_kernel(int64_t rows, int nb, const T* __restrict__ L,
                                                              int64_t ldl, const T* __restrict__ ce,
                                                              const T* __restrict__ cw, int64_t ldc,
                                                              const T* __restrict__ mc, int64_t ldcm,
                                                              T* __restrict__ re, T* __restrict__ rw,
                                                              T* __restrict__ rm) {
  __shared__ T sv[3][1024];
  __shared__ T part[8][3][64];
  for (int q = threadIdx.x; q < nb; q += blockDim.x) {
    sv[0][q] = ce[(int64_t)q * ldc];
    sv[1][q] = cw[(int64_t)q * ldc];
    sv[2][q] = mc ? mc[(int64_t)q * ldcm] : T(0);
  }
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t x = (int64_t)blockIdx.x * 64 + 2 * lane;  // this lane's rows x, x + 1
  const int qn = nb / 8, q0 = warp * qn;
  T se0 = T(0), sw0 = T(0), sm0 = T(0), se1 = T(0), sw1 = T(0), sm1 = T(0);
  if (x < rows) {  // rows is even: both rows exist
    const T* Lx = L + x + (int64_t)q0 * ldl;
    for (int q = 0; q < qn; q += 8) {
      V2 l[8];
#pragma unroll
      for (int u = 0; u < 8; ++u)
        if (q + u < qn) l[u] = __ldg(reinterpret_cast<const V2*>(Lx + (int64_t)(q + u) * ldl));
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        if (q + u < qn) {
          const T a = sv[0][q0 + q + u], b = sv[1][q0 + q + u], c = sv[2][q0 + q + u];
          se0 = fma(l[u].x, a, se0);
          sw0 = fma(l[u].x, b, sw0);
          sm0 = fma(fabs(l[u].x), c, sm0);
          se1 = fma(l[u].y, a, se1);
          sw1 = fma(l[u].y, b, sw1);
          sm1 = fma(fabs(l[u].y), c, sm1);
        }
      }
    }
  }
  part[warp][0][2 * lane] = se0;
  part[warp][1][2 * lane] = sw0;
  part[warp][2][2 * lane] = sm0;
  part[warp][0][2 * lane + 1] = se1;
  part[warp][1][2 * lane + 1] = sw1;
  part[warp][2][2 * lane + 1] = sm1;
  __syncthreads();
  // 64 rows x 3 sums, warp order (deterministic); threads 0..63 finish one row each
  const int r = threadIdx.x;
  const int64_t xr = (int64_t)blockIdx.x * 64 + r;
  if (r < 64 && xr < rows) {
    T e = T(0), w = T(0), m = T(0);
#pragma unroll
    for (int g = 0; g < 8; ++g) {
      e += part[g][0][r];
      w += part[g][1][r];
      m += part[g][2][r];
    }
    re[xr] -= e;
    rw[xr] -= w;
    if (rm) rm[xr] += m;
  }
}

int panel_row_rule(int32_t dtype, int64_t rows, int64_t nb, const void* L, int64_t ldl, const void* ce, const void* cw,
                   int64_t ldc, const void* mc, int64_t ldcm, void* re, void* rw, void* rm, cudaStream_t s) {
  if (rows <= 0) return 0;
  if (nb % 8 || nb > 1024) return ABFT_E_UNSUPPORTED;
  const size_t es = dtype == ABFT_F64 ? 8 : 4;
  if (rows % 2 == 0 && (uintptr_t)L % (2 * es) == 0 && (ldl * es) % (2 * es) == 0) {
    const unsigned grid2 = (unsigned)((rows + 63) / 64);
    if (dtype == ABFT_F64)
      panel_row_rule2_kernel<double, double2><<<grid2, 256, 0, s>>>(
          rows, (int)nb, (const double*)L, ldl, (const double*)ce, (const double*)cw, ldc, (const double*)mc, ldcm,
          (double*)re, (double*)rw, (double*)rm);
    else
      panel_row_rule2_kernel<float, float2><<<grid2, 256, 0, s>>>(
          rows, (int)nb, (const float*)L, ldl, (const float*)ce, (const float*)cw, ldc, (const float*)mc, ldcm,
          (float*)re, (float*)rw, (float*)rm);
    ABFT_CUDA_TRY(cudaGetLastError());
    return 0;
  }
  const unsigned grid = (unsigned)((rows + 31) / 32);
  if (dtype == ABFT_F64)
    panel_row_rule_kernel<double><<<grid, 256, 0, s>>>(rows, (int)nb, (const double*)L, ldl, (const double*)ce,
                                                       (const double*)cw, ldc, (const double*)mc, ldcm, (double*)re,
                                                       (double*)rw, (double*)rm);
  else
    panel_row_rule_kernel<float><<<grid, 256, 0, s>>>(rows, (int)nb, (const float*)L, ldl, (const float*)ce,
                                                      (const float*)cw, ldc, (const float*)mc, ldcm, (float*)re,
                                                      (float*)rw, (float*)rm);
  ABFT_CUDA_TRY(cudaGetLastError());
  return 0;
}

}  // namespace abft

extern "C" int abft_update_trsm(int32_t dtype, char side, char uplo, char trans, char diag, int64_t nb, const void* T,
                                int64_t ldt, void* chk, int64_t ldchk, int64_t nvec, void* mag, int64_t ldmag,
                                int64_t nmag, abft_stream_t stream) {
  if (dtype != ABFT_F32 && dtype != ABFT_F64) return -1;
  if (side != 'L' && side != 'R') return -2;
  if (uplo != 'L' && uplo != 'U') return -3;
  if (trans != 'N' && trans != 'T') return -4;
  if (diag != 'N' && diag != 'U') return -5;
  if (nb <= 0) return -6;
  if (!T || ldt < nb) return -7;
  if (nvec < 0) return -11;
  if (nvec > 0 && (!chk || ldchk < (side == 'R' ? nvec : nb))) return -10;
  if (mag && nmag > 0 && ldmag < (side == 'R' ? nmag : nb)) return -13;
  cudaStream_t s = (cudaStream_t)stream;
  return dtype == ABFT_F64 ? abft::update_trsm_t<double>(side, uplo, trans, diag, nb, T, ldt, chk, ldchk, nvec, mag,
                                                         ldmag, nmag, s)
                           : abft::update_trsm_t<float>(side, uplo, trans, diag, nb, T, ldt, chk, ldchk, nvec, mag,
                                                        ldmag, nmag, s);
}

extern "C" int abft_update_gemm(int32_t dtype, int32_t which, char transX, char transY, double alpha, const void* Xchk,
                                int64_t ldx, const void* Y, int64_t ldy, void* Cchk, int64_t ldcc, int64_t M2,
                                int64_t N, int64_t K, const void* Xmag, int64_t ldxm, void* Cmag, int64_t ldcm,
                                abft_stream_t stream) {
  if (dtype != ABFT_F32 && dtype != ABFT_F64) return -1;
  if (which != ABFT_COL && which != ABFT_ROW) return -2;
  if (transX != 'N' && transX != 'T') return -3;
  if (transY != 'N' && transY != 'T') return -4;
  if (M2 < 0 || M2 % 2) return -12;
  if (N < 0) return -13;
  if (K < 0) return -14;
  if (!Xchk || !Y || !Cchk) return -6;
  if ((Xmag == nullptr) != (Cmag == nullptr)) return -15;
  cudaStream_t s = (cudaStream_t)stream;
  return dtype == ABFT_F64
             ? abft::update_gemm_t<double>(which, transX, transY, alpha, Xchk, ldx, Y, ldy, Cchk, ldcc, M2, N, K,
                                           Xmag, ldxm, Cmag, ldcm, s)
             : abft::update_gemm_t<float>(which, transX, transY, alpha, Xchk, ldx, Y, ldy, Cchk, ldcc, M2, N, K,
                                          Xmag, ldxm, Cmag, ldcm, s);
}

extern "C" int abft_tri_inverse(int32_t dtype, char uplo, char diag, int64_t nb, const void* T, int64_t ldt, void* W,
                                int64_t ldw, abft_stream_t stream) {
  if (dtype != ABFT_F32 && dtype != ABFT_F64) return -1;
  if (uplo != 'L' && uplo != 'U') return -2;
  if (diag != 'N' && diag != 'U') return -3;
  if (nb <= 0) return -4;
  if (!T || ldt < nb) return -5;
  if (!W || ldw < nb) return -7;
  cudaStream_t s = (cudaStream_t)stream;
  return dtype == ABFT_F64
             ? abft::tri_inverse_t<double>(uplo, diag, (int)nb, (const double*)T, (int)ldt, (double*)W, (int)ldw, s)
             : abft::tri_inverse_t<float>(uplo, diag, (int)nb, (const float*)T, (int)ldt, (float*)W, (int)ldw, s);
}

extern "C" int abft_update_trsm_inv(int32_t dtype, char side, char trans, int64_t nb, const void* W, int64_t ldw,
                                    void* chk, int64_t ldchk, int64_t nvec, void* mag, int64_t ldmag, int64_t nmag,
                                    abft_stream_t stream) {
  if (dtype != ABFT_F32 && dtype != ABFT_F64) return -1;
  if (side != 'L' && side != 'R') return -2;
  if (trans != 'N' && trans != 'T') return -3;
  if (nb <= 0) return -4;
  if (!W || ldw < nb) return -5;
  if (nvec < 0) return -9;
  if (nvec > 0 && (!chk || ldchk < (side == 'R' ? nvec : nb))) return -7;
  if (mag && nmag > 0 && ldmag < (side == 'R' ? nmag : nb)) return -11;
  cudaStream_t s = (cudaStream_t)stream;
  if (dtype == ABFT_F64)
    return abft::update_trsm_inv_t<double>(side, trans, nb, (const double*)W, ldw, (double*)chk, ldchk, nvec,
                                           (double*)mag, ldmag, nmag, s);
  return abft::update_trsm_inv_t<float>(side, trans, nb, (const float*)W, ldw, (float*)chk, ldchk, nvec, (float*)mag,
                                        ldmag, nmag, s);
}

extern "C" int abft_update_syrk(int32_t dtype, int64_t nb, int64_t ntk, const void* L21, int64_t ldl, const void* cL,
                                int64_t ldc, const void* mL, int64_t ldcm, void* Cc, void* Rr, int64_t ldr, void* Cm,
                                void* Rm, int64_t ldrm, abft_stream_t stream) {
  if (dtype != ABFT_F32 && dtype != ABFT_F64) return -1;
  if (nb <= 0) return -2;
  if (ntk < 0) return -3;
  if (ntk == 0) return 0;
  if (!L21 || ldl < ntk * nb) return -4;
  if (!cL || !Cc || ldc < 2 * ntk) return -6;
  if (Rr && ldr < ntk * nb) return -11;
  if (mL && (!Cm || (Rr && !Rm) || ldcm < ntk || (Rm && ldrm < ntk * nb))) return -8;
  cudaStream_t s = (cudaStream_t)stream;
  if (dtype == ABFT_F64)
    return abft::update_syrk_t<double>(nb, ntk, (const double*)L21, ldl, (const double*)cL, ldc, (const double*)mL,
                                       ldcm, (double*)Cc, (double*)Rr, ldr, (double*)Cm, (double*)Rm, ldrm, s);
  return abft::update_syrk_t<float>(nb, ntk, (const float*)L21, ldl, (const float*)cL, ldc, (const float*)mL, ldcm,
                                    (float*)Cc, (float*)Rr, ldr, (float*)Cm, (float*)Rm, ldrm, s);
}
