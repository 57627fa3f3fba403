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
#include <unordered_map>

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
Handles& handles_for_device() {
  static auto* m = new std::unordered_map<int, Handles*>();
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> g(g_hmu);
  auto it = m->find(dev);
  if (it != m->end()) return *it->second;
  Handles* h = new Handles();
  cublasCreate(&h->blas);
  cusolverDnCreate(&h->solver);
  (*m)[dev] = h;
  return *h;
}

// Scratch buffers private to the update ops (distinct from the pass pools).
struct Scratch {
  void* p = nullptr;
  size_t bytes = 0;
};
std::mutex g_smu;
int scratch_get(cudaStream_t s, int slot, size_t bytes, void** out) {
  static auto* m = new std::unordered_map<uint64_t, Scratch>();
  int dev = 0;
  cudaGetDevice(&dev);
  uint64_t key = (reinterpret_cast<uint64_t>(s) << 12) ^ ((uint64_t)dev << 4) ^ (uint64_t)slot;
  std::lock_guard<std::mutex> g(g_smu);
  Scratch& sc = (*m)[key];
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
  Handles& h = handles_for_device();
  lk = std::unique_lock<std::mutex>(h.mu);
  cublasSetStream(h.blas, s);
  return h.blas;
}
cusolverDnHandle_t solver_handle(cudaStream_t s, std::unique_lock<std::mutex>& lk) {
  Handles& h = handles_for_device();
  lk = std::unique_lock<std::mutex>(h.mu);
  cusolverDnSetStream(h.solver, s);
  cublasSetStream(h.blas, s);
  return h.solver;
}
int scratch(cudaStream_t s, int slot, size_t bytes, void** out) { return scratch_get(s, slot, bytes, out); }

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
static cublasStatus_t trsm(cublasHandle_t h, cublasSideMode_t sd, cublasFillMode_t ul, cublasOperation_t tr,
                           cublasDiagType_t dg, int m, int n, const double* al, const double* A, int lda, double* B,
                           int ldb) {
  return cublasDtrsm(h, sd, ul, tr, dg, m, n, al, A, lda, B, ldb);
}
static cublasStatus_t trsm(cublasHandle_t h, cublasSideMode_t sd, cublasFillMode_t ul, cublasOperation_t tr,
                           cublasDiagType_t dg, int m, int n, const float* al, const float* A, int lda, float* B,
                           int ldb) {
  return cublasStrsm(h, sd, ul, tr, dg, m, n, al, A, lda, B, ldb);
}

static cublasOperation_t op_of(char t) { return (t == 'T' || t == 't') ? CUBLAS_OP_T : CUBLAS_OP_N; }

// |op(T)^-1| (nb x nb, ld nb) into scratch slot 1.
template <typename T>
int abs_tri_inverse(cublasHandle_t h, char side, char uplo, char trans, char diag, int nb, const T* Tm, int ldt,
                    cudaStream_t s, T** out) {
  void* w = nullptr;
  int rc = scratch_get(s, 1, (size_t)nb * nb * sizeof(T), &w);
  if (rc) return rc;
  T* W = reinterpret_cast<T*>(w);
  identity_kernel<T><<<grid_for((int64_t)nb * nb), 256, 0, s>>>(W, nb);
  ABFT_CUDA_TRY(cudaGetLastError());
  const T one = T(1);
  // W = I * op(T)^-1 (right) or op(T)^-1 * I (left) -- the same matrix
  ABFT_CUBLAS_TRY(trsm(h, (side == 'L' || side == 'l') ? CUBLAS_SIDE_LEFT : CUBLAS_SIDE_RIGHT,
                       (uplo == 'U' || uplo == 'u') ? CUBLAS_FILL_MODE_UPPER : CUBLAS_FILL_MODE_LOWER, op_of(trans),
                       (diag == 'U' || diag == 'u') ? CUBLAS_DIAG_UNIT : CUBLAS_DIAG_NON_UNIT, nb, nb, &one, Tm, ldt,
                       W, nb));
  abs_inplace_kernel<T><<<grid_for((int64_t)nb * nb), 256, 0, s>>>(W, (int64_t)nb * nb);
  ABFT_CUDA_TRY(cudaGetLastError());
  *out = W;
  return 0;
}

template <typename T>
int update_trsm_t(char side, char uplo, char trans, char diag, int64_t nb, const void* Tv, int64_t ldt, void* chkv,
                  int64_t ldchk, int64_t nvec, void* magv, int64_t ldmag, int64_t nmag, cudaStream_t s) {
  std::unique_lock<std::mutex> lk;
  cublasHandle_t h = blas_handle(s, lk);
  const T* Tm = reinterpret_cast<const T*>(Tv);
  T* chk = reinterpret_cast<T*>(chkv);
  const bool left = side == 'L' || side == 'l';
  const T one = T(1), zero = T(0);
  if (nvec > 0) {
    ABFT_CUBLAS_TRY(trsm(h, left ? CUBLAS_SIDE_LEFT : CUBLAS_SIDE_RIGHT,
                         (uplo == 'U' || uplo == 'u') ? CUBLAS_FILL_MODE_UPPER : CUBLAS_FILL_MODE_LOWER,
                         op_of(trans), (diag == 'U' || diag == 'u') ? CUBLAS_DIAG_UNIT : CUBLAS_DIAG_NON_UNIT,
                         left ? (int)nb : (int)nvec, left ? (int)nvec : (int)nb, &one, Tm, (int)ldt, chk, (int)ldchk));
  }
  if (magv && nmag > 0) {
    T* W = nullptr;
    int rc = abs_tri_inverse<T>(h, side, uplo, trans, diag, (int)nb, Tm, (int)ldt, s, &W);
    if (rc) return rc;
    T* mag = reinterpret_cast<T*>(magv);
    void* tmpv = nullptr;
    rc = scratch_get(s, 2, (size_t)nb * nmag * sizeof(T), &tmpv);
    if (rc) return rc;
    T* tmp = reinterpret_cast<T*>(tmpv);
    if (!left) {  // tmp (nmag x nb) = mag * |W|
      ABFT_CUBLAS_TRY(gemm(h, CUBLAS_OP_N, CUBLAS_OP_N, (int)nmag, (int)nb, (int)nb, &one, mag, (int)ldmag, W,
                           (int)nb, &zero, tmp, (int)nmag));
      ABFT_CUDA_TRY(cudaMemcpy2DAsync(mag, ldmag * sizeof(T), tmp, nmag * sizeof(T), nmag * sizeof(T), nb,
                                      cudaMemcpyDeviceToDevice, s));
    } else {  // tmp (nb x nmag) = |W| * mag
      ABFT_CUBLAS_TRY(gemm(h, CUBLAS_OP_N, CUBLAS_OP_N, (int)nb, (int)nmag, (int)nb, &one, W, (int)nb, mag,
                           (int)ldmag, &zero, tmp, (int)nb));
      ABFT_CUDA_TRY(cudaMemcpy2DAsync(mag, ldmag * sizeof(T), tmp, nb * sizeof(T), nb * sizeof(T), nmag,
                                      cudaMemcpyDeviceToDevice, s));
    }
  }
  return 0;
}

template <typename T>
int update_gemm_t(int which, char transX, char transY, double alpha, const void* Xv, int64_t ldx, const void* Yv,
                  int64_t ldy, void* Cv, int64_t ldcc, int64_t M2, int64_t N, int64_t K, const void* Xmv,
                  int64_t ldxm, void* Cmv, int64_t ldcm, cudaStream_t s) {
  if (M2 == 0 || N == 0) return 0;
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
