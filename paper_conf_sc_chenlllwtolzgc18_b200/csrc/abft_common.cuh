// Internal helpers of the sm_100a ABFT library (not part of the C ABI).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#include "abft.h"

#define ABFT_CUDA_TRY(expr)                                                              \
  do {                                                                                   \
    cudaError_t _e = (expr);                                                             \
    if (_e != cudaSuccess) {                                                             \
      fprintf(stderr, "[abft] CUDA error %s at %s:%d: %s\n", cudaGetErrorName(_e),      \
              __FILE__, __LINE__, cudaGetErrorString(_e));                               \
      return ABFT_E_CUDA;                                                                \
    }                                                                                    \
  } while (0)

namespace abft {

// ---------------------------------------------------------------- tiles --
// Enumerate the tiles of a range in column-major tile order (J outer, I
// inner), skipping I < J when lower_only.  Device and host.
__host__ __device__ inline int64_t tiles_count(const abft_tiles_t& t) {
  int64_t c = 0;
  for (int J = t.J0; J < t.J1; ++J) {
    int lo = t.lower_only ? (t.I0 > J ? t.I0 : J) : t.I0;
    if (t.I1 > lo) c += t.I1 - lo;
  }
  return c;
}

__host__ __device__ inline void tile_of(const abft_tiles_t& t, int64_t idx, int& I, int& J) {
  for (J = t.J0; J < t.J1; ++J) {
    int lo = t.lower_only ? (t.I0 > J ? t.I0 : J) : t.I0;
    int64_t cnt = t.I1 > lo ? t.I1 - lo : 0;
    if (idx < cnt) {
      I = lo + (int)idx;
      return;
    }
    idx -= cnt;
  }
  I = -1;
}

// ------------------------------------------------------------ precision --
template <typename T> struct Prec;
template <> struct Prec<double> {
  static constexpr double u = 1.1102230246251565e-16;  // 2^-53
};
template <> struct Prec<float> {
  static constexpr double u = 5.9604644775390625e-08;  // 2^-24
};

// tau_e = scale * 2 * gamma_nb * m  (DESIGN.md c-6; gamma_k = k u/(1-k u), L133)
template <typename T>
__host__ __device__ inline double tau_factor(int nb, double scale) {
  double ku = nb * Prec<T>::u;
  return scale * 2.0 * ku / (1.0 - ku);
}

// ------------------------------------------------------------- PTX bits --
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_fence_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      " .reg .pred p;\n"
      "WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// 1-D TMA bulk copy global -> shared, completion counted on `bar` (bytes).
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
// 1-D TMA bulk copy shared -> global (bulk-group completion).
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
// at most N of this thread's committed bulk groups may still be reading shared memory
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
// every committed bulk group of this thread is complete (writes performed)
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// --------------------------------------------------------------- math --
// Explicit round-to-nearest ops so the compiler cannot re-contract: the
// encode and verify instantiations then produce bit-identical sums.
__device__ __forceinline__ double fadd(double a, double b) { return __dadd_rn(a, b); }
__device__ __forceinline__ float fadd(float a, float b) { return __fadd_rn(a, b); }
__device__ __forceinline__ double ffma(double a, double b, double c) { return __fma_rn(a, b, c); }
__device__ __forceinline__ float ffma(float a, float b, float c) { return __fmaf_rn(a, b, c); }

template <typename T>
__device__ __forceinline__ T shfl_xor(T v, int m) {
  return __shfl_xor_sync(0xffffffffu, v, m);
}

// Value of view element (i, j) of a diagonal tile (c-3) given the stored
// element x = A[i][j] (for SYM the caller handles mirroring).
template <typename T>
__device__ __forceinline__ T view_mask(int view, int i, int j, T x) {
  switch (view) {
    case ABFT_LOWER: return i >= j ? x : T(0);
    case ABFT_UNIT_LOWER: return i > j ? x : (i == j ? T(1) : T(0));
    case ABFT_UPPER: return i <= j ? x : T(0);
    default: return x;
  }
}

}  // namespace abft

// Runtime (abft_runtime.cu)
namespace abft {
struct Workspace {
  void* ptr = nullptr;
  size_t bytes = 0;
};
// Per-stream scratch of at least `bytes` (grown on demand, never shrunk).
int workspace_get(cudaStream_t s, size_t bytes, void** out);
// Per-stream zero-initialised counter area (self-resetting kernels use it).
int counters_get(cudaStream_t s, size_t n_ints, int** out);
// Device-to-device 2-D copy (pitches and width in bytes) with an SM kernel:
// cudaMemcpy2DAsync D2D of column panels runs far below HBM bandwidth.
// Honours launch_gate() (below) like the verify / locate launches.
int copy2d(void* dst, size_t dpitch, const void* src, size_t spitch, size_t width, size_t height, cudaStream_t s);
// C (M x N, ld ldc) = op(A) op(B) with optional |.| on A or B, every CTA
// returning at once when *gate == 0 (abft_gated.cu; the local-restart redo).
int gemm_gated(int32_t dtype, bool ta, bool tb, bool absa, bool absb, int64_t M, int64_t N, int64_t K, const void* A,
               int64_t lda, const void* B, int64_t ldb, void* C, int64_t ldc, const int32_t* gate, cudaStream_t s);
struct GatedGemm {
  int64_t M, N, K;
  const void* A;
  int64_t lda;
  const void* B;
  int64_t ldb;
  void* C;
  int64_t ldc;
  int ta, tb, absa, absb;
};
// fp64 abft_update_gemm on the DMMA rule kernel (abft_rule_dmma.cu);
// ABFT_E_UNSUPPORTED for shapes it does not take
int update_gemm_dmma(int which, char transX, char transY, double alpha, const double* X, int64_t ldx,
                     const double* Y, int64_t ldy, double* C, int64_t ldcc, int64_t M2, int64_t N, int64_t K,
                     const double* Xm, int64_t ldxm, double* Cm, int64_t ldcm, cudaStream_t s);
// up to 3 gated products in one launch (same dtype and gate)
int gemm_gated_multi(int32_t dtype, const GatedGemm* g, int n, const int32_t* gate, cudaStream_t s);
// up to 6 2-D copies (as copy2d) in one launch; honours launch_gate()
struct Copy2D {
  void* dst;
  size_t dpitch;
  const void* src;
  size_t spitch, width, height;
};
int copy2d_multi(const Copy2D* c, int n, cudaStream_t s);
// Cholesky TMU row-checksum rule of one trailing tile column (look-ahead):
// re/rw (rows) -= L (rows x nb) [ce cw] and rm += |L| mc, ce/cw/mc strided
// (abft_update.cu).
int panel_row_rule(int32_t dtype, int64_t rows, int64_t nb, const void* L, int64_t ldl, const void* ce, const void* cw,
                   int64_t ldc, const void* mc, int64_t ldcm, void* re, void* rw, void* rm, cudaStream_t s);
// fp64 Cholesky TMU checksum rule in one DMMA kernel (abft_rule_dmma.cu);
// ABFT_E_UNSUPPORTED when nb % 32 != 0
int update_syrk_dmma(int64_t nb, int64_t ntk, const double* L21, int64_t ldl, const double* cL, int64_t ldc,
                     const double* mL, int64_t ldcm, double* Cc, double* Rr, int64_t ldr, double* Cm, double* Rm,
                     int64_t ldrm, cudaStream_t s, int64_t ntc = -1);
// abft_check (verify + locate in one launch) that also writes the checked
// range's stored elements, as corrected, to ckpt (ld ldk; element (gi, gj)
// of the range at ckpt[(gi - I0 nb) + (gj - J0 nb) ldk]): the drivers'
// local-restart copy of an op's input (f1) folded into its pre-op check
// (abft_pass.cu; a plain copy after the check when the ring cannot carry it)
int check_ckpt(const abft_mat_t* mat, const abft_tiles_t* tiles, int32_t which, const abft_tol_t* tol,
               const abft_report_t* report, abft_fix_t* fixes, int32_t max_fixes, int32_t* n_fixes, void* ckpt,
               int64_t ldk, cudaStream_t s);
// Free the per-stream pools (workspace, counters: abft_runtime.cu) and the
// per-stream library handles and scratch (abft_update.cu) of a stream that is
// about to be destroyed.  The stream must be idle.
void release_stream_pools(cudaStream_t s);
void release_stream_handles(cudaStream_t s);

// Device-side gate of the verify / locate launches issued by this host
// thread (drivers only, not part of the C ABI): when non-null, every CTA of
// those kernels returns at once unless *gate != 0, so a conditional check
// (Fig. 4b, f1) costs two empty launches and no host synchronisation.
const int32_t*& launch_gate();
struct GateScope {
  const int32_t* prev;
  explicit GateScope(const int32_t* g) : prev(launch_gate()) { launch_gate() = g; }
  ~GateScope() { launch_gate() = prev; }
};
}  // namespace abft
