// abft_gated.cu — kernels for the device-decided local restart (f1, L430:
// "initiate local in-memory restart of the last PD/PU").
//
// The restart of a PU is decided on the device: after the post-PU check a
// one-thread kernel compares the uncorrectable counter with the snapshot
// taken before the check and sets a gate word; the redo (restore from the
// pre-PU copy, PU data step, PU checksum rule, re-check) is queued
// unconditionally as gated kernels that return at once when the gate is 0.
// No host wait, no graph: an error-free iteration pays a handful of empty
// launches.  The redo's GEMMs are written here (plain shared-memory-tiled FMA,
// C = op(A)·op(B) with optional |.| on either operand for the magnitude rule
// of reading c-6) because a library GEMM cannot read a device gate; they run
// for real only when a restart happens, so they are sized for correctness,
// not for peak.
#include <algorithm>

#include "abft_common.cuh"

namespace abft {

template <typename T>
__device__ __forceinline__ void gemm_tile(int64_t M, int64_t N, int64_t K, const T* __restrict__ A, int64_t lda,
                                          const T* __restrict__ B, int64_t ldb, T* __restrict__ C, int64_t ldc, int ta,
                                          int tb, int absa, int absb) {
  __shared__ T As[16][64 + 1];
  __shared__ T Bs[16][64 + 1];
  const int64_t m0 = (int64_t)blockIdx.x * 64, n0 = (int64_t)blockIdx.y * 64;
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  T acc[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[i][j] = T(0);
  for (int64_t k0 = 0; k0 < K; k0 += 16) {
    for (int e = threadIdx.x; e < 16 * 64; e += 256) {
      const int r = e & 63, kk = e >> 6;
      const int64_t gm = m0 + r, gn = n0 + r, gk = k0 + kk;
      T a = T(0), b = T(0);
      if (gm < M && gk < K) a = ta ? A[gk + gm * lda] : A[gm + gk * lda];
      if (gn < N && gk < K) b = tb ? B[gn + gk * ldb] : B[gk + gn * ldb];
      As[kk][r] = absa ? (a < T(0) ? -a : a) : a;
      Bs[kk][r] = absb ? (b < T(0) ? -b : b) : b;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < 16; ++kk) {
      T a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) a[i] = As[kk][tx + 16 * i];
#pragma unroll
      for (int j = 0; j < 4; ++j) b[j] = Bs[kk][ty + 16 * j];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fma(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const int64_t gn = n0 + ty + 16 * j;
    if (gn >= N) continue;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int64_t gm = m0 + tx + 16 * i;
      if (gm < M) C[gm + gn * ldc] = acc[i][j];
    }
  }
}

// up to 3 independent products per launch (blockIdx.z): the restart redo's
// data, checksum and magnitude GEMMs are one gated launch
struct GatedBatch {
  GatedGemm g[3];
  int n;
};

template <typename T>
__global__ void __launch_bounds__(256) gemm_gated_kernel(const __grid_constant__ GatedBatch b, const int32_t* gate) {
  if (gate && *gate == 0) return;
  const GatedGemm& q = b.g[blockIdx.z];
  if ((int64_t)blockIdx.x * 64 >= q.M || (int64_t)blockIdx.y * 64 >= q.N) return;  // uniform per CTA
  gemm_tile<T>(q.M, q.N, q.K, reinterpret_cast<const T*>(q.A), q.lda, reinterpret_cast<const T*>(q.B), q.ldb,
               reinterpret_cast<T*>(q.C), q.ldc, q.ta, q.tb, q.absa, q.absb);
}

int gemm_gated_multi(int32_t dtype, const GatedGemm* g, int n, const int32_t* gate, cudaStream_t s) {
  GatedBatch b{};
  int64_t gx = 0, gy = 0;
  for (int i = 0; i < n; ++i) {
    if (g[i].M <= 0 || g[i].N <= 0) continue;
    b.g[b.n++] = g[i];
    gx = std::max<int64_t>(gx, (g[i].M + 63) / 64);
    gy = std::max<int64_t>(gy, (g[i].N + 63) / 64);
  }
  if (b.n == 0) return 0;
  const dim3 grid((unsigned)gx, (unsigned)gy, (unsigned)b.n);
  if (dtype == ABFT_F64)
    gemm_gated_kernel<double><<<grid, 256, 0, s>>>(b, gate);
  else
    gemm_gated_kernel<float><<<grid, 256, 0, s>>>(b, gate);
  ABFT_CUDA_TRY(cudaGetLastError());
  return 0;
}

int gemm_gated(int32_t dtype, bool ta, bool tb, bool absa, bool absb, int64_t M, int64_t N, int64_t K, const void* A,
               int64_t lda, const void* B, int64_t ldb, void* C, int64_t ldc, const int32_t* gate, cudaStream_t s) {
  const GatedGemm g{M, N, K, A, lda, B, ldb, C, ldc, ta, tb, absa, absb};
  return gemm_gated_multi(dtype, &g, 1, gate, s);
}

}  // namespace abft
