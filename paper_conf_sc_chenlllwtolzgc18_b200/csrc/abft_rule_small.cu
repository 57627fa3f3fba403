// abft_rule_small.cu — the PD / PU checksum rules with an explicit inverse
// (a5, `abft_update_trsm_inv`) as ONE launch on the FP64 tensor cores.
//
// Paper: checksums are updated by applying the operation to them (L149,
// §IV); the PU of Cholesky / LU / QR is a TRSM, so its checksum rule is a
// product with the triangular factor's inverse (c-12): c(L_ik) = c(A_ik) L_kk^-T
// (Cholesky), c(U_kj) rows = L_kk^-1 r(A_kj) (LU, left side); the magnitude
// rows of reading c-6 take |op(W)|.
//
//   side R: chk (nvec x nb) <- chk op(W),   mag (nmag x nb) <- mag |op(W)|
//   side L: chk (nb x nvec) <- op(W) chk,   mag (nb x nmag) <- |op(W)| mag
//
// The library route is a GEMM into scratch + a copy back per array plus an
// |W| copy (5-7 launches, 25-35 us of dependent latency on the side chain of
// the look-ahead drivers).  Here every checksum vector v (a row for side R,
// a column for side L) is independent: out_v = old_v M with M = op(W) (side
// R) or op(W)^T (side L).  A thread-block cluster owns 32 vectors and spans
// all nb output columns (JB = 32 per CTA, nb / 32 <= 16 CTAs): each CTA runs
// a DMMA (mma.sync m8n8k4 f64) main loop over q with a 4-stage cp.async ring,
// then the cluster barrier orders every CTA's reads of the old vectors
// before any CTA stores its columns — so the update runs IN PLACE, no
// scratch, no copy back.  Summation order: one DMMA chain per output over q
// ascending (deterministic).  fp64 only (fp32 and nb = 1024 keep the library
// route).
#include <cooperative_groups.h>

#include "abft_common.cuh"

namespace cg = cooperative_groups;

namespace abft {
namespace {

constexpr int kVB = 32;   // vectors per cluster (rows of the product)
constexpr int kJB = 32;   // output columns per CTA
#ifndef ABFT_SMALL_RULE_BK
#define ABFT_SMALL_RULE_BK 16
#endif
constexpr int kBK = ABFT_SMALL_RULE_BK;  // q per stage (32: 73 KB of shared memory next to the DSYRK, ft_potrf 0.1-0.4 ms slower)
constexpr int kStages = 4;
constexpr int kThr = 128;  // 4 warps: 2 (vectors, 16 each) x 2 (columns, 16 each)
constexpr int kLd = kVB + 4;  // stage row stride (doubles): 4 (mod 16) keeps fragments conflict-free
static_assert(kVB == kJB, "one stage layout for both operands");

struct SmallRuleArgs {
  const double* W;
  int64_t ldw;
  int tW;     // M[q][j] = tW ? W[j + q ldw] : W[q + j ldw]
  int sideR;  // vector v element q at base[v + q ld] (R) or base[q + v ld] (L)
  int nb;
  double* chk;
  int64_t ldchk;
  int nvec;
  double* mag;
  int64_t ldmag;
  int nmag;
  int nblk_chk;  // vector blocks of chk (the rest are magnitude blocks)
};

__device__ __forceinline__ void cp_async8(void* smem, const void* gmem, bool valid) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(smem_u32(smem)), "l"(gmem),
               "r"(valid ? 8 : 0)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void dmma(double (&d)[2], double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
               : "+d"(d[0]), "+d"(d[1])
               : "d"(a), "d"(b));
}

constexpr size_t kSmem = 2 * (size_t)kStages * kBK * kLd * sizeof(double);

__global__ void __launch_bounds__(kThr) trsm_inv_rule_kernel(const __grid_constant__ SmallRuleArgs a) {
  extern __shared__ __align__(16) double rs_sm[];
  double(*Vs)[kBK][kLd] = reinterpret_cast<double(*)[kBK][kLd]>(rs_sm);                         // [q][v]
  double(*Ms)[kBK][kLd] = reinterpret_cast<double(*)[kBK][kLd]>(rs_sm + kStages * kBK * kLd);  // [q][j]
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int wv = warp & 1, wj = warp >> 1;
  const int g = lane >> 2, t = lane & 3;
  const int nb = a.nb;
  const int vb = blockIdx.y;
  const bool mag = vb >= a.nblk_chk;
  double* base = mag ? a.mag : a.chk;
  const int64_t ld = mag ? a.ldmag : a.ldchk;
  const int nv = mag ? a.nmag : a.nvec;
  const int v0 = (mag ? vb - a.nblk_chk : vb) * kVB;
  const int j0 = blockIdx.x * kJB;
  const int64_t sv = a.sideR ? 1 : ld, sq = a.sideR ? ld : 1;  // vector / q strides of base
  const int64_t mj = a.tW ? 1 : a.ldw, mq = a.tW ? a.ldw : 1;  // column / q strides of M in W
  // fill roles: 128 threads x 8 elements per operand per stage (32 q x 32);
  // the contiguous index of each operand runs fastest over the threads
  auto fill = [&](int kt, int st) {
    const int q0 = kt * kBK;
#pragma unroll
    for (int u = 0; u < kBK * kVB / kThr; ++u) {
      const int idx = tid + u * kThr;
      int x, qq;  // V: x = vector
      if (a.sideR) {
        x = idx % kVB;
        qq = idx / kVB;
      } else {
        qq = idx % kBK;
        x = idx / kBK;
      }
      const bool ok = v0 + x < nv;
      cp_async8(&Vs[st][qq][x], base + (ok ? (v0 + x) * sv + (int64_t)(q0 + qq) * sq : 0), ok);
      int y, qm;  // M: y = column
      if (a.tW) {
        y = idx % kJB;
        qm = idx / kJB;
      } else {
        qm = idx % kBK;
        y = idx / kBK;
      }
      cp_async8(&Ms[st][qm][y], a.W + (int64_t)(j0 + y) * mj + (int64_t)(q0 + qm) * mq, true);
    }
  };
  const int ksteps = nb / kBK;
#pragma unroll
  for (int s = 0; s < kStages - 1; ++s) {
    if (s < ksteps) fill(s, s);
    cp_async_commit();
  }
  double acc[2][2][2] = {};  // [v-tile][j-tile][2]
  for (int kt = 0; kt < ksteps; ++kt) {
    cp_async_wait<kStages - 2>();
    __syncthreads();
    const int nx = kt + kStages - 1;
    if (nx < ksteps) fill(nx, nx % kStages);
    cp_async_commit();
    const int st = kt % kStages;
#pragma unroll
    for (int k4 = 0; k4 < kBK; k4 += 4) {
      double bf[2];
#pragma unroll
      for (int n = 0; n < 2; ++n) {
        const double w = Ms[st][k4 + t][wj * 16 + n * 8 + g];
        bf[n] = mag ? fabs(w) : w;
      }
#pragma unroll
      for (int m = 0; m < 2; ++m) {
        const double af = Vs[st][k4 + t][wv * 16 + m * 8 + g];
#pragma unroll
        for (int n = 0; n < 2; ++n) dmma(acc[m][n], af, bf[n]);
      }
    }
  }
  cp_async_wait<0>();
  // every CTA of the cluster has read all of the cluster's old vectors
  cg::this_cluster().sync();
  // lane holds out[v][j], out[v][j+1]: v = v0 + 16 wv + 8 m + g, j = j0 + 16 wj + 8 n + 2 t
#pragma unroll
  for (int m = 0; m < 2; ++m) {
    const int v = v0 + wv * 16 + m * 8 + g;
    if (v >= nv) continue;
#pragma unroll
    for (int n = 0; n < 2; ++n)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int j = j0 + wj * 16 + n * 8 + 2 * t + h;
        base[(int64_t)v * sv + (int64_t)j * sq] = acc[m][n][h];
      }
  }
}

}  // namespace

// Returns ABFT_E_UNSUPPORTED outside fp64 with nb in {32, ..., 512} powers of
// two (the caller then takes the library route).
int trsm_inv_rule(char side, char trans, int64_t nb, const double* W, int64_t ldw, double* chk, int64_t ldchk,
                  int64_t nvec, double* mag, int64_t ldmag, int64_t nmag, cudaStream_t s) {
  if (nb < 32 || nb > 16 * kJB || (nb & (nb - 1))) return ABFT_E_UNSUPPORTED;
  const bool right = side == 'R' || side == 'r';
  const bool tr = trans == 'T' || trans == 't';
  if (!mag) nmag = 0;
  if (!chk) nvec = 0;
  if (nvec <= 0 && nmag <= 0) return 0;
  SmallRuleArgs a{};
  a.W = W;
  a.ldw = ldw;
  a.tW = right ? tr : !tr;
  a.sideR = right;
  a.nb = (int)nb;
  a.chk = chk;
  a.ldchk = ldchk;
  a.nvec = (int)(nvec > 0 ? nvec : 0);
  a.mag = mag;
  a.ldmag = ldmag;
  a.nmag = (int)(nmag > 0 ? nmag : 0);
  a.nblk_chk = (a.nvec + kVB - 1) / kVB;
  const int nblk = a.nblk_chk + (a.nmag + kVB - 1) / kVB;
  const unsigned cs = (unsigned)(nb / kJB);
  static bool attr = false;
  if (!attr) {
    ABFT_CUDA_TRY(cudaFuncSetAttribute(trsm_inv_rule_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
    ABFT_CUDA_TRY(cudaFuncSetAttribute(trsm_inv_rule_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmem));
    attr = true;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(cs, (unsigned)nblk, 1);
  cfg.blockDim = dim3(kThr, 1, 1);
  cfg.dynamicSmemBytes = kSmem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = cs;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  ABFT_CUDA_TRY(cudaLaunchKernelEx(&cfg, trsm_inv_rule_kernel, a));
  return 0;
}

}  // namespace abft
