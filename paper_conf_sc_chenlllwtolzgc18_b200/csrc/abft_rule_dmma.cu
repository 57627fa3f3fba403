// abft_rule_dmma.cu — the Cholesky TMU checksum rule (c-12, L189; c-6) for
// fp64 as ONE kernel on the FP64 tensor cores (DMMA, mma.sync m8n8k4).
//
// The rule of abft_update_syrk (abft_update.cu) for the trailing sub-problem
// of ntk tile rows, nk = ntk * nb rows of L21:
//   P = c(L21) L21^T   (M2 = 2 ntk rows:  c_e, c_w of every panel tile)
//   Q = m_c(L21) |L21|^T (ntk rows: the magnitude row of every panel tile)
//   c(A_IJ) -= P[2I.., cols of J],  r(A_IJ) -= P[2J.., cols of I]^T  (I >= J)
//   m_c(A_IJ) += Q[I, cols of J],   m_r(A_IJ) += Q[J, cols of I]^T
// The cuBLAS route materialises |L21| (abs_copy), runs two DGEMMs into a
// scratch P / Q and scatters both (4 extra passes over L21-sized or P-sized
// data, 5 launches).  Here A = [c(L21); m_c(L21)] (Mt = 3 ntk rows, padded)
// times L21^T is ONE tiled product: the B fragment serves the checksum rows
// as b and the magnitude rows as |b|, and the accumulators are scattered
// straight into the four arrays (one writer per element: a fire-and-forget
// reduction, no P / Q scratch).
//
// Tiling: CTA tile 64 rows of A x 32 columns, 4 warps of 32 x 16 (4 x 2
// DMMA tiles), K = nb in 16-deep stages through a 4-stage cp.async ring
// (53 KB: 4 CTAs per SM); grid (Mt / 64, nk / 32), row tiles fastest so the
// CTAs that share an L21 slice run together (a 64 x 64 tile with 32 x 32
// warps measured no faster: 225 vs 212-231 us at ntk = 59, slower at 30).
// Small grids split K over a cluster (below).  (A bulk-copy fill — one
// thread issuing a cp.async.bulk per k-row of the checksum rows and of B,
// 32 small copies per stage on an mbarrier — measured 1.6x slower than the
// per-thread 8-byte cp.async: 365 vs 230 us at ntk = 59.)  Summation order: one fixed DMMA chain per output
// element over k ascending (deterministic; not the cuBLAS order, so P and Q
// agree with the GEMM route to rounding, well inside the checks' tau).
#include <cooperative_groups.h>

#include <algorithm>

#include "abft_common.cuh"

namespace cg = cooperative_groups;

namespace abft {
namespace {

constexpr int kTM = 64;       // rows of A per CTA
constexpr int kTN = 32;       // columns per CTA
constexpr int kBK = 16;       // k per stage
#ifndef ABFT_RULE_STAGES
#define ABFT_RULE_STAGES 4
#endif
constexpr int kStages = ABFT_RULE_STAGES;
constexpr int kThr = 128;     // 4 warps: 2 (m, 32 rows) x 2 (n, 16 columns)
constexpr int kWM = 4;        // m-tiles per warp
constexpr int kWN = 2;        // n-tiles per warp
constexpr int kWNC = kWN * 8;  // columns per warp
constexpr int kLdA = kTM + 4;  // row stride = 4 (mod 16 doubles): conflict-free fragments
constexpr int kLdB = kTN + 4;
constexpr size_t kRuleSmem = (size_t)kStages * kBK * (kLdA + kLdB) * sizeof(double);

struct RuleArgs {
  // the product P = A B, A = [checksum rows (M2); pad to M2p; magnitude rows (M)]
  const double* X;  // A(y, k) = X[y xy + k xk], y < M2
  int64_t xy, xk;
  const double* Xm;  // A(M2p + q, k) = Xm[q my + k mk], q < M (nullable: no magnitude rows)
  int64_t my, mk;
  const double* Y;  // B(k, x) = Y[k yk + x yx]; the magnitude rows take |B|
  int64_t yk, yx;
  int M2, M, M2p;
  int N, K;   // columns and depth of the product
  int split;  // K split over a (1, 1, split) cluster (small grids), partials reduced in rank order
  int mode;   // 0: Cholesky scatter (c / r of the lower tiles, below); 1: plain (C, Cmo)
  // mode 0: c(A_IJ) -= P[2I.., cols of J] (I >= J), r(A_IJ) -= P[2J.., cols of I]^T,
  // m_c += Q[I, cols of J], m_r += Q[J, cols of I]^T
  double* Cc;  // c of the trailing tiles, ld oldc
  double* Rr;  // r, ld ldr (nullable)
  int64_t oldc, ldr;
  double* Cm;  // m_c, ld oldcm (nullable)
  double* Rm;  // m_r, ld ldrm (nullable)
  int64_t oldcm, ldrm;
  int nb;
  // mode 1: C[y cy + x cx] += alpha P(y, x), Cmo[q cmy + x cmx] += |alpha| Q(q, x)
  double* C;
  int64_t cy, cx;
  double* Cmo;
  int64_t cmy, cmx;
  double alpha;
};

__device__ __forceinline__ void cp_async8(void* smem, const void* gmem, bool valid) {
  // src-size 0: the 8 bytes are zero-filled (padding rows of A)
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

// One stage of the warp's kWM x kWN DMMA tiles: m-tiles a < AQ take b
// (checksum rows), a >= AQ take |b| (magnitude rows).
template <int AQ>
__device__ __forceinline__ void stage_mma(double (&acc)[kWM][kWN][2], const double* as, const double* bs, int t) {
#pragma unroll
  for (int k4 = 0; k4 < kBK; k4 += 4) {
    double bf[kWN], ba[kWN];
#pragma unroll
    for (int n = 0; n < kWN; ++n) {
      bf[n] = bs[(k4 + t) * kLdB + n * 8];
      if constexpr (AQ < kWM) ba[n] = fabs(bf[n]);
    }
#pragma unroll
    for (int a = 0; a < kWM; ++a) {
      const double af = as[(k4 + t) * kLdA + a * 8];
#pragma unroll
      for (int n = 0; n < kWN; ++n) {
        if constexpr (AQ < kWM) {
          if (a >= AQ) {
            dmma(acc[a][n], af, ba[n]);
            continue;
          }
        }
        dmma(acc[a][n], af, bf[n]);
      }
    }
  }
}

__global__ void __launch_bounds__(kThr, 4) syrk_rule_dmma_kernel(RuleArgs p) {
  extern __shared__ __align__(16) double sm[];
  double* As = sm;                                 // [kStages][kBK][kLdA]
  double* Bs = sm + (size_t)kStages * kBK * kLdA;  // [kStages][kBK][kLdB]
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int wm = warp & 1, wn = warp >> 1;
  const int g = lane >> 2, t = lane & 3;
  const int r0 = blockIdx.x * kTM;                // first row of A
  const int x0 = blockIdx.y * kTN;                // first column (row of L21)
  // this CTA's k-steps: all of them, or its rank's share of a K-split cluster
  const int kall = (p.K + kBK - 1) / kBK, z = blockIdx.z;
  const int kbeg = z * kall / p.split, ksteps = (z + 1) * kall / p.split - kbeg;
  const int M2 = p.M2;
  // fill roles, the contiguous index of each operand fastest over the
  // threads: A 64 rows x 16 k (8 loads), B 16 k x 32 x (4 loads).  With rows
  // (columns) fastest a thread keeps one row (column) for the whole loop, so
  // its source pointer is computed once (the Cholesky and LU-COL shapes).
  const bool akf = p.xk == 1, bkf = p.yk == 1;
  auto a_row = [&](int y, const double*& src, int64_t& kst) -> bool {
    const int q = y - p.M2p;
    if (y < M2) {
      src = p.X + y * p.xy;
      kst = p.xk;
      return true;
    }
    if (p.Xm && q >= 0 && q < p.M) {
      src = p.Xm + q * p.my;
      kst = p.mk;
      return true;
    }
    src = p.Y;  // any valid address (zero-filled)
    kst = 0;
    return false;
  };
  const double* srcA0 = p.Y;
  int64_t kA0 = 0;
  const bool okA0 = akf ? false : a_row(r0 + tid % kTM, srcA0, kA0);
  const int xb = tid % kTN;
  const bool okB0 = !bkf && x0 + xb < p.N;
  const double* srcB0 = p.Y + (okB0 ? (int64_t)(x0 + xb) * p.yx : 0);
  // running source pointers of the row- / column-fastest fills (fill() is
  // called for k-steps 0, 1, 2, ... in order)
  const int64_t sA = (int64_t)(kThr / kTM) * kA0, sB = (int64_t)(kThr / kTN) * p.yk;
  const double* pA = srcA0 + ((int64_t)kbeg * kBK + tid / kTM) * kA0;
  const double* pB = srcB0 + ((int64_t)kbeg * kBK + tid / kTN) * p.yk;
  auto fill = [&](int kt, int st) {
    const int64_t kb = (int64_t)(kbeg + kt) * kBK;
    double* as = As + (size_t)st * kBK * kLdA;
    if (!akf) {  // running pointer: one 64-bit add per load, compile-time smem offsets
      double* ad = as + (tid / kTM) * kLdA + tid % kTM;
      const double* ag = pA;
#pragma unroll
      for (int u = 0; u < kTM * kBK / kThr; ++u) {
        cp_async8(ad + u * (kThr / kTM) * kLdA, ag, okA0);
        ag += sA;
      }
      pA += sA * (kTM * kBK / kThr);
    } else {
      const int kk = tid % kBK;
#pragma unroll 1
      for (int u = 0; u < kTM * kBK / kThr; ++u) {
        const int rr = tid / kBK + u * (kThr / kBK);
        const double* src;
        int64_t kst;
        const bool ok = a_row(r0 + rr, src, kst);
        cp_async8(as + kk * kLdA + rr, src + (kb + kk) * kst, ok);
      }
    }
    double* bs = Bs + (size_t)st * kBK * kLdB;
    if (!bkf) {
      double* bd = bs + (tid / kTN) * kLdB + xb;
      const double* bg = pB;
#pragma unroll
      for (int u = 0; u < kTN * kBK / kThr; ++u) {
        cp_async8(bd + u * (kThr / kTN) * kLdB, bg, okB0);
        bg += sB;
      }
      pB += sB * (kTN * kBK / kThr);
    } else {
      const int kk = tid % kBK;
#pragma unroll
      for (int u = 0; u < kTN * kBK / kThr; ++u) {
        const int cc = tid / kBK + u * (kThr / kBK);
        const bool ok = x0 + cc < p.N;
        cp_async8(bs + kk * kLdB + cc, ok ? p.Y + (kb + kk) + (int64_t)(x0 + cc) * p.yx : p.Y, ok);
      }
    }
  };
#pragma unroll
  for (int s = 0; s < kStages - 1; ++s) {
    if (s < ksteps) fill(s, s);
    cp_async_commit();
  }
  double acc[kWM][kWN][2];
#pragma unroll
  for (int a = 0; a < kWM; ++a)
#pragma unroll
    for (int n = 0; n < kWN; ++n) acc[a][n][0] = acc[a][n][1] = 0.0;
  // this warp's m-tiles (rows r0 + 32 wm + 8a): checksum rows below aq,
  // magnitude rows from aq on
  const int wr0 = r0 + wm * 32;
  const int aq = min(kWM, max(0, (p.M2p - wr0) / 8));
  for (int kt = 0; kt < ksteps; ++kt) {
    cp_async_wait<kStages - 2>();
    __syncthreads();
    const int nx = kt + kStages - 1;
    if (nx < ksteps) fill(nx, nx % kStages);
    cp_async_commit();
    const double* as = As + (size_t)(kt % kStages) * kBK * kLdA + wm * 32 + g;
    const double* bs = Bs + (size_t)(kt % kStages) * kBK * kLdB + wn * kWNC + g;
    switch (aq) {  // warp-uniform
      case 0: stage_mma<0>(acc, as, bs, t); break;
      case 1: stage_mma<1>(acc, as, bs, t); break;
      case 2: stage_mma<2>(acc, as, bs, t); break;
      case 3: stage_mma<3>(acc, as, bs, t); break;
      default: stage_mma<4>(acc, as, bs, t); break;
    }
  }
  cp_async_wait<0>();
  if (p.split > 1) {
    // K-split partials: every rank parks its accumulators (thread-major) in
    // its own ring, rank 0 adds ranks 1, 2, ... in order (deterministic) and
    // scatters; the second barrier keeps the other ranks' shared memory
    // alive until rank 0 has read it
    __syncthreads();
    double* part = sm;
#pragma unroll
    for (int a = 0; a < kWM; ++a)
#pragma unroll
      for (int n = 0; n < kWN; ++n)
#pragma unroll
        for (int h = 0; h < 2; ++h) part[((a * kWN + n) * 2 + h) * kThr + tid] = acc[a][n][h];
    cg::cluster_group cl = cg::this_cluster();
    cl.sync();
    if (z == 0) {
      for (int r = 1; r < p.split; ++r) {
        const double* rp = cl.map_shared_rank(part, r);
#pragma unroll
        for (int a = 0; a < kWM; ++a)
#pragma unroll
          for (int n = 0; n < kWN; ++n)
#pragma unroll
            for (int h = 0; h < 2; ++h) acc[a][n][h] += rp[((a * kWN + n) * 2 + h) * kThr + tid];
      }
    }
    cl.sync();
    if (z != 0) return;
  }
  if (p.mode == 1) {  // plain: C += alpha P, Cmo += |alpha| Q (one writer per element)
    const double aa = fabs(p.alpha);
#pragma unroll
    for (int a = 0; a < kWM; ++a) {
      const int y = wr0 + a * 8 + g;
      const bool q = a >= aq;
      const int yq = y - p.M2p;
      if (!q && y >= M2) continue;
      if (q && (!p.Cmo || yq >= p.M)) continue;
#pragma unroll
      for (int n = 0; n < kWN; ++n)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int x = x0 + wn * kWNC + n * 8 + 2 * t + h;
          if (x >= p.N) continue;
          if (q)
            atomicAdd(p.Cmo + (int64_t)yq * p.cmy + (int64_t)x * p.cmx, aa * acc[a][n][h]);
          else
            atomicAdd(p.C + (int64_t)y * p.cy + (int64_t)x * p.cx, p.alpha * acc[a][n][h]);
        }
    }
    return;
  }
  // scatter: lane holds P/Q[y][x], [y][x+1] with y = wr0 + 8a + g,
  // x = x0 + 16 wn + 8n + 2t, tile column J = x / nb.  One writer per
  // element: a reduction adds exactly what load + add + store would.
#pragma unroll
  for (int a = 0; a < kWM; ++a) {
    const int y = wr0 + a * 8 + g;
    const bool q = a >= aq;
    const int yq = y - p.M2p;
    if (!q && y >= M2) continue;
    if (q && (!p.Cm || yq >= p.M)) continue;
    const int I = q ? yq : y / 2;
    double* Cp = q ? p.Cm + yq : p.Cc + y;  // + x * ldC
    double* Rp = q ? p.Rm : p.Rr;           // + x + row * ldR
    const int64_t ldC = q ? p.oldcm : p.oldc;
    const int64_t rowR = (int64_t)(q ? yq : y) * (q ? p.ldrm : p.ldr);
    const double sgn = q ? 1.0 : -1.0;
#pragma unroll
    for (int n = 0; n < kWN; ++n)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int xx = wn * kWNC + n * 8 + 2 * t + h;
        if (x0 + xx >= p.N) continue;
        const int J = (x0 + xx) / p.nb;
        const double v = sgn * acc[a][n][h];
        if (I >= J) atomicAdd(Cp + (int64_t)(x0 + xx) * ldC, v);
        if (Rp && J >= I) atomicAdd(Rp + (x0 + xx) + rowR, v);
      }
  }
}

static int launch_rule(RuleArgs& a, cudaStream_t s) {
  static bool attr = false;
  if (!attr) {
    ABFT_CUDA_TRY(cudaFuncSetAttribute(syrk_rule_dmma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)kRuleSmem));
    attr = true;
  }
  const int64_t Mt = a.M2p + (a.Xm ? (a.M + 7) / 8 * 8 : 0);
  const dim3 grid((unsigned)((Mt + kTM - 1) / kTM), (unsigned)((a.N + kTN - 1) / kTN));
  // small grids (the look-ahead's single tile column, late iterations) are
  // bound by the k-loop's latency, not by the DMMA rate: split K over a
  // cluster while the grid stays under ~4 CTAs per SM
  const int64_t ctas = (int64_t)grid.x * grid.y;
  const int kall = (a.K + kBK - 1) / kBK;
  int split = 1;
  while (split < 8 && ctas * split * 2 <= 4 * 148 && kall % (split * 2) == 0) split *= 2;
  a.split = split;
  if (split == 1) {
    syrk_rule_dmma_kernel<<<grid, kThr, kRuleSmem, s>>>(a);
    ABFT_CUDA_TRY(cudaGetLastError());
    return 0;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid.x, grid.y, (unsigned)split);
  cfg.blockDim = dim3(kThr, 1, 1);
  cfg.dynamicSmemBytes = kRuleSmem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = 1;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = (unsigned)split;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  ABFT_CUDA_TRY(cudaLaunchKernelEx(&cfg, syrk_rule_dmma_kernel, a));
  return 0;
}

}  // namespace

// Returns ABFT_E_UNSUPPORTED when the shape is not covered (the caller takes
// the cuBLAS route): nb must be a multiple of 32.  ntc < ntk restricts the
// product to the first ntc tile columns (x < ntc nb; the look-ahead's single
// tile column: ntc = 1 with Rr = Rm = null, c and m_c of every tile I >= J0).
int update_syrk_dmma(int64_t nb, int64_t ntk, const double* L21, int64_t ldl, const double* cL, int64_t ldc,
                     const double* mL, int64_t ldcm, double* Cc, double* Rr, int64_t ldr, double* Cm, double* Rm,
                     int64_t ldrm, cudaStream_t s, int64_t ntc) {
  if (nb % kTN || nb <= 0) return ABFT_E_UNSUPPORTED;
  if (ntc < 0) ntc = ntk;
  const int64_t nk = ntc * nb;  // columns: the first ntc tiles of L21's rows
  if (nk == 0) return 0;
  if (nk > (1LL << 30)) return ABFT_E_UNSUPPORTED;  // 32-bit column indices inside the kernel
  RuleArgs a{};
  const bool mags = mL && Cm;
  a.X = cL;  // c(L21): 2 ntk x nb, ld ldc
  a.xy = 1;
  a.xk = ldc;
  a.Xm = mags ? mL : nullptr;  // m_c(L21): ntk x nb, ld ldcm
  a.my = 1;
  a.mk = ldcm;
  a.Y = L21;  // B(k, x) = L21[x, k]
  a.yk = ldl;
  a.yx = 1;
  a.M2 = (int)(2 * ntk);
  a.M = mags ? (int)ntk : 0;
  a.M2p = (int)((2 * ntk + 7) / 8 * 8);
  a.N = (int)nk;
  a.K = (int)nb;
  a.mode = 0;
  a.Cc = Cc;
  a.Rr = Rr;
  a.oldc = ldc;
  a.ldr = ldr;
  a.Cm = mags ? Cm : nullptr;
  a.Rm = mags ? Rm : nullptr;
  a.oldcm = ldcm;
  a.ldrm = ldrm;
  a.nb = (int)nb;
  return launch_rule(a, s);
}

// abft_update_gemm (a6) in fp64 on the same kernel: the COL rule
//   C (M2 x N) += alpha op(X) op(Y),  Cm (M2/2 x N) += |alpha| op(Xm) |op(Y)|
// and the ROW rule as its transpose
//   C^T (M2 x N) += alpha op(X)^T op(Y)^T,  Cm^T += |alpha| op(Xm)^T |op(Y)^T|
// (LU's c(A22) -= c(L21) U12 and r(A22) -= L21 r(U12), QR's c(A2) -= c(V) W
// with their magnitudes, c-6 / c-13): one launch instead of the |op(Y)| copy
// and two library GEMMs.
int update_gemm_dmma(int which, char transX, char transY, double alpha, const double* X, int64_t ldx,
                     const double* Y, int64_t ldy, double* C, int64_t ldcc, int64_t M2, int64_t N, int64_t K,
                     const double* Xm, int64_t ldxm, double* Cm, int64_t ldcm, cudaStream_t s) {
  if (M2 <= 0 || N <= 0) return 0;
  if (N > (1LL << 30) || M2 > (1 << 20) || K > (1 << 20) || K % kBK) return ABFT_E_UNSUPPORTED;
  const bool tX = transX == 'T' || transX == 't', tY = transY == 'T' || transY == 't';
  const bool col = which == ABFT_COL;
  RuleArgs a{};
  const bool mags = Xm && Cm;
  // A(y, k): COL op(X)(y, k); ROW op(X)(k, y)
  const bool x_yfast = col ? !tX : tX;  // y runs along X's leading dimension
  a.X = X;
  a.xy = x_yfast ? 1 : ldx;
  a.xk = x_yfast ? ldx : 1;
  a.Xm = mags ? Xm : nullptr;
  a.my = x_yfast ? 1 : ldxm;
  a.mk = x_yfast ? ldxm : 1;
  // B(k, x): COL op(Y)(k, x); ROW op(Y)(x, k)
  const bool y_kfast = col ? !tY : tY;  // k runs along Y's leading dimension
  a.Y = Y;
  a.yk = y_kfast ? 1 : ldy;
  a.yx = y_kfast ? ldy : 1;
  a.M2 = (int)M2;
  a.M = mags ? (int)(M2 / 2) : 0;
  a.M2p = (int)((M2 + 7) / 8 * 8);
  a.N = (int)N;
  a.K = (int)K;
  a.mode = 1;
  a.C = C;
  a.cy = col ? 1 : ldcc;
  a.cx = col ? ldcc : 1;
  a.Cmo = mags ? Cm : nullptr;
  a.cmy = col ? 1 : ldcm;
  a.cmx = col ? ldcm : 1;
  a.alpha = alpha;
  a.nb = 1;
  return launch_rule(a, s);
}

}  // namespace abft
