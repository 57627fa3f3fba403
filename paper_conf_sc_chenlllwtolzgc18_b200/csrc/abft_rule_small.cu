// abft_rule_small.cu — the PD / PU checksum rules with an explicit inverse
// (a5, `abft_update_trsm_inv`) as ONE launch.
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
// The library route was a GEMM into scratch + a copy back per array plus an
// |W| copy (5-7 launches, 25-35 us of dependent latency on the side chain of
// the look-ahead drivers).  Here every checksum vector v (a row for side R,
// a column for side L) is independent: out_v = old_v M with M = op(W) (side
// R) or op(W)^T (side L), so the update runs IN PLACE as one clustered
// launch.  A cluster owns VB vectors and spans the nb output columns (JB per
// CTA); every CTA stages the cluster's old vectors in shared memory, the
// cluster barrier orders all reads before any write, then each CTA computes
// and stores its JB columns.  W is streamed through shared memory in
// QB-row chunks with a register prefetch of the next chunk.  Summation
// order: q ascending, one FMA chain per output (deterministic).  Each CTA
// reads its nb x JB slice of W from L2 (512 KB at nb=512 fp64); thread groups
// whose vectors are all past the end (the 2 + 1 vectors of the PD rule) skip
// the FMAs.
#include <cooperative_groups.h>

#include "abft_common.cuh"

namespace cg = cooperative_groups;

namespace abft {
namespace {

constexpr int kVB = 16;   // vectors per cluster
constexpr int kThr = 256;

template <typename T>
struct SmallRuleArgs {
  const T* W;
  int64_t ldw;
  int tW;     // M[q][j] = tW ? W[j + q ldw] : W[q + j ldw]
  int sideR;  // vector v element q at base[v + q ld] (R) or base[q + v ld] (L)
  int nb;
  T* chk;
  int64_t ldchk;
  int nvec;
  T* mag;
  int64_t ldmag;
  int nmag;
  int nblk_chk;  // vector blocks of chk (the rest are magnitude blocks)
};

// rows of M per staged chunk: 16 prefetched values per thread
template <int JB>
constexpr int qb_of() {
  return 4096 / JB;
}

template <typename T, int JB>
__global__ void __launch_bounds__(kThr) trsm_inv_rule_kernel(SmallRuleArgs<T> a) {
  constexpr int kQB = qb_of<JB>();
  extern __shared__ __align__(16) unsigned char rs_smem[];
  constexpr int WLD = JB + 2;  // row stride of the W chunk (even: 16-B aligned pairs)
  T* Vs = reinterpret_cast<T*>(rs_smem);  // [kVB][nb]
  T* Ws = Vs + (size_t)kVB * a.nb;        // [kQB][WLD]
  const int tid = threadIdx.x;
  const int nb = a.nb;
  const int vb = blockIdx.y;
  const bool mag = vb >= a.nblk_chk;
  T* base = mag ? a.mag : a.chk;
  const int64_t ld = mag ? a.ldmag : a.ldchk;
  const int nv = mag ? a.nmag : a.nvec;
  const int v0 = (mag ? vb - a.nblk_chk : vb) * kVB;
  const int j0 = blockIdx.x * JB;

  // 1. the cluster's old vectors
  if (a.sideR) {
    for (int idx = tid; idx < kVB * nb; idx += kThr) {
      const int v = idx % kVB, q = idx / kVB;
      Vs[v * nb + q] = v0 + v < nv ? base[(v0 + v) + (int64_t)q * ld] : T(0);
    }
  } else {
    for (int idx = tid; idx < kVB * nb; idx += kThr) {
      const int q = idx % nb, v = idx / nb;
      Vs[v * nb + q] = v0 + v < nv ? base[q + (int64_t)(v0 + v) * ld] : T(0);
    }
  }
  // every CTA of the cluster has read the old values before anyone writes
  cg::this_cluster().sync();

  // 2. out[v][j] = sum_q Vs[v][q] M[q][j]; thread: column pair jp, vector group g
  constexpr int NP = JB / 2;         // column pairs
  constexpr int NG = kThr / NP;      // vector groups
  constexpr int VPG = kVB / NG;      // vectors per thread
  static_assert(VPG >= 1 && kVB % NG == 0, "tile shape");
  const int jp = tid % NP, g = tid / NP;
  const bool active = v0 + g * VPG < nv;  // uniform per group of NP threads
  T acc[VPG][2];
#pragma unroll
  for (int i = 0; i < VPG; ++i) acc[i][0] = acc[i][1] = T(0);
  constexpr int PER = kQB * JB / kThr;  // chunk elements loaded per thread
  T pre[PER];
  auto load_chunk = [&](int q0) {
#pragma unroll
    for (int u = 0; u < PER; ++u) {
      const int idx = tid + u * kThr;
      int qq, jj;
      if (a.tW) {  // contiguous along j
        jj = idx % JB;
        qq = idx / JB;
      } else {     // contiguous along q
        qq = idx % kQB;
        jj = idx / kQB;
      }
      const int q = q0 + qq, j = j0 + jj;
      pre[u] = q < nb ? (a.tW ? a.W[j + (int64_t)q * a.ldw] : a.W[q + (int64_t)j * a.ldw]) : T(0);
    }
  };
  auto store_chunk = [&]() {
#pragma unroll
    for (int u = 0; u < PER; ++u) {
      const int idx = tid + u * kThr;
      int qq, jj;
      if (a.tW) {
        jj = idx % JB;
        qq = idx / JB;
      } else {
        qq = idx % kQB;
        jj = idx / kQB;
      }
      const T w = pre[u];
      Ws[qq * WLD + jj] = mag ? T(fabs(w)) : w;
    }
  };
  load_chunk(0);
  for (int q0 = 0; q0 < nb; q0 += kQB) {
    __syncthreads();  // the previous chunk's readers are done
    store_chunk();
    __syncthreads();
    if (q0 + kQB < nb) load_chunk(q0 + kQB);  // in flight during the FMAs below
    const int qn = !active ? 0 : (nb - q0 < kQB ? nb - q0 : kQB);
    for (int qq = 0; qq < qn; ++qq) {
      const T w0 = Ws[qq * WLD + 2 * jp], w1 = Ws[qq * WLD + 2 * jp + 1];
#pragma unroll
      for (int i = 0; i < VPG; ++i) {
        const T x = Vs[(g * VPG + i) * nb + q0 + qq];
        acc[i][0] = fma(x, w0, acc[i][0]);
        acc[i][1] = fma(x, w1, acc[i][1]);
      }
    }
  }
  // 3. store this CTA's columns of the cluster's vectors
#pragma unroll
  for (int i = 0; i < VPG; ++i) {
    const int v = v0 + g * VPG + i;
    if (v >= nv) continue;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int j = j0 + 2 * jp + h;
      if (a.sideR)
        base[v + (int64_t)j * ld] = acc[i][h];
      else
        base[j + (int64_t)v * ld] = acc[i][h];
    }
  }
}

template <typename T, int JB>
int launch_small_rule(const SmallRuleArgs<T>& a, int nblk, cudaStream_t s) {
  auto kern = trsm_inv_rule_kernel<T, JB>;
  const size_t smem = ((size_t)kVB * a.nb + (size_t)qb_of<JB>() * (JB + 2)) * sizeof(T);
  static size_t attr = 0;
  if (attr < smem) {
    ABFT_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    attr = smem;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(a.nb / JB), (unsigned)nblk, 1);
  cfg.blockDim = dim3(kThr, 1, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = (unsigned)(a.nb / JB);
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  ABFT_CUDA_TRY(cudaLaunchKernelEx(&cfg, kern, a));
  return 0;
}

}  // namespace

// Returns ABFT_E_UNSUPPORTED for shapes outside nb in {32, ..., 1024} powers
// of two (the caller then takes the library route).
template <typename T>
int trsm_inv_rule(char side, char trans, int64_t nb, const T* W, int64_t ldw, T* chk, int64_t ldchk, int64_t nvec,
                  T* mag, int64_t ldmag, int64_t nmag, cudaStream_t s) {
  if (nb < 32 || nb > 1024 || (nb & (nb - 1))) return ABFT_E_UNSUPPORTED;
  const bool right = side == 'R' || side == 'r';
  const bool tr = trans == 'T' || trans == 't';
  if (!mag) nmag = 0;
  if (!chk) nvec = 0;
  if (nvec <= 0 && nmag <= 0) return 0;
  SmallRuleArgs<T> a{};
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
  if (nb >= 128) return launch_small_rule<T, 128>(a, nblk, s);
  if (nb == 64) return launch_small_rule<T, 64>(a, nblk, s);
  return launch_small_rule<T, 32>(a, nblk, s);
}

template int trsm_inv_rule<double>(char, char, int64_t, const double*, int64_t, double*, int64_t, int64_t, double*,
                                   int64_t, int64_t, cudaStream_t);
template int trsm_inv_rule<float>(char, char, int64_t, const float*, int64_t, float*, int64_t, int64_t, float*,
                                  int64_t, int64_t, cudaStream_t);

}  // namespace abft
