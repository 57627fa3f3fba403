// abft_pass.cu — the fused 2D weighted-checksum pass (encode a1 / verify a2).
//
// Paper: c(A) = [v1 v2]^T A, r(A) = A [v1 v2] per NB x NB block (L108-L112,
// L446); the same kernel recomputes checksums for every check (L442);
// v1 is a plain sum and v2's weights are generated, not loaded (L446:
// 6 NB^2 flops per block); tiles are staged through shared memory with
// prefetch (L448-L454, Fig. 5).
//
// B200 design:
//  * work unit = one NB-row x S-column slab of one tile (S = NB unless the
//    grid would be too small); 256 threads; a TMA bulk-copy ring
//    (cp.async.bulk + mbarrier, one 16-B-aligned NB*s-byte copy per tile
//    column) keeps NSTAGE-1 stages of ~32 KiB in flight per CTA;
//  * phase A (column sums): one warp per column (or per column half), each
//    lane sums rows lane+32k, butterfly-shuffle reduction -> c_e, c_w, |.|;
//  * phase B (row sums): each thread owns NB/256 rows and accumulates
//    r_e, r_w, |.| across the stage's columns in registers;
//  * canonical summation order (row sums: sequential inside 64-column
//    groups, group partials added in group order; column sums: fixed lane
//    mapping + butterfly) is independent of how the tile is split into slabs,
//    so encode and verify of the same tile are bit-identical on any grid;
//  * slabbed tiles reduce row partials through a per-stream workspace; the
//    last-arriving CTA of a tile (atomic ticket) finishes it and resets the
//    ticket (no memset launches, no host sync).
#include <algorithm>

#include "abft_common.cuh"

namespace abft {

constexpr int kThreads = 256;
constexpr int kWarps = kThreads / 32;

template <typename T, int NB>
struct PassCfg {
  static constexpr int GC = NB < 64 ? NB : 64;  // group columns (slab granularity)
  static constexpr int COL_BYTES = NB * (int)sizeof(T);
  // ~32 KiB stages, 16 KiB when a column is 8 KiB (nb = 1024 fp64) so that the
  // ring still holds >= 4 stages within the 2-CTAs-per-SM budget
  static constexpr int STAGE_TARGET = COL_BYTES >= 8192 ? 16 * 1024 : 32 * 1024;
  static constexpr int CC_RAW = STAGE_TARGET / COL_BYTES;
  static constexpr int CC = CC_RAW < GC ? (CC_RAW < 1 ? 1 : CC_RAW) : GC;  // columns per stage
  static constexpr int STAGE_ELEMS = CC * NB;
  static constexpr int STAGE_BYTES = STAGE_ELEMS * (int)sizeof(T);
  static constexpr int WPC = 1;  // one warp per column in phase A (columns rotate over warps)
  // keep the whole CTA <= ~110 KiB (2 CTAs / SM): ring = budget - SYM area
  static constexpr int SIDE_BYTES = NB * 3 * (int)sizeof(T);
  static constexpr int RING_BYTES = NB >= 256 ? (96 * 1024 < 108 * 1024 - SIDE_BYTES ? 96 * 1024
                                                                                        : 108 * 1024 - SIDE_BYTES)
                                              : 48 * 1024;
  static constexpr int NSTAGE_RAW = RING_BYTES / STAGE_BYTES;
  static constexpr int NSTAGE = NSTAGE_RAW < 2 ? 2 : (NSTAGE_RAW > 8 ? 8 : NSTAGE_RAW);
  static constexpr int RH = NB / WPC;                         // rows per phase-A warp
  static constexpr int LPR = RH / 32;                         // rows per lane (phase A)
  static constexpr int RPT = NB >= kThreads ? NB / kThreads : 1;  // rows per thread (phase B)
  static constexpr int GROUPS = NB / GC;
  // phase-A vector width: one 16-B shared load per lane when the column half
  // spans >= 32 vectors
  static constexpr int VEC = RH >= 32 * (16 / (int)sizeof(T)) ? 16 / (int)sizeof(T) : 1;
  static constexpr int KV = RH / (32 * VEC);
  static constexpr size_t SMEM = (size_t)NSTAGE * STAGE_BYTES   // ring
                                 + (size_t)NB * 3 * sizeof(T)   // SYM column accumulators
                                 + 2 * NSTAGE * sizeof(uint64_t) + 64;  // full / empty barriers
  static_assert(CC >= 1 && GC % CC == 0, "stage must divide group");
  static_assert(RH % 32 == 0, "a column must be a multiple of 32 rows");
};

struct PassArgs {
  const void* A;
  int64_t lda;
  void* colchk;
  int64_t ldc;
  void* rowchk;
  int64_t ldr;
  void* colmag;
  int64_t ldcm;
  void* rowmag;
  int64_t ldrm;
  abft_tiles_t tiles;
  int which;
  int nslab;
  int use_bulk;
  int use_mag;      // verify: thresholds from maintained magnitude arrays
  int refresh;      // verify: rebase unflagged entries on the recomputed checksums (c-6)
  double tau_fac;   // scale * 2 * gamma_nb
  int32_t* status;
  int64_t ld_status;
  void* dcol;
  void* drow;
  int32_t* counts;
  void* part;       // [ntiles][GROUPS][NB][3] (slabbed tiles only)
  void* symws;      // [ntiles][3][NB] SYM column sums of slabbed diagonal tiles
  int* ticket;      // [ntiles] self-resetting
  int* tflags;      // [ntiles] self-resetting
};

template <typename T, int VEC>
__device__ __forceinline__ void load_vec(T (&x)[VEC], const T* p) {
  if constexpr (VEC == 1) {
    x[0] = p[0];
  } else if constexpr (sizeof(T) == 8) {
    const double2 v = *reinterpret_cast<const double2*>(p);
    x[0] = v.x;
    x[1] = v.y;
  } else {
    const float4 v = *reinterpret_cast<const float4*>(p);
    x[0] = v.x;
    x[1] = v.y;
    x[2] = v.z;
    x[3] = v.w;
  }
}

template <typename T>
struct Acc3 {
  T e, w, a;
};

// Verify one column or row checksum component pair: returns flag bits
// (1 = flagged, 2 = non-finite).  Oracle rule: !isfinite(d) || |d| > tau.
template <typename T>
__device__ __forceinline__ int check_pair(T me, T mw, T re, T rw, double m, double tau_fac, int nb, T* de_out,
                                          T* dw_out) {
  T de = me - re;
  T dw = mw - rw;
  *de_out = de;
  *dw_out = dw;
  double t = tau_fac * m;
  bool nf = !isfinite((double)de) || !isfinite((double)dw);
  bool fl = nf || fabs((double)de) > t || fabs((double)dw) > (double)nb * t;
  return (fl ? 1 : 0) | (nf ? 2 : 0);
}

__device__ __forceinline__ void consumer_sync() { asm volatile("bar.sync 1, 256;" ::: "memory"); }
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// 8 consumer warps + 1 producer warp.  The producer's lane 0 streams the
// unit's stages through the ring (full[] barriers count the TMA bytes); each
// consumer warp releases a stage through empty[] as soon as it is done with
// it, so warps never wait for each other inside the stage loop.
constexpr int kBlock = kThreads + 32;

template <typename T, int NB, bool VERIFY>
__global__ void __launch_bounds__(kBlock) checksum_pass_kernel(PassArgs p) {
  using C = PassCfg<T, NB>;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  T* ring = reinterpret_cast<T*>(smem_raw);
  T* symacc = ring + (size_t)C::NSTAGE * C::STAGE_ELEMS;  // [3][NB]
  uint64_t* full = reinterpret_cast<uint64_t*>(symacc + 3 * NB);
  uint64_t* empty = full + C::NSTAGE;
  __shared__ int s_colflags, s_ncols, s_nrows, s_last, s_rowflags;

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t unit = blockIdx.x;
  const int64_t tile = unit / p.nslab;
  const int slab = (int)(unit % p.nslab);
  int I, J;
  tile_of(p.tiles, tile, I, J);
  const int view = (I == J) ? p.tiles.diag_view : ABFT_GENERAL;
  const bool sym = view == ABFT_SYM_LOWER;
  const int nslab = p.nslab;
  // SYM column sums of a split tile go through the workspace (the finishing
  // CTA adds them to the row sums); an unsplit tile keeps them in smem
  T* symcol = (sym && nslab > 1) ? reinterpret_cast<T*>(p.symws) + (size_t)tile * NB * 3 : symacc;
  const int cols = NB / nslab;
  const int c0 = slab * cols;
  const int nst = cols / C::CC;
  const T* A = reinterpret_cast<const T*>(p.A);
  const T* tileA = A + (int64_t)J * NB * p.lda + (int64_t)I * NB;
  // phase-A and phase-B masks: SYM uses LOWER for columns, strict lower for rows
  const int viewA = sym ? ABFT_LOWER : view;

  if (tid == 0) {
    s_colflags = 0;
    s_ncols = 0;
    s_nrows = 0;
    s_rowflags = 0;
    if (p.use_bulk) {
      for (int s = 0; s < C::NSTAGE; ++s) {
        mbar_init(&full[s], 1);
        mbar_init(&empty[s], kWarps);
      }
      mbar_fence_init();
    }
  }
  __syncthreads();

  // ------------------------------------------------------------ producer --
  if (warp == kWarps) {
    if (p.use_bulk && lane == 0) {
      for (int g = 0; g < nst; ++g) {
        const int slot = g % C::NSTAGE;
        if (g >= C::NSTAGE) mbar_wait(&empty[slot], (uint32_t)(((g / C::NSTAGE) - 1) & 1));
        T* dst = ring + (size_t)slot * C::STAGE_ELEMS;
        fence_proxy_async();
        mbar_arrive_expect_tx(&full[slot], C::STAGE_BYTES);
        const T* src = tileA + (int64_t)(c0 + g * C::CC) * p.lda;
#pragma unroll 1
        for (int cc = 0; cc < C::CC; ++cc)
          bulk_g2s(dst + cc * NB, src + (int64_t)cc * p.lda, NB * sizeof(T), &full[slot]);
      }
    }
    return;
  }

  // ----------------------------------------------------------- consumers --
  Acc3<T> grp[C::RPT], tot[C::RPT];
#pragma unroll
  for (int q = 0; q < C::RPT; ++q) {
    grp[q] = {T(0), T(0), T(0)};
    tot[q] = {T(0), T(0), T(0)};
  }
  T* partT = reinterpret_cast<T*>(p.part);
  T* colchk = reinterpret_cast<T*>(p.colchk);
  T* colmag = reinterpret_cast<T*>(p.colmag);
  T* dcol = reinterpret_cast<T*>(p.dcol);
  int my_colflags = 0, my_ncols = 0;
  // verify: fetch the maintained column checksums (and magnitudes) of this
  // slab once, while the TMA prologue is in flight, instead of one dependent
  // strided load per column inside the stage loop.  For non-SYM tiles the
  // SYM accumulator area is free and holds them: [e | w | mag] x cols.
  if (VERIFY && !sym && (p.which & ABFT_COL)) {
    for (int idx = tid; idx < cols; idx += kThreads) {
      const int64_t gj = (int64_t)J * NB + c0 + idx;
      symacc[idx] = colchk[(int64_t)2 * I + gj * p.ldc];
      symacc[NB + idx] = colchk[(int64_t)2 * I + 1 + gj * p.ldc];
      if (p.use_mag) symacc[2 * NB + idx] = colmag[I + gj * p.ldcm];
    }
    consumer_sync();
  }
  // column finish: encode writes c (and m_c); verify compares (c-6, c-7)
  auto finish_col = [&](int jl, T pe, T pw, T pa) {
    if (sym) {
      symcol[jl] = pe;
      symcol[NB + jl] = pw;
      symcol[2 * NB + jl] = pa;
      return;
    }
    if (!(p.which & ABFT_COL)) return;
    const int64_t gj = (int64_t)J * NB + jl;
    if (!VERIFY) {
      T* cc2 = colchk + (int64_t)2 * I + gj * p.ldc;
      cc2[0] = pe;
      cc2[1] = pw;
      if (colmag) colmag[I + gj * p.ldcm] = pa;
    } else {
      const int idx = jl - c0;
      double m = p.use_mag ? (double)symacc[2 * NB + idx] : (double)pa;
      T de, dw;
      int f = check_pair<T>(symacc[idx], symacc[NB + idx], pe, pw, m, p.tau_fac, NB, &de, &dw);
      if (dcol) {
        dcol[(int64_t)2 * I + gj * p.ldc] = de;
        dcol[(int64_t)2 * I + 1 + gj * p.ldc] = dw;
      }
      my_colflags |= f;
      my_ncols += f & 1;
      if (p.refresh && !(f & 1)) {
        T* cc2 = colchk + (int64_t)2 * I + gj * p.ldc;
        cc2[0] = pe;
        cc2[1] = pw;
        if (colmag) colmag[I + gj * p.ldcm] = pa;
      }
    }
  };

  for (int s = 0; s < nst; ++s) {
    const int slot = s % C::NSTAGE;
    T* buf = ring + (size_t)slot * C::STAGE_ELEMS;
    if (p.use_bulk) {
      mbar_wait(&full[slot], (uint32_t)((s / C::NSTAGE) & 1));
    } else {
      consumer_sync();  // every warp is done with this slot's previous use
      const T* src = tileA + (int64_t)(c0 + s * C::CC) * p.lda;
      for (int idx = tid; idx < C::STAGE_ELEMS; idx += kThreads) {
        int cc = idx / NB, r = idx % NB;
        buf[idx] = src[(int64_t)cc * p.lda + r];
      }
      consumer_sync();
    }
    // ---------------- phase A: column sums (one warp per column) ----------
#pragma unroll 1
    for (int cc = 0; cc < C::CC; ++cc) {
      if (((s * C::CC + cc) & (kWarps - 1)) != warp) continue;
      const int jl = c0 + s * C::CC + cc;  // tile-local column
      const T* col = buf + cc * NB;
      T pe = T(0), pw = T(0), pa = T(0);
      if (viewA == ABFT_GENERAL) {
        // sum_i (i+1) x_i with i = (32k + lane)*VEC + v
        //   = (lane*VEC + 1) * S0 + sum_{k,v} (32*VEC*k + v) x   (compile-time weights)
        T s1 = T(0);
#pragma unroll
        for (int k = 0; k < C::KV; ++k) {
          T xv[C::VEC];
          load_vec<T, C::VEC>(xv, col + (32 * k + lane) * C::VEC);
#pragma unroll
          for (int v = 0; v < C::VEC; ++v) {
            pe = fadd(pe, xv[v]);
            s1 = ffma(T(32 * C::VEC * k + v), xv[v], s1);
            pa = fadd(pa, fabs(xv[v]));
          }
        }
        pw = ffma(T(lane * C::VEC + 1), pe, s1);
      } else {
#pragma unroll 4
        for (int k = 0; k < NB / 32; ++k) {
          const int i = lane + 32 * k;
          T x = view_mask(viewA, i, jl, col[i]);
          pe = fadd(pe, x);
          pw = ffma(T(i + 1), x, pw);
          pa = fadd(pa, fabs(x));
        }
      }
#pragma unroll
      for (int m = 16; m >= 1; m >>= 1) {
        pe = fadd(pe, shfl_xor(pe, m));
        pw = fadd(pw, shfl_xor(pw, m));
        pa = fadd(pa, shfl_xor(pa, m));
      }
      if (lane == 0) finish_col(jl, pe, pw, pa);
    }
    // ---------------- phase B: row sums ---------------------------------
#pragma unroll
    for (int q = 0; q < C::RPT; ++q) {
      const int r = tid + q * kThreads;
      if (r < NB) {
        if (view == ABFT_GENERAL) {
          // sum_cc (jl+1) x with jl = c0 + s*CC + cc  =  (c0 + s*CC + 1) * S0 + sum_cc cc*x
          T se = T(0), s1 = T(0), sa = T(0);
#pragma unroll
          for (int cc = 0; cc < C::CC; ++cc) {
            const T x = buf[cc * NB + r];
            se = fadd(se, x);
            s1 = ffma(T(cc), x, s1);
            sa = fadd(sa, fabs(x));
          }
          grp[q].e = fadd(grp[q].e, se);
          grp[q].w = fadd(grp[q].w, ffma(T(c0 + s * C::CC + 1), se, s1));
          grp[q].a = fadd(grp[q].a, sa);
        } else {
          for (int cc = 0; cc < C::CC; ++cc) {
            const int jl = c0 + s * C::CC + cc;
            T x = buf[cc * NB + r];
            x = sym ? (r > jl ? x : T(0)) : view_mask(view, r, jl, x);
            grp[q].e = fadd(grp[q].e, x);
            grp[q].w = ffma(T(jl + 1), x, grp[q].w);
            grp[q].a = fadd(grp[q].a, fabs(x));
          }
        }
      }
    }
    // stage consumed by this warp: release the slot to the producer
    if (p.use_bulk) {
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[slot]);
    }
    const bool group_end = (((s + 1) * C::CC) % C::GC) == 0;
    if (group_end) {
      const int g = (c0 + (s + 1) * C::CC) / C::GC - 1;
#pragma unroll
      for (int q = 0; q < C::RPT; ++q) {
        const int r = tid + q * kThreads;
        if (r < NB) {
          if (nslab == 1) {
            tot[q].e = fadd(tot[q].e, grp[q].e);
            tot[q].w = fadd(tot[q].w, grp[q].w);
            tot[q].a = fadd(tot[q].a, grp[q].a);
          } else {
            T* dst = partT + (((size_t)tile * C::GROUPS + g) * NB + r) * 3;
            dst[0] = grp[q].e;
            dst[1] = grp[q].w;
            dst[2] = grp[q].a;
          }
        }
        grp[q] = {T(0), T(0), T(0)};
      }
    }
  }

  // ---------------- column flags of this CTA ------------------------------
  if (VERIFY && (my_colflags | my_ncols)) {
    atomicOr(&s_colflags, my_colflags);
    atomicAdd(&s_ncols, my_ncols);
  }
  // ---------------- slab reduction: last CTA finishes the tile ------------
  if (nslab > 1) {
    __threadfence();
    consumer_sync();
    if (tid == 0) {
      if (VERIFY && s_colflags) atomicOr(&p.tflags[tile], s_colflags);
      __threadfence();
      int old = atomicAdd(&p.ticket[tile], 1);
      s_last = (old == nslab - 1);
    }
    consumer_sync();
    if (VERIFY && tid == 0 && s_ncols) atomicAdd(&p.counts[ABFT_CNT_COLS_FLAGGED], s_ncols);
    if (!s_last) return;
    __threadfence();
#pragma unroll
    for (int q = 0; q < C::RPT; ++q) {
      const int r = tid + q * kThreads;
      if (r < NB) {
        for (int g = 0; g < C::GROUPS; ++g) {
          const T* src = partT + (((size_t)tile * C::GROUPS + g) * NB + r) * 3;
          tot[q].e = fadd(tot[q].e, __ldcg(src + 0));
          tot[q].w = fadd(tot[q].w, __ldcg(src + 1));
          tot[q].a = fadd(tot[q].a, __ldcg(src + 2));
        }
      }
    }
    if (tid == 0) {
      if (VERIFY) s_colflags |= atomicExch(&p.tflags[tile], 0);
      p.ticket[tile] = 0;
    }
  } else {
    consumer_sync();
    if (VERIFY && tid == 0 && s_ncols) atomicAdd(&p.counts[ABFT_CNT_COLS_FLAGGED], s_ncols);
  }

  // ---------------- finish rows (and SYM columns) -------------------------
  T* rowchk = reinterpret_cast<T*>(p.rowchk);
  T* rowmag = reinterpret_cast<T*>(p.rowmag);
  T* drow = reinterpret_cast<T*>(p.drow);
  int my_rowflags = 0, my_nrows = 0, my_symcols = 0;
#pragma unroll
  for (int q = 0; q < C::RPT; ++q) {
    const int r = tid + q * kThreads;
    if (r >= NB) continue;
    T re = tot[q].e, rw = tot[q].w, ra = tot[q].a;
    if (sym) {  // c_sym[r] = colsum_lower[r] + rowsum_strict[r]; r_sym = c_sym^T
      if (nslab > 1) {
        re = fadd(__ldcg(symcol + r), re);
        rw = fadd(__ldcg(symcol + NB + r), rw);
        ra = fadd(__ldcg(symcol + 2 * NB + r), ra);
      } else {
        re = fadd(symacc[r], re);
        rw = fadd(symacc[NB + r], rw);
        ra = fadd(symacc[2 * NB + r], ra);
      }
    }
    const int64_t gi = (int64_t)I * NB + r;
    const int64_t gj = (int64_t)J * NB + r;
    if (!VERIFY) {
      if (p.which & ABFT_ROW) {
        rowchk[gi + (int64_t)(2 * J) * p.ldr] = re;
        rowchk[gi + (int64_t)(2 * J + 1) * p.ldr] = rw;
        if (rowmag) rowmag[gi + (int64_t)J * p.ldrm] = ra;
      }
      if (sym && (p.which & ABFT_COL)) {
        colchk[(int64_t)2 * I + gj * p.ldc] = re;
        colchk[(int64_t)2 * I + 1 + gj * p.ldc] = rw;
        if (colmag) colmag[I + gj * p.ldcm] = ra;
      }
    } else {
      if (p.which & ABFT_ROW) {
        double m = p.use_mag ? (double)rowmag[gi + (int64_t)J * p.ldrm] : (double)ra;
        T de, dw;
        int f = check_pair<T>(rowchk[gi + (int64_t)(2 * J) * p.ldr], rowchk[gi + (int64_t)(2 * J + 1) * p.ldr], re, rw,
                              m, p.tau_fac, NB, &de, &dw);
        if (drow) {
          drow[gi + (int64_t)(2 * J) * p.ldr] = de;
          drow[gi + (int64_t)(2 * J + 1) * p.ldr] = dw;
        }
        my_rowflags |= f;
        my_nrows += f & 1;
        if (p.refresh && !(f & 1)) {
          rowchk[gi + (int64_t)(2 * J) * p.ldr] = re;
          rowchk[gi + (int64_t)(2 * J + 1) * p.ldr] = rw;
          if (rowmag) rowmag[gi + (int64_t)J * p.ldrm] = ra;
        }
      }
      if (sym && (p.which & ABFT_COL)) {
        double m = p.use_mag ? (double)colmag[I + gj * p.ldcm] : (double)ra;
        T de, dw;
        int f = check_pair<T>(colchk[(int64_t)2 * I + gj * p.ldc], colchk[(int64_t)2 * I + 1 + gj * p.ldc], re, rw, m,
                              p.tau_fac, NB, &de, &dw);
        if (dcol) {
          dcol[(int64_t)2 * I + gj * p.ldc] = de;
          dcol[(int64_t)2 * I + 1 + gj * p.ldc] = dw;
        }
        my_colflags |= f;
        my_symcols += f & 1;
        if (p.refresh && !(f & 1)) {
          colchk[(int64_t)2 * I + gj * p.ldc] = re;
          colchk[(int64_t)2 * I + 1 + gj * p.ldc] = rw;
          if (colmag) colmag[I + gj * p.ldcm] = ra;
        }
      }
    }
  }
  if (!VERIFY) return;
  if (my_rowflags | my_nrows | my_symcols) {
    atomicOr(&s_rowflags, my_rowflags);
    atomicAdd(&s_nrows, my_nrows);
    if (my_symcols) {
      atomicOr(&s_colflags, my_colflags);
      atomicAdd(&s_ncols, my_symcols);
    }
  }
  consumer_sync();
  if (tid == 0) {
    int cf = s_colflags, rf = s_rowflags;
    int st = ((cf & 1) ? ABFT_ST_COL : 0) | ((rf & 1) ? ABFT_ST_ROW : 0) | (((cf | rf) & 2) ? ABFT_ST_NONFINITE : 0);
    p.status[I + (int64_t)J * p.ld_status] = st;
    if (st & (ABFT_ST_COL | ABFT_ST_ROW)) atomicAdd(&p.counts[ABFT_CNT_TILES_FLAGGED], 1);
    if (st & ABFT_ST_NONFINITE) atomicAdd(&p.counts[ABFT_CNT_NONFINITE], 1);
    if (s_nrows) atomicAdd(&p.counts[ABFT_CNT_ROWS_FLAGGED], s_nrows);
    if (sym && s_ncols) atomicAdd(&p.counts[ABFT_CNT_COLS_FLAGGED], s_ncols);
  }
}

// ------------------------------------------------------------ launcher --
template <typename T, int NB, bool VERIFY>
static int launch_nb(PassArgs& a, int64_t ntiles, cudaStream_t s) {
  using C = PassCfg<T, NB>;
  auto kern = checksum_pass_kernel<T, NB, VERIFY>;
  static bool attr_done = false;  // per instantiation
  if (!attr_done) {
    ABFT_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C::SMEM));
    attr_done = true;
  }
  // slabs: aim for >= 2 CTAs per SM when the tile count is small
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || sms <= 0) sms = 148;
  }
  int nslab = 1;
  const int max_slab = C::GROUPS;
  while (nslab < max_slab && ntiles * nslab < 2LL * sms) nslab *= 2;
  a.nslab = nslab;
  if (nslab > 1) {
    void* ws = nullptr;
    size_t bytes = (size_t)ntiles * (C::GROUPS + 1) * NB * 3 * sizeof(T);
    int rc = workspace_get(s, bytes, &ws);
    if (rc) return rc;
    int* ctr = nullptr;
    rc = counters_get(s, (size_t)2 * ntiles, &ctr);
    if (rc) return rc;
    a.part = ws;
    a.symws = reinterpret_cast<T*>(ws) + (size_t)ntiles * C::GROUPS * NB * 3;
    a.ticket = ctr;
    a.tflags = ctr + ntiles;
  }
  dim3 grid((unsigned)(ntiles * nslab));
  kern<<<grid, kBlock, C::SMEM, s>>>(a);
  ABFT_CUDA_TRY(cudaGetLastError());
  return 0;
}

template <typename T, bool VERIFY>
static int launch_t(PassArgs& a, int64_t nb, int64_t ntiles, cudaStream_t s) {
  switch (nb) {
    case 32: return launch_nb<T, 32, VERIFY>(a, ntiles, s);
    case 64: return launch_nb<T, 64, VERIFY>(a, ntiles, s);
    case 128: return launch_nb<T, 128, VERIFY>(a, ntiles, s);
    case 256: return launch_nb<T, 256, VERIFY>(a, ntiles, s);
    case 512: return launch_nb<T, 512, VERIFY>(a, ntiles, s);
    case 1024: return launch_nb<T, 1024, VERIFY>(a, ntiles, s);
    default: return ABFT_E_UNSUPPORTED;
  }
}

int validate_mat(const abft_mat_t* m, const abft_tiles_t* t, int which) {
  if (!m) return -1;
  if (!t) return -2;
  if (m->dtype != ABFT_F32 && m->dtype != ABFT_F64) return -1;
  if (m->nb < 32 || m->nb > 1024 || (m->nb & (m->nb - 1))) return -1;
  if (m->m < 0 || m->n < 0 || m->m % m->nb || m->n % m->nb) return -1;
  if (!m->A || m->lda < std::max<int64_t>(1, m->m)) return -1;
  const int64_t mt = m->m / m->nb, nt = m->n / m->nb;
  if ((which & ABFT_COL) && (!m->colchk || m->ldc < 2 * mt)) return -1;
  if ((which & ABFT_ROW) && (!m->rowchk || m->ldr < m->m)) return -1;
  if (m->colmag && m->ldcm < mt) return -1;
  if (m->rowmag && m->ldrm < m->m) return -1;
  if (t->I0 < 0 || t->J0 < 0 || t->I1 > mt || t->J1 > nt || t->I0 > t->I1 || t->J0 > t->J1) return -2;
  if (t->diag_view < ABFT_GENERAL || t->diag_view > ABFT_SYM_LOWER) return -2;
  if (which < ABFT_COL || which > ABFT_BOTH) return -3;
  return 0;
}

static int run_pass(const abft_mat_t* m, const abft_tiles_t* t, int which, const abft_tol_t* tol,
                    const abft_report_t* rep, cudaStream_t s, bool verify) {
  int rc = validate_mat(m, t, which);
  if (rc) return rc;
  const int64_t ntiles = tiles_count(*t);
  if (ntiles == 0) return 0;
  PassArgs a{};
  a.A = m->A;
  a.lda = m->lda;
  a.colchk = m->colchk;
  a.ldc = m->ldc;
  a.rowchk = m->rowchk;
  a.ldr = m->ldr;
  a.colmag = m->colmag;
  a.ldcm = m->ldcm;
  a.rowmag = m->rowmag;
  a.ldrm = m->ldrm;
  a.tiles = *t;
  a.which = which;
  const size_t es = m->dtype == ABFT_F64 ? 8 : 4;
  a.use_bulk = ((uintptr_t)m->A % 16 == 0) && ((m->lda * es) % 16 == 0);
  if (verify) {
    if (!tol) return -4;
    if (!rep || !rep->status || !rep->counts || rep->ld_status < m->m / m->nb) return -5;
    // thresholds from the maintained magnitudes when every checked direction has them (c-6)
    a.use_mag = tol->kind == ABFT_TOL_MAGNITUDE && (!(which & ABFT_COL) || m->colmag) &&
                (!(which & ABFT_ROW) || m->rowmag);
    a.tau_fac = m->dtype == ABFT_F64 ? tau_factor<double>((int)m->nb, tol->scale)
                                     : tau_factor<float>((int)m->nb, tol->scale);
    a.refresh = tol->refresh;
    a.status = rep->status;
    a.ld_status = rep->ld_status;
    a.dcol = rep->dcol;
    a.drow = rep->drow;
    a.counts = rep->counts;
  }
  if (m->dtype == ABFT_F64)
    return verify ? launch_t<double, true>(a, m->nb, ntiles, s) : launch_t<double, false>(a, m->nb, ntiles, s);
  return verify ? launch_t<float, true>(a, m->nb, ntiles, s) : launch_t<float, false>(a, m->nb, ntiles, s);
}

}  // namespace abft

extern "C" int abft_encode(const abft_mat_t* mat, const abft_tiles_t* tiles, int32_t which, abft_stream_t stream) {
  return abft::run_pass(mat, tiles, which, nullptr, nullptr, (cudaStream_t)stream, false);
}

extern "C" int abft_verify(const abft_mat_t* mat, const abft_tiles_t* tiles, int32_t which, const abft_tol_t* tol,
                           const abft_report_t* report, abft_stream_t stream) {
  return abft::run_pass(mat, tiles, which, tol, report, (cudaStream_t)stream, true);
}

extern "C" int abft_sizes(int64_t m, int64_t n, int64_t nb, int64_t* colchk_elems, int64_t* rowchk_elems,
                          int64_t* colmag_elems, int64_t* rowmag_elems) {
  if (m < 0) return -1;
  if (n < 0) return -2;
  if (nb <= 0 || m % nb || n % nb) return -3;
  if (colchk_elems) *colchk_elems = (2 * m / nb) * n;
  if (rowchk_elems) *rowchk_elems = m * (2 * n / nb);
  if (colmag_elems) *colmag_elems = (m / nb) * n;
  if (rowmag_elems) *rowmag_elems = m * (n / nb);
  return 0;
}
