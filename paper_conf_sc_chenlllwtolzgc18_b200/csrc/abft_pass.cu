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
#include <cstdlib>

#include "abft_locate.cuh"

namespace abft {

constexpr int kThreads = 256;
constexpr int kWarps = kThreads / 32;

// NB = checksum tile; K = vertically adjacent tiles streamed by one CTA
// (K > 1 for small tiles: one K*NB-row bulk copy per column and a K-times
// longer CTA lifetime; GENERAL views only).
// LEAN (verify launches of at most one wave: the drivers' per-iteration
// checks): a 64 KiB ring instead of 96 KiB.  Such a check runs next to the
// factorization's DSYRK on the look-ahead side stream; every KiB it holds is
// shared memory a DSYRK CTA cannot have (a 110 KiB check CTA displaced two
// of them, a 76 KiB one displaces one): ft_potrf n=30720 6.70% -> 5.74%,
// while the full-matrix pass keeps the deeper ring (7.06 vs 6.85 TB/s).
template <typename T, int NB, int K, bool VERIFY = false, bool LEAN = false>
struct PassCfg {
  static constexpr int RK = K * NB;              // rows per CTA
  // group columns (slab granularity).  (32-column groups for NB >= 256 were
  // measured: single diagonal-tile checks 11.6 -> 7.8 us (LOWER col), 18.6
  // -> 16.7 (SYM both), but 59-tile both-direction panels 31.9 -> 39.6 us
  // from the doubled row-partial traffic; ft_potrf unchanged.)
  static constexpr int GC = NB < 64 ? NB : 64;
  static constexpr int COL_BYTES = RK * (int)sizeof(T);
  // 32 KiB stages for every column size (fp64 nb=1024, 8-KiB columns, had
  // 16 KiB stages of 2 columns: the row-sum chunk CQ fell to 2 columns, the
  // per-chunk work per element rose ~1.5x, and the pass ran at 5.1-6.1 TB/s;
  // with 4-column stages 6.3-7.0 TB/s, pass_views r01)
  static constexpr int STAGE_TARGET = 32 * 1024;
  static constexpr int CC_RAW = STAGE_TARGET / COL_BYTES;
  static constexpr int CC = CC_RAW < GC ? (CC_RAW < 1 ? 1 : CC_RAW) : GC;  // columns per stage
  static constexpr int STAGE_ELEMS = CC * RK;
  static constexpr int STAGE_BYTES = STAGE_ELEMS * (int)sizeof(T);
  // keep the whole CTA <= ~110 KiB (2 CTAs / SM): ring = budget - side area.
  // Side area: SYM column sums / maintained column checksums, and for verify
  // the recomputed column sums (compared after the stage loop, see below)
  // verify parks the recomputed column sums of a non-SYM tile in the SYM
  // area (a SYM tile keeps its column sums there and parks nothing), so the
  // side area is RK*3 for both; the maintained checksums are read from
  // global memory at compare time (a 12 KiB smaller side area gives fp64
  // nb=512 verify a third 32 KiB ring stage)
  static constexpr int REC_ELEMS = 0;
  static constexpr int SIDE_BYTES = (RK * 3 + REC_ELEMS) * (int)sizeof(T);
  static constexpr int RING_CAP = LEAN ? 64 * 1024 : 96 * 1024;
  static constexpr int RING_BYTES = RK >= 256 ? (RING_CAP < 108 * 1024 - SIDE_BYTES ? RING_CAP
                                                                                        : 108 * 1024 - SIDE_BYTES)
                                              : 48 * 1024;
  static constexpr int NSTAGE_RAW = RING_BYTES / STAGE_BYTES;
  static constexpr int NSTAGE = NSTAGE_RAW < 2 ? 2 : (NSTAGE_RAW > 8 ? 8 : NSTAGE_RAW);
  static constexpr int RPT = RK >= kThreads ? RK / kThreads : 1;  // rows per thread (phase B)
  static constexpr int GROUPS = NB / GC;
  // phase-A vector width: one 16-B shared load per lane when a tile column
  // spans >= 32 vectors (and a vector never straddles two tiles)
  static constexpr int VEC = NB >= 32 * (16 / (int)sizeof(T)) ? 16 / (int)sizeof(T) : 1;
  static constexpr int KV = RK / (32 * VEC);   // vector loads per lane per column
  static constexpr int KPT = NB / (32 * VEC);  // ... of them per tile
  // Canonical row-sum chunk: the stage width of the deepest stacking used for
  // this (T, NB).  Row sums are accumulated per CQ-column chunk whatever K and
  // CC are, so every launch shape gives bit-identical checksums.
  static constexpr int KBIG_RAW = 4096 / (NB * (int)sizeof(T));
  static constexpr int KBIG = KBIG_RAW < 1 ? 1 : (KBIG_RAW > 8 ? 8 : KBIG_RAW);
  static constexpr int COLB_BIG = KBIG * NB * (int)sizeof(T);
  static constexpr int CC_BIG_RAW = (32 * 1024) / COLB_BIG;
  static constexpr int CQ = CC_BIG_RAW < GC ? (CC_BIG_RAW < 1 ? 1 : CC_BIG_RAW) : GC;
  static_assert(CC % CQ == 0, "row-sum chunk must divide the stage");
  static constexpr size_t SMEM = (size_t)NSTAGE * STAGE_BYTES   // ring
                                 + (size_t)(RK * 3 + REC_ELEMS) * sizeof(T)  // side area
                                 + 2 * NSTAGE * sizeof(uint64_t) + 64;  // full / empty barriers
  static_assert(CC >= 1 && GC % CC == 0, "stage must divide group");
  static_assert(NB % 32 == 0, "a tile column must be a multiple of 32 rows");
  static_assert(K == 1 || NB % (32 * VEC) == 0, "stacked tiles need whole vectors per tile");
  static_assert(K <= 8, "at most 8 stacked tiles");
  // the fused check's locate_tile fits in the ring + side area
  static constexpr bool FUSE_OK =
      VERIFY && locate_smem_bytes(NB, (int)sizeof(T)) <= (size_t)NSTAGE * STAGE_BYTES + (RK * 3 + REC_ELEMS) * sizeof(T);
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
  int K;            // tiles per unit (vertical stack), see PassCfg
  int mode;         // unit decode: PASS_RECT / PASS_SEG / PASS_DIAG (see below)
  void* part;       // [nsuper][GROUPS][K*NB][3] (slabbed units only)
  void* symws;      // [ntiles][3][NB] SYM column sums of slabbed diagonal tiles
  int* ticket;      // [nsuper] self-resetting
  int* tflags;      // [ntiles] self-resetting
  const int32_t* gate;  // nullable: run only if *gate != 0 (driver-side conditional checks)
  // fused check (abft_check): the finishing CTA of a flagged tile runs
  // locate_tile on it before exiting (no separate locate launch)
  int fuse;
  LocArgs loc;
  // local-restart checkpoint (f1, drivers only): the producer also writes
  // every landed stage's columns to ckpt (element (gi, gj) of the range at
  // ckpt[(gi - I0 nb) + (gj - J0 nb) ldk]) with bulk shared->global copies,
  // so the pre-op check and the copy of its input are one pass over HBM
  void* ckpt;
  int64_t ldk;
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

// Masked diagonal views (c-3), one template per view so that the inner loops
// carry no view switch; weights are compile-time or stepped in floating point
// (an int->fp64 conversion per element, I2F.F64, made a masked diagonal tile
// ~6x slower than a GENERAL one: pass_views r01).
template <int VIEW, typename T>
__device__ __forceinline__ T masked(int i, int j, T x) {  // X[i, j] under VIEW
  if (VIEW == ABFT_LOWER) return i >= j ? x : T(0);
  if (VIEW == ABFT_UNIT_LOWER) return i > j ? x : (i == j ? T(1) : T(0));
  if (VIEW == ABFT_UPPER) return i <= j ? x : T(0);
  if (VIEW == ABFT_SYM_LOWER) return i > j ? x : T(0);  // strict lower (the row-sum half of SYM)
  return x;
}
template <int VIEW, int CC, int RK, typename T>
__device__ __forceinline__ void masked_rowsum(const T* buf, int r, int jl0, Acc3<T>& g) {
  T wj = T(jl0 + 1);
#pragma unroll 8
  for (int cc = 0; cc < CC; ++cc) {
    const T x = masked<VIEW>(r, jl0 + cc, buf[cc * RK + r]);
    g.e = fadd(g.e, x);
    g.w = ffma(wj, x, g.w);
    g.a = fadd(g.a, fabs(x));
    wj = fadd(wj, T(1));
  }
}

// Masked column sums with the GENERAL path's vector loads and compile-time
// weights: a warp-uniform test per vector iteration skips row blocks the view
// zeroes entirely and masks element-wise only in the block the diagonal
// crosses (a masked diagonal tile then streams about half of its column work).
template <int VIEW, int NB, int VEC, typename T>
__device__ __forceinline__ void masked_colsum_vec(const T* col, int jl, int lane, T& e, T& w, T& a) {
  constexpr int KV = NB / (32 * VEC);
  T pe = T(0), s1 = T(0), pa = T(0);
#pragma unroll
  for (int k = 0; k < KV; ++k) {
    const int blo = 32 * VEC * k, bhi = blo + 32 * VEC - 1;  // the warp's rows this iteration
    bool out, in;
    if (VIEW == ABFT_UPPER) {
      out = blo > jl;
      in = bhi <= jl;
    } else if (VIEW == ABFT_LOWER) {
      out = bhi < jl;
      in = blo >= jl;
    } else {  // UNIT_LOWER: the diagonal element reads as 1
      out = bhi < jl;
      in = blo > jl;
    }
    if (out) continue;
    T xv[VEC];
    load_vec<T, VEC>(xv, col + (32 * k + lane) * VEC);
    if (!in) {
#pragma unroll
      for (int v = 0; v < VEC; ++v) xv[v] = masked<VIEW>((32 * k + lane) * VEC + v, jl, xv[v]);
    }
#pragma unroll
    for (int v = 0; v < VEC; ++v) {
      pe = fadd(pe, xv[v]);
      s1 = ffma(T(32 * VEC * k + v), xv[v], s1);
      pa = fadd(pa, fabs(xv[v]));
    }
  }
  e = pe;
  w = ffma(T(lane * VEC + 1), pe, s1);
  a = pa;
}

// Masked row sums of one stage for row r: a stage entirely inside the view
// takes the GENERAL chunk formula, one entirely outside is skipped, only the
// stage the diagonal crosses is masked element-wise.
template <int VIEW, int CC, int CQ, int RK, typename T>
__device__ __forceinline__ void masked_rowsum_fast(const T* buf, int r, int jl0, Acc3<T>& g) {
  const int jl1 = jl0 + CC - 1;
  bool in, out;
  if (VIEW == ABFT_UPPER) {  // keep jl >= r
    in = jl0 >= r;
    out = jl1 < r;
  } else if (VIEW == ABFT_LOWER) {  // keep jl <= r
    in = jl1 <= r;
    out = jl0 > r;
  } else if (VIEW == ABFT_SYM_LOWER) {  // keep jl < r
    in = jl1 < r;
    out = jl0 >= r;
  } else {  // UNIT_LOWER: keep jl < r, jl == r reads 1
    in = jl1 < r;
    out = jl0 > r;
  }
  if (out) return;
  if (!in) {
    masked_rowsum<VIEW, CC, RK>(buf, r, jl0, g);
    return;
  }
#pragma unroll
  for (int ch = 0; ch < CC / CQ; ++ch) {
    T se = T(0), s1 = T(0), sa = T(0);
#pragma unroll
    for (int cq = 0; cq < CQ; ++cq) {
      const T x = buf[(ch * CQ + cq) * RK + r];
      se = fadd(se, x);
      s1 = ffma(T(cq), x, s1);
      sa = fadd(sa, fabs(x));
    }
    g.e = fadd(g.e, se);
    g.w = fadd(g.w, ffma(T(jl0 + ch * CQ + 1), se, s1));
    g.a = fadd(g.a, sa);
  }
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

// Unit decode.
//  PASS_RECT: K == 1 follows the tile enumeration (lower_only aware, the
//    diagonal tiles in diag_view); K > 1 stacks K consecutive tile rows of one
//    tile column of a rectangular range whose height K divides.
//  PASS_SEG: the tiles of each tile column that are checked in the GENERAL
//    view form <= 2 contiguous segments (lower_only clips the top; a diagonal
//    tile with a masked view is left out and splits the column); each segment
//    is cut into stacks of K tiles, the last one ragged (kv < K tiles).
//  PASS_DIAG: only the diagonal tiles of the range, one per unit (K == 1),
//    in diag_view — the companion launch of a PASS_SEG launch.
enum { PASS_RECT = 0, PASS_SEG = 1, PASS_DIAG = 2 };

__host__ __device__ __forceinline__ int64_t seg_units(int len, int K) { return len > 0 ? (len + K - 1) / K : 0; }

// returns the number of units when u is past the end (host: count with u = -1)
__host__ __device__ inline int64_t seg_of(const abft_tiles_t& t, int K, int64_t u, int& Ib, int& J, int& kv) {
  const bool split = t.diag_view != ABFT_GENERAL;
  int64_t seen = 0;
  for (int Jc = t.J0; Jc < t.J1; ++Jc) {
    const int lo = t.lower_only ? (t.I0 > Jc ? t.I0 : Jc) : t.I0;
    int a1 = t.I1, b0 = 0, b1 = 0;
    if (split && Jc >= lo && Jc < t.I1) {
      a1 = Jc;
      b0 = Jc + 1;
      b1 = t.I1;
    }
    const int64_t ua = seg_units(a1 - lo, K), ub = seg_units(b1 - b0, K);
    if (u >= seen && u < seen + ua) {
      J = Jc;
      Ib = lo + (int)(u - seen) * K;
      kv = a1 - Ib < K ? a1 - Ib : K;
      return -1;
    }
    if (u >= seen + ua && u < seen + ua + ub) {
      J = Jc;
      Ib = b0 + (int)(u - seen - ua) * K;
      kv = b1 - Ib < K ? b1 - Ib : K;
      return -1;
    }
    seen += ua + ub;
  }
  return seen;
}

__device__ __forceinline__ void super_of(const abft_tiles_t& t, int mode, int K, int64_t su, int& Ib, int& J,
                                         int& kv) {
  kv = K;
  if (mode == PASS_SEG) {
    seg_of(t, K, su, Ib, J, kv);
    return;
  }
  if (mode == PASS_DIAG) {
    Ib = J = (t.I0 > t.J0 ? t.I0 : t.J0) + (int)su;
    return;
  }
  if (K == 1) {
    tile_of(t, su, Ib, J);
    return;
  }
  const int64_t nIk = (t.I1 - t.I0) / K;
  J = t.J0 + (int)(su / nIk);
  Ib = t.I0 + (int)(su % nIk) * K;
}

// Two CTAs per SM need <= 96 registers per thread: 2 x 9 warps spread over
// the 4 SM sub-partitions put 5 warps on one of them (16K registers each).
// The verify variant of stacked tiles otherwise takes 111 and runs one CTA
// per SM (fp32 nb=256 verify at 2.5 TB/s, ncu r01).
template <typename T, int NB, int K, bool VERIFY, bool LEAN>
__global__ void __maxnreg__(96) checksum_pass_kernel(const __grid_constant__ PassArgs p) {  // kBlock threads
  using C = PassCfg<T, NB, K, VERIFY, LEAN>;
  constexpr int RK = C::RK;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  T* ring = reinterpret_cast<T*>(smem_raw);
  T* symacc = ring + (size_t)C::NSTAGE * C::STAGE_ELEMS;  // [K][3][NB]
  T* rec = symacc;                                        // verify: recomputed [K][3][NB] (non-SYM tiles)
  uint64_t* full = reinterpret_cast<uint64_t*>(symacc + 3 * RK + C::REC_ELEMS);
  uint64_t* empty = full + C::NSTAGE;
  __shared__ int s_colflags[K], s_ncols[K], s_nrows[K], s_rowflags[K], s_st[K];
  __shared__ int s_last;

  if (p.gate && *p.gate == 0) return;  // whole grid skips (uniform): no barrier or ticket touched
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t unit = blockIdx.x;
  const int64_t sup = unit / p.nslab;
  const int slab = (int)(unit % p.nslab);
  int Ib, J, kv;
  super_of(p.tiles, p.mode, K, sup, Ib, J, kv);
  const int RV = K == 1 ? NB : kv * NB;  // valid rows of this unit (ragged PASS_SEG stacks: kv < K)
  const int view = (K == 1 && Ib == J && p.mode != PASS_SEG) ? p.tiles.diag_view : ABFT_GENERAL;
  const bool sym = view == ABFT_SYM_LOWER;
  const int nslab = p.nslab;
  // SYM column sums of a split tile go through the workspace (the finishing
  // CTA adds them to the row sums); an unsplit tile keeps them in smem
  T* symcol = (sym && nslab > 1) ? reinterpret_cast<T*>(p.symws) + (size_t)sup * NB * 3 : symacc;
  const int cols = NB / nslab;
  const int c0 = slab * cols;
  const int nst = cols / C::CC;
  const T* A = reinterpret_cast<const T*>(p.A);
  const T* tileA = A + (int64_t)J * NB * p.lda + (int64_t)Ib * NB;
  // phase-A and phase-B masks: SYM uses LOWER for columns, strict lower for rows
  const int viewA = sym ? ABFT_LOWER : view;
  // a single-side check skips the other direction's sums (a SYM tile needs
  // both: its column checksums are colsum(lower) + rowsum(strict lower));
  // uniform per CTA.  COL-only verifies (post-PD / post-PU / Fig. 4a re-checks)
  // then do half the consumer work per element.
  const bool do_cols = sym || (p.which & ABFT_COL);
  const bool do_rows = sym || (p.which & ABFT_ROW);

  if (tid == 0) {
    for (int t = 0; t < K; ++t) {
      s_colflags[t] = 0;
      s_ncols[t] = 0;
      s_nrows[t] = 0;
      s_rowflags[t] = 0;
    }
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
    T* ck = p.ckpt ? reinterpret_cast<T*>(p.ckpt) + ((int64_t)(Ib - p.tiles.I0) * NB) +
                         ((int64_t)(J - p.tiles.J0) * NB) * p.ldk
                   : nullptr;
    if (p.use_bulk && lane == 0) {
      // checkpoint: once stage h has landed, its columns go back out to ck
      auto store_stage = [&](int h) {
        const int sl = h % C::NSTAGE;
        mbar_wait(&full[sl], (uint32_t)((h / C::NSTAGE) & 1));
        const T* sb = ring + (size_t)sl * C::STAGE_ELEMS;
#pragma unroll 1
        for (int cc = 0; cc < C::CC; ++cc)
          bulk_s2g(ck + (int64_t)(c0 + h * C::CC + cc) * p.ldk, sb + cc * RK, RV * sizeof(T));
        bulk_commit();
      };
      for (int g = 0; g < nst; ++g) {
        const int slot = g % C::NSTAGE;
        if (g >= C::NSTAGE) {
          mbar_wait(&empty[slot], (uint32_t)(((g / C::NSTAGE) - 1) & 1));
          if (ck) bulk_wait_read<C::NSTAGE - 2>();  // stage g - NSTAGE's store has read the slot
        }
        T* dst = ring + (size_t)slot * C::STAGE_ELEMS;
        fence_proxy_async();
        mbar_arrive_expect_tx(&full[slot], (uint32_t)(C::CC * RV * sizeof(T)));
        const T* src = tileA + (int64_t)(c0 + g * C::CC) * p.lda;
#pragma unroll 1
        for (int cc = 0; cc < C::CC; ++cc)
          bulk_g2s(dst + cc * RK, src + (int64_t)cc * p.lda, RV * sizeof(T), &full[slot]);
        if (ck && g >= 1) store_stage(g - 1);
      }
      if (ck) {
        store_stage(nst - 1);
        bulk_wait_all();
        asm volatile("fence.proxy.async.global;" ::: "memory");
        __threadfence();
      }
    }
    // the checkpoint is complete before this CTA's tile can be finished (and
    // corrected by the fused locate, which patches the checkpoint too)
    if (ck) asm volatile("bar.sync 2, %0;" ::"n"(kBlock) : "memory");
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
  int my_colflags[K], my_ncols[K];
#pragma unroll
  for (int t = 0; t < K; ++t) {
    my_colflags[t] = 0;
    my_ncols[t] = 0;
  }
  // column finish of tile row Ib+t: encode writes c (and m_c); verify compares (c-6, c-7)
  auto finish_col = [&](int t, int jl, T pe, T pw, T pa) {
    if (sym) {
      symcol[jl] = pe;
      symcol[NB + jl] = pw;
      symcol[2 * NB + jl] = pa;
      return;
    }
    if (!(p.which & ABFT_COL)) return;
    {  // park the sums; encode's stores / verify's comparisons run after the
      // stage loop, one column per thread (a per-column compare by one lane
      // inside the loop serialised the warps: fp32 nb=256 verify 3.9 vs 5.4 TB/s)
      T* rc = rec + (size_t)t * 3 * NB;
      const int idx = jl - c0;
      rc[idx] = pe;
      rc[NB + idx] = pw;
      rc[2 * NB + idx] = pa;
    }
  };
  // verify: compare the slab's columns (recomputed in rec, maintained from global)
  auto compare_cols = [&]() {
#pragma unroll
    for (int t = 0; t < K; ++t) {
      if (t >= kv) break;
      const int I = Ib + t;
      const T* rc = rec + (size_t)t * 3 * NB;
      for (int idx = tid; idx < cols; idx += kThreads) {
        const int64_t gj = (int64_t)J * NB + c0 + idx;
        const T me = colchk[(int64_t)2 * I + gj * p.ldc], mw = colchk[(int64_t)2 * I + 1 + gj * p.ldc];
        const T pe = rc[idx], pw = rc[NB + idx], pa = rc[2 * NB + idx];
        const double m = p.use_mag ? (double)colmag[I + gj * p.ldcm] : (double)pa;
        T de, dw;
        const int f = check_pair<T>(me, mw, pe, pw, m, p.tau_fac, NB, &de, &dw);
        if (dcol) {
          dcol[(int64_t)2 * I + gj * p.ldc] = de;
          dcol[(int64_t)2 * I + 1 + gj * p.ldc] = dw;
        }
        my_colflags[t] |= f;
        my_ncols[t] += f & 1;
        if (p.refresh && !(f & 1)) {
          T* cc2 = colchk + (int64_t)2 * I + gj * p.ldc;
          cc2[0] = pe;
          cc2[1] = pw;
          if (colmag) colmag[I + gj * p.ldcm] = pa;
        }
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
        int cc = idx / RK, r = idx % RK;
        if (r < RV) buf[idx] = src[(int64_t)cc * p.lda + r];
      }
      consumer_sync();
    }
    // ---------------- phase A: column sums (one warp per column) ----------
    // this warp's columns of the stage: (s*CC + cc) % kWarps == warp (no per-column skip test)
#pragma unroll 1
    for (int cc = (warp - s * C::CC) & (kWarps - 1); do_cols && cc < C::CC; cc += kWarps) {
      const int jl = c0 + s * C::CC + cc;  // tile-local column
      const T* col = buf + cc * RK;
      if (viewA == ABFT_GENERAL) {
        // per tile t: sum_i (i+1) x_i with i = (32k' + lane)*VEC + v (k' = k - t*KPT)
        //   = (lane*VEC + 1) * S0 + sum (32*VEC*k' + v) x   (compile-time weights)
        T pe[K], s1[K], pa[K];
#pragma unroll
        for (int t = 0; t < K; ++t) pe[t] = s1[t] = pa[t] = T(0);
#pragma unroll
        for (int k = 0; k < C::KV; ++k) {
          constexpr int dummy = 0;
          (void)dummy;
          const int t = k / C::KPT;
          const int kl = k - t * C::KPT;
          T xv[C::VEC];  // rows of a ragged stack's missing tiles (t >= kv) are stale smem, never finished
          load_vec<T, C::VEC>(xv, col + (32 * k + lane) * C::VEC);
#pragma unroll
          for (int v = 0; v < C::VEC; ++v) {
            pe[t] = fadd(pe[t], xv[v]);
            s1[t] = ffma(T(32 * C::VEC * kl + v), xv[v], s1[t]);
            pa[t] = fadd(pa[t], fabs(xv[v]));
          }
        }
#pragma unroll
        for (int t = 0; t < K; ++t) {
          T e = pe[t], w = ffma(T(lane * C::VEC + 1), pe[t], s1[t]), a2 = pa[t];
#pragma unroll
          for (int m = 16; m >= 1; m >>= 1) {
            e = fadd(e, shfl_xor(e, m));
            w = fadd(w, shfl_xor(w, m));
            a2 = fadd(a2, shfl_xor(a2, m));
          }
          if (lane == t && t < kv) finish_col(t, jl, e, w, a2);  // tiles finished by different lanes in parallel
        }
      } else {  // masked diagonal views (K == 1 only)
        T pe = T(0), pw = T(0), pa = T(0);
        switch (viewA) {  // uniform per CTA
          case ABFT_LOWER: masked_colsum_vec<ABFT_LOWER, NB, C::VEC>(col, jl, lane, pe, pw, pa); break;
          case ABFT_UNIT_LOWER: masked_colsum_vec<ABFT_UNIT_LOWER, NB, C::VEC>(col, jl, lane, pe, pw, pa); break;
          default: masked_colsum_vec<ABFT_UPPER, NB, C::VEC>(col, jl, lane, pe, pw, pa); break;
        }
#pragma unroll
        for (int m = 16; m >= 1; m >>= 1) {
          pe = fadd(pe, shfl_xor(pe, m));
          pw = fadd(pw, shfl_xor(pw, m));
          pa = fadd(pa, shfl_xor(pa, m));
        }
        if (lane == 0) finish_col(0, jl, pe, pw, pa);
      }
    }
    // ---------------- phase B: row sums ---------------------------------
#pragma unroll
    for (int q = 0; q < C::RPT; ++q) {
      const int r = tid + q * kThreads;
      if (do_rows && r < RV) {
        if (view == ABFT_GENERAL) {
          // per CQ-column chunk: sum (jl+1) x with jl = base + cq  =  (base + 1) * S0 + sum_cq cq*x
#pragma unroll
          for (int ch = 0; ch < C::CC / C::CQ; ++ch) {
            T se = T(0), s1 = T(0), sa = T(0);
#pragma unroll
            for (int cq = 0; cq < C::CQ; ++cq) {
              const T x = buf[(ch * C::CQ + cq) * RK + r];
              se = fadd(se, x);
              s1 = ffma(T(cq), x, s1);
              sa = fadd(sa, fabs(x));
            }
            grp[q].e = fadd(grp[q].e, se);
            grp[q].w = fadd(grp[q].w, ffma(T(c0 + s * C::CC + ch * C::CQ + 1), se, s1));
            grp[q].a = fadd(grp[q].a, sa);
          }
        } else {
          const int jl0 = c0 + s * C::CC;
          switch (sym ? (int)ABFT_SYM_LOWER : view) {  // uniform per CTA
            case ABFT_SYM_LOWER: masked_rowsum_fast<ABFT_SYM_LOWER, C::CC, C::CQ, RK>(buf, r, jl0, grp[q]); break;
            case ABFT_LOWER: masked_rowsum_fast<ABFT_LOWER, C::CC, C::CQ, RK>(buf, r, jl0, grp[q]); break;
            case ABFT_UNIT_LOWER: masked_rowsum_fast<ABFT_UNIT_LOWER, C::CC, C::CQ, RK>(buf, r, jl0, grp[q]); break;
            default: masked_rowsum_fast<ABFT_UPPER, C::CC, C::CQ, RK>(buf, r, jl0, grp[q]); break;
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
    if (group_end && do_rows) {
      const int g = (c0 + (s + 1) * C::CC) / C::GC - 1;
#pragma unroll
      for (int q = 0; q < C::RPT; ++q) {
        const int r = tid + q * kThreads;
        if (r < RV) {
          if (nslab == 1) {
            tot[q].e = fadd(tot[q].e, grp[q].e);
            tot[q].w = fadd(tot[q].w, grp[q].w);
            tot[q].a = fadd(tot[q].a, grp[q].a);
          } else {
            T* dst = partT + (((size_t)sup * C::GROUPS + g) * RK + r) * 3;
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
  if (!sym && (p.which & ABFT_COL)) {
    consumer_sync();  // every column of the slab is parked in rec
    if (VERIFY) {
      compare_cols();
    } else {  // encode: one column per thread
#pragma unroll
      for (int t = 0; t < K; ++t) {
        if (t >= kv) break;
        const int I = Ib + t;
        const T* rc = rec + (size_t)t * 3 * NB;
        for (int idx = tid; idx < cols; idx += kThreads) {
          const int64_t gj = (int64_t)J * NB + c0 + idx;
          T* cc2 = colchk + (int64_t)2 * I + gj * p.ldc;
          cc2[0] = rc[idx];
          cc2[1] = rc[NB + idx];
          if (colmag) colmag[I + gj * p.ldcm] = rc[2 * NB + idx];
        }
      }
    }
  }
  if (VERIFY) {
#pragma unroll
    for (int t = 0; t < K; ++t) {
      const int f = __reduce_or_sync(0xffffffffu, my_colflags[t]);
      const int nc = __reduce_add_sync(0xffffffffu, my_ncols[t]);
      if (lane == 0 && (f | nc)) {
        atomicOr(&s_colflags[t], f);
        atomicAdd(&s_ncols[t], nc);
      }
    }
  }
  if (p.ckpt) asm volatile("bar.sync 2, %0;" ::"n"(kBlock) : "memory");  // the producer's checkpoint stores are done
  // ---------------- slab reduction: last CTA finishes the unit ------------
  if (nslab > 1) {
    __threadfence();
    consumer_sync();
    if (tid == 0) {
      if (VERIFY)
        for (int t = 0; t < K; ++t)
          if (s_colflags[t]) atomicOr(&p.tflags[sup * K + t], s_colflags[t]);
      __threadfence();
      int old = atomicAdd(&p.ticket[sup], 1);
      s_last = (old == nslab - 1);
    }
    consumer_sync();
    if (VERIFY && tid == 0)
      for (int t = 0; t < K; ++t)
        if (s_ncols[t]) atomicAdd(&p.counts[ABFT_CNT_COLS_FLAGGED], s_ncols[t]);
    if (!s_last) return;
    __threadfence();
#pragma unroll
    for (int q = 0; q < C::RPT; ++q) {
      const int r = tid + q * kThreads;
      if (do_rows && r < RV) {
        for (int g = 0; g < C::GROUPS; ++g) {
          const T* src = partT + (((size_t)sup * C::GROUPS + g) * RK + r) * 3;
          tot[q].e = fadd(tot[q].e, __ldcg(src + 0));
          tot[q].w = fadd(tot[q].w, __ldcg(src + 1));
          tot[q].a = fadd(tot[q].a, __ldcg(src + 2));
        }
      }
    }
    if (tid == 0) {
      if (VERIFY)
        for (int t = 0; t < K; ++t) {
          s_colflags[t] |= atomicExch(&p.tflags[sup * K + t], 0);
          s_ncols[t] = 0;  // already counted
        }
      p.ticket[sup] = 0;
    }
  } else {
    consumer_sync();
    if (VERIFY && tid == 0)
      for (int t = 0; t < K; ++t) {
        if (s_ncols[t]) atomicAdd(&p.counts[ABFT_CNT_COLS_FLAGGED], s_ncols[t]);
        s_ncols[t] = 0;
      }
  }

  // ---------------- finish rows (and SYM columns) -------------------------
  T* rowchk = reinterpret_cast<T*>(p.rowchk);
  T* rowmag = reinterpret_cast<T*>(p.rowmag);
  T* drow = reinterpret_cast<T*>(p.drow);
#pragma unroll
  for (int q = 0; q < C::RPT; ++q) {
    const int rr = tid + q * kThreads;
    if (rr >= RV) continue;
    const int t = rr / NB, r = rr - t * NB;
    const int I = Ib + t;
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
      int fr = 0, fc = 0;
      if (p.which & ABFT_ROW) {
        double m = p.use_mag ? (double)rowmag[gi + (int64_t)J * p.ldrm] : (double)ra;
        T de, dw;
        fr = check_pair<T>(rowchk[gi + (int64_t)(2 * J) * p.ldr], rowchk[gi + (int64_t)(2 * J + 1) * p.ldr], re, rw,
                           m, p.tau_fac, NB, &de, &dw);
        if (drow) {
          drow[gi + (int64_t)(2 * J) * p.ldr] = de;
          drow[gi + (int64_t)(2 * J + 1) * p.ldr] = dw;
        }
        if (p.refresh && !(fr & 1)) {
          rowchk[gi + (int64_t)(2 * J) * p.ldr] = re;
          rowchk[gi + (int64_t)(2 * J + 1) * p.ldr] = rw;
          if (rowmag) rowmag[gi + (int64_t)J * p.ldrm] = ra;
        }
      }
      if (sym && (p.which & ABFT_COL)) {
        double m = p.use_mag ? (double)colmag[I + gj * p.ldcm] : (double)ra;
        T de, dw;
        fc = check_pair<T>(colchk[(int64_t)2 * I + gj * p.ldc], colchk[(int64_t)2 * I + 1 + gj * p.ldc], re, rw, m,
                           p.tau_fac, NB, &de, &dw);
        if (dcol) {
          dcol[(int64_t)2 * I + gj * p.ldc] = de;
          dcol[(int64_t)2 * I + 1 + gj * p.ldc] = dw;
        }
        if (p.refresh && !(fc & 1)) {
          colchk[(int64_t)2 * I + gj * p.ldc] = re;
          colchk[(int64_t)2 * I + 1 + gj * p.ldc] = rw;
          if (colmag) colmag[I + gj * p.ldcm] = ra;
        }
      }
      if (fr) {
        atomicOr(&s_rowflags[t], fr);
        if (fr & 1) atomicAdd(&s_nrows[t], 1);
      }
      if (fc) {
        atomicOr(&s_colflags[t], fc);
        if (fc & 1) atomicAdd(&s_ncols[t], 1);
      }
    }
  }
  if (!VERIFY) return;
  consumer_sync();
  if (tid < kv) {
    const int t = tid, I = Ib + t;
    const int cf = s_colflags[t], rf = s_rowflags[t];
    const int st = ((cf & 1) ? ABFT_ST_COL : 0) | ((rf & 1) ? ABFT_ST_ROW : 0) | (((cf | rf) & 2) ? ABFT_ST_NONFINITE : 0);
    p.status[I + (int64_t)J * p.ld_status] = st;
    s_st[t] = st;
    if (st & (ABFT_ST_COL | ABFT_ST_ROW)) atomicAdd(&p.counts[ABFT_CNT_TILES_FLAGGED], 1);
    if (st & ABFT_ST_NONFINITE) atomicAdd(&p.counts[ABFT_CNT_NONFINITE], 1);
    if (s_nrows[t]) atomicAdd(&p.counts[ABFT_CNT_ROWS_FLAGGED], s_nrows[t]);
    if (s_ncols[t]) atomicAdd(&p.counts[ABFT_CNT_COLS_FLAGGED], s_ncols[t]);
  }
  if constexpr (C::FUSE_OK) {
    if (!p.fuse) return;
    // fused locate (a3): the tile's sums are final; its flagged tiles are
    // classified and corrected by this CTA, the ring and side area reused
    // as locate_tile's shared memory (every stage is consumed, the producer
    // warp has exited)
    consumer_sync();
    for (int t = 0; t < kv; ++t) {
      if (!(s_st[t] & (ABFT_ST_COL | ABFT_ST_ROW))) continue;  // uniform
      __threadfence();
      locate_tile<T>(p.loc, Ib + t, J, p.status + (Ib + t) + (int64_t)J * p.ld_status, smem_raw);
    }
  }
}

// ------------------------------------------------------------ launcher --
// set by launch_k when a fused check fell on an instantiation whose locate
// tables do not fit (fp64 nb=1024): run_pass then launches locate itself
static thread_local bool g_fuse_missed = false;

template <typename T, int NB, int K, bool VERIFY, bool LEAN>
static int launch_cfg(PassArgs& a, int64_t nsup, int nslab, cudaStream_t s) {
  using C = PassCfg<T, NB, K, VERIFY, LEAN>;
  auto kern = checksum_pass_kernel<T, NB, K, VERIFY, LEAN>;
  static bool attr_done = false;  // per instantiation
  if (!attr_done) {
    ABFT_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)C::SMEM));
    attr_done = true;
  }
  const int64_t ntiles = nsup * K;  // tile slots of the workspace (ragged stacks included)
  a.nslab = nslab;
  a.K = K;
  const int want_fuse = a.fuse;
  a.fuse = want_fuse && C::FUSE_OK;
  if (want_fuse && !C::FUSE_OK) g_fuse_missed = true;  // the caller launches locate separately
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
  dim3 grid((unsigned)(nsup * nslab));
  kern<<<grid, kBlock, C::SMEM, s>>>(a);
  a.fuse = want_fuse;
  ABFT_CUDA_TRY(cudaGetLastError());
  return 0;
}

template <typename T, int NB, int K, bool VERIFY>
static int launch_k(PassArgs& a, int64_t nsup, cudaStream_t s) {
  using C = PassCfg<T, NB, K, VERIFY>;
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || sms <= 0) sms = 148;
  }
  // slabs: split the units of a small launch so that it fills, but does not
  // spill past, one wave of 2 CTAs per SM (a spilled second wave cost more
  // than the halved slab saved: 40-59-tile panels 10% slower, slab_tune r01)
  int nslab = 1;
  const int max_slab = C::GROUPS;
  while (nslab < max_slab && nsup * nslab * 2 <= 2LL * sms) nslab *= 2;
  static const int force_slab = getenv("ABFT_NSLAB") ? atoi(getenv("ABFT_NSLAB")) : 0;  // tuning experiments only
  if (force_slab > 0) nslab = std::min(force_slab, max_slab);
  if constexpr (VERIFY) {
    if (nsup * nslab <= 2LL * sms) return launch_cfg<T, NB, K, VERIFY, true>(a, nsup, nslab, s);
  }
  return launch_cfg<T, NB, K, VERIFY, false>(a, nsup, nslab, s);
}

// Small tiles are streamed K at a time (K*NB*s >= 4 KiB per column copy):
// a rectangular GENERAL range whose height K divides in one PASS_RECT
// launch; any other range (lower_only, ragged height, masked diagonal view)
// as PASS_SEG stacks of its GENERAL tiles plus, when the diagonal view is
// masked, one PASS_DIAG launch over the diagonal tiles.
template <typename T, int NB, bool VERIFY>
static int launch_nb(PassArgs& a, int64_t ntiles, cudaStream_t s) {
  constexpr int KR = 4096 / (NB * (int)sizeof(T));
  constexpr int KBIG = KR < 1 ? 1 : (KR > 8 ? 8 : KR);
  constexpr int VEC = NB >= 32 * (16 / (int)sizeof(T)) ? 16 / (int)sizeof(T) : 1;
  constexpr bool can = KBIG > 1 && NB % (32 * VEC) == 0;
  a.mode = PASS_RECT;
  if constexpr (can) {
    const abft_tiles_t& t = a.tiles;
    const int D0 = std::max(t.I0, t.J0), D1 = std::min(t.I1, t.J1);
    const bool split = t.diag_view != ABFT_GENERAL && D1 > D0;
    if (!t.lower_only && !split && (t.I1 - t.I0) % KBIG == 0) return launch_k<T, NB, KBIG, VERIFY>(a, ntiles / KBIG, s);
    if (split) {
      a.mode = PASS_DIAG;
      const int rc = launch_k<T, NB, 1, VERIFY>(a, D1 - D0, s);
      if (rc) return rc;
    }
    int Ib, J, kv;
    const int64_t nseg = seg_of(t, KBIG, -1, Ib, J, kv);
    if (nseg == 0) return 0;
    a.mode = PASS_SEG;
    return launch_k<T, NB, KBIG, VERIFY>(a, nseg, s);
  }
  return launch_k<T, NB, 1, VERIFY>(a, ntiles, s);
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
                    const abft_report_t* rep, cudaStream_t s, bool verify, const LocArgs* loc = nullptr,
                    void* ckpt = nullptr, int64_t ldk = 0) {
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
  a.gate = launch_gate();
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
  // the checkpoint rides on the bulk-copy ring (16-B aligned columns)
  const bool ck_fused = ckpt && a.use_bulk && (uintptr_t)ckpt % 16 == 0 && (ldk * (int64_t)es) % 16 == 0;
  if (loc) {
    a.fuse = 1;
    a.loc = *loc;
    if (ck_fused) {
      a.loc.ckpt = ckpt;
      a.loc.ldk = ldk;
    }
  }
  if (ck_fused) {
    a.ckpt = ckpt;
    a.ldk = ldk;
  }
  g_fuse_missed = false;
  if (m->dtype == ABFT_F64)
    rc = verify ? launch_t<double, true>(a, m->nb, ntiles, s) : launch_t<double, false>(a, m->nb, ntiles, s);
  else
    rc = verify ? launch_t<float, true>(a, m->nb, ntiles, s) : launch_t<float, false>(a, m->nb, ntiles, s);
  if (rc) return rc;
  if (loc && g_fuse_missed) {
    LocArgs la = a.loc;
    rc = launch_locate_args(la, m->dtype, s);
    if (rc) return rc;
  }
  if (ckpt && !ck_fused) {  // the checkpoint as a plain copy of the checked (and corrected) range
    const int64_t nb = m->nb;
    return copy2d(ckpt, ldk * es, (const char*)m->A + ((int64_t)t->I0 * nb + (int64_t)t->J0 * nb * m->lda) * es,
                  m->lda * es, (size_t)(t->I1 - t->I0) * nb * es, (size_t)(t->J1 - t->J0) * nb, s);
  }
  return 0;
}

int check_ckpt(const abft_mat_t* mat, const abft_tiles_t* tiles, int32_t which, const abft_tol_t* tol,
               const abft_report_t* report, abft_fix_t* fixes, int32_t max_fixes, int32_t* n_fixes, void* ckpt,
               int64_t ldk, cudaStream_t s) {
  LocArgs la;
  const int rc = fill_loc_args(la, mat, tiles, which, tol, report, fixes, max_fixes, n_fixes);
  if (rc) return rc;
  return run_pass(mat, tiles, which, tol, report, s, true, &la, ckpt, ldk);
}

}  // namespace abft

extern "C" int abft_encode(const abft_mat_t* mat, const abft_tiles_t* tiles, int32_t which, abft_stream_t stream) {
  return abft::run_pass(mat, tiles, which, nullptr, nullptr, (cudaStream_t)stream, false);
}

extern "C" int abft_verify(const abft_mat_t* mat, const abft_tiles_t* tiles, int32_t which, const abft_tol_t* tol,
                           const abft_report_t* report, abft_stream_t stream) {
  return abft::run_pass(mat, tiles, which, tol, report, (cudaStream_t)stream, true);
}

extern "C" int abft_check(const abft_mat_t* mat, const abft_tiles_t* tiles, int32_t which, const abft_tol_t* tol,
                          const abft_report_t* report, abft_fix_t* fixes, int32_t max_fixes, int32_t* n_fixes,
                          abft_stream_t stream) {
  abft::LocArgs la;
  const int rc = abft::fill_loc_args(la, mat, tiles, which, tol, report, fixes, max_fixes, n_fixes);
  if (rc) return rc;
  return abft::run_pass(mat, tiles, which, tol, report, (cudaStream_t)stream, true, &la);
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
