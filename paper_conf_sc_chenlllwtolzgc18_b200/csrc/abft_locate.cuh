// abft_locate.cuh — the per-tile locate / classify / correct routine (a3),
// shared by locate_correct_kernel (abft_locate.cu) and the fused check
// (abft_pass.cu).  See abft_locate.cu for the paper passages and readings.
#pragma once
#include "abft_common.cuh"

namespace abft {

constexpr int kLThreads = 256;
constexpr int kLWarps = kLThreads / 32;
constexpr int kMaxRounds = 3;

enum ActKind { ACT_FIX_COL = 0, ACT_FIX_ROW = 1, ACT_REENC_COL = 2, ACT_REENC_ROW = 3 };

struct LocArgs {
  void* A;
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
  int nb;
  int which;
  int use_mag;
  double tau_fac;
  int32_t* status;
  int64_t ld_status;
  int32_t* counts;
  abft_fix_t* fixes;
  int32_t max_fixes;
  int32_t* n_fixes;
  int64_t ntiles;
  const int32_t* gate;  // nullable: run only if *gate != 0
  // drivers' local-restart checkpoint of the checked range (nullable): a
  // data fix also lands at ckpt[(gi - I0 nb) + (gj - J0 nb) ldk]
  void* ckpt;
  int64_t ldk;
};

template <typename T>
struct TileCtx {
  const LocArgs* p;
  int I, J, view;
  T* A;
  __device__ __forceinline__ void stored(int i, int j, int& si, int& sj) const {
    if (view == ABFT_SYM_LOWER) {
      si = i > j ? i : j;
      sj = i > j ? j : i;
    } else {
      si = i;
      sj = j;
    }
  }
  __device__ __forceinline__ T* addr(int i, int j) const {
    int si, sj;
    stored(i, j, si, sj);
    return A + ((int64_t)J * p->nb + sj) * p->lda + (int64_t)I * p->nb + si;
  }
  __device__ __forceinline__ T x(int i, int j) const {
    T v = *addr(i, j);
    switch (view) {
      case ABFT_LOWER: return i >= j ? v : T(0);
      case ABFT_UNIT_LOWER: return i > j ? v : (i == j ? T(1) : T(0));
      case ABFT_UPPER: return i <= j ? v : T(0);
      default: return v;
    }
  }
  __device__ __forceinline__ bool live(int i, int j) const {
    switch (view) {
      case ABFT_LOWER: return i >= j;
      case ABFT_UNIT_LOWER: return i > j;
      case ABFT_UPPER: return i <= j;
      default: return true;
    }
  }
  __device__ __forceinline__ T* colchk_e(int j) const {
    return reinterpret_cast<T*>(p->colchk) + (int64_t)2 * I + ((int64_t)J * p->nb + j) * p->ldc;
  }
  __device__ __forceinline__ T* rowchk_e(int i) const {
    return reinterpret_cast<T*>(p->rowchk) + (int64_t)I * p->nb + i + (int64_t)(2 * J) * p->ldr;
  }
  __device__ __forceinline__ T* colmag_at(int j) const {
    return reinterpret_cast<T*>(p->colmag) + I + ((int64_t)J * p->nb + j) * p->ldcm;
  }
  __device__ __forceinline__ T* rowmag_at(int i) const {
    return reinterpret_cast<T*>(p->rowmag) + (int64_t)I * p->nb + i + (int64_t)J * p->ldrm;
  }
};

// Per-direction tables in shared memory (index = column or row of the tile).
template <typename T>
struct Dir {
  T *se, *sw, *sa;      // recomputed sums
  T *de, *dw;           // delta = maintained - recomputed
  double* tau;          // tau_e
  unsigned char* fl;    // bit0 e flagged, bit1 w flagged, bit2 non-finite
  int* loc;             // located index, -1 = none
};

template <typename T>
__device__ T warp_sum(T v) {
#pragma unroll
  for (int m = 16; m >= 1; m >>= 1) v = fadd(v, shfl_xor(v, m));
  return v;
}

__device__ __forceinline__ int locate_ratio(double de, double dw, double te, int nb) {
  // c-5: q = dw/de in fp64, j = rint(q), |q-j| <= 0.25, 1 <= j <= nb,
  // |dw - j de| <= tau_w + j tau_e (tau_w = nb tau_e)
  if (!isfinite(de) || !isfinite(dw) || de == 0.0) return -1;
  double q = dw / de;
  if (!isfinite(q)) return -1;
  double j = rint(q);
  if (fabs(q - j) > 0.25 || j < 1.0 || j > (double)nb) return -1;
  if (!(fabs(dw - j * de) <= (double)nb * te + j * te)) return -1;
  return (int)j - 1;
}

struct Action {
  short kind, cls;
  int i, j;
};

struct LocShared {
  int nact, cls, nfc, nfr, fc0, fr0, done, final, data_fixes, chk_fixes;
};

// Named barrier 1 over the 256 locate threads (the fused check's producer
// warp has exited by then; the standalone kernel has exactly 256 threads).
__device__ __forceinline__ void loc_sync() { asm volatile("bar.sync 1, 256;" ::: "memory"); }

// Shared memory of locate_tile: two Dir tables, the action list (2 nb), the
// per-round words.
__host__ __device__ constexpr size_t loc_tables_bytes(int nb, int es) {
  return 2 * (((size_t)nb * (5 * es + 8 + 4 + 1) + 15) / 16 * 16);
}
__host__ __device__ constexpr size_t locate_smem_bytes(int nb, int es) {
  return loc_tables_bytes(nb, es) + (size_t)2 * nb * sizeof(Action) + sizeof(LocShared) + 16;
}

// One flagged tile (I, J), status word stp: up to kMaxRounds rounds of
// recompute -> classify (c-11) -> correct.  Run by the 256 threads 0..255
// of the calling CTA (named barrier 1), with `sm` = locate_smem_bytes(nb,
// sizeof(T)) bytes of shared memory.  Called by locate_correct_kernel and by
// the fused check (abft_pass.cu: the finishing CTA of a flagged tile).
template <typename T>
__device__ __noinline__ void locate_tile(const LocArgs& p, int I, int J, int32_t* stp, unsigned char* sm) {
  const int nb = p.nb;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  Dir<T> D[2];
  unsigned char* q = sm;
  for (int d = 0; d < 2; ++d) {
    D[d].se = reinterpret_cast<T*>(q); q += nb * sizeof(T);
    D[d].sw = reinterpret_cast<T*>(q); q += nb * sizeof(T);
    D[d].sa = reinterpret_cast<T*>(q); q += nb * sizeof(T);
    D[d].de = reinterpret_cast<T*>(q); q += nb * sizeof(T);
    D[d].dw = reinterpret_cast<T*>(q); q += nb * sizeof(T);
    D[d].tau = reinterpret_cast<double*>(q); q += nb * sizeof(double);
    D[d].loc = reinterpret_cast<int*>(q); q += nb * sizeof(int);
    D[d].fl = q; q += nb;
    q = reinterpret_cast<unsigned char*>(((uintptr_t)q + 15) & ~(uintptr_t)15);
  }
  Action* acts = reinterpret_cast<Action*>(sm + loc_tables_bytes(nb, (int)sizeof(T)));
  LocShared* sh = reinterpret_cast<LocShared*>(acts + 2 * nb);
  const int max_act = 2 * nb;
  const bool has_c = p.which & ABFT_COL, has_r = p.which & ABFT_ROW;
    TileCtx<T> X{&p, I, J, (I == J) ? p.tiles.diag_view : ABFT_GENERAL, reinterpret_cast<T*>(p.A)};
    const bool sym = X.view == ABFT_SYM_LOWER;
    if (tid == 0) {
      sh->data_fixes = 0;
      sh->chk_fixes = 0;
      sh->final = ABFT_CLS_2D;
    }
    for (int round = 0; round <= kMaxRounds; ++round) {
      // ---- recompute sums and flags -----------------------------------
      if (has_c) {
        for (int j = warp; j < nb; j += kLWarps) {
          T e = T(0), w = T(0), a = T(0);
          for (int i = lane; i < nb; i += 32) {
            T v = X.x(i, j);
            e = fadd(e, v);
            w = ffma(T(i + 1), v, w);
            a = fadd(a, fabs(v));
          }
          e = warp_sum(e);
          w = warp_sum(w);
          a = warp_sum(a);
          if (lane == 0) {
            D[0].se[j] = e;
            D[0].sw[j] = w;
            D[0].sa[j] = a;
          }
        }
      }
      if (has_r) {
        for (int i = tid; i < nb; i += kLThreads) {
          T e = T(0), w = T(0), a = T(0);
          for (int j = 0; j < nb; ++j) {
            T v = X.x(i, j);
            e = fadd(e, v);
            w = ffma(T(j + 1), v, w);
            a = fadd(a, fabs(v));
          }
          D[1].se[i] = e;
          D[1].sw[i] = w;
          D[1].sa[i] = a;
        }
      }
      loc_sync();
      for (int k = tid; k < nb; k += kLThreads) {
        for (int d = 0; d < 2; ++d) {
          if ((d == 0 && !has_c) || (d == 1 && !has_r)) {
            D[d].fl[k] = 0;
            continue;
          }
          T me, mw;
          double m;
          if (d == 0) {
            me = X.colchk_e(k)[0];
            mw = X.colchk_e(k)[1];
            m = p.use_mag ? (double)*X.colmag_at(k) : (double)D[0].sa[k];
          } else {
            me = X.rowchk_e(k)[0];
            mw = X.rowchk_e(k)[p.ldr];
            m = p.use_mag ? (double)*X.rowmag_at(k) : (double)D[1].sa[k];
          }
          T de = me - D[d].se[k], dw = mw - D[d].sw[k];
          double tau = p.tau_fac * m;
          bool nfe = !isfinite((double)de), nfw = !isfinite((double)dw);
          bool fe = nfe || fabs((double)de) > tau;
          bool fw = nfw || fabs((double)dw) > (double)nb * tau;
          D[d].de[k] = de;
          D[d].dw[k] = dw;
          D[d].tau[k] = tau;
          D[d].fl[k] = (fe ? 1 : 0) | (fw ? 2 : 0) | ((nfe || nfw) ? 4 : 0);
          D[d].loc[k] = -1;
        }
      }
      loc_sync();
      if (tid == 0) {
        int nfc = 0, nfr = 0, fc0 = -1, fr0 = -1;
        for (int k = 0; k < nb; ++k) {
          if (D[0].fl[k] & 3) {
            if (fc0 < 0) fc0 = k;
            ++nfc;
          }
          if (D[1].fl[k] & 3) {
            if (fr0 < 0) fr0 = k;
            ++nfr;
          }
        }
        sh->nfc = nfc;
        sh->nfr = nfr;
        sh->fc0 = fc0;
        sh->fr0 = fr0;
        sh->done = 0;
        if (nfc == 0 && nfr == 0) {
          sh->done = 1;
          sh->final = ABFT_CLS_CLEAN;
        } else if (round == kMaxRounds) {
          sh->done = 1;
          sh->final = ABFT_CLS_2D;
        }
      }
      loc_sync();
      if (sh->done) break;
      const int nfc = sh->nfc, nfr = sh->nfr;
      // ---- locate every flagged column / row (c-5, c-7) ------------------
      for (int d = 0; d < 2; ++d) {
        const bool active = d == 0 ? has_c : has_r;
        if (!active) continue;
        for (int k = warp; k < nb; k += kLWarps) {
          if (!(D[d].fl[k] & 3)) continue;
          int li = locate_ratio((double)D[d].de[k], (double)D[d].dw[k], D[d].tau[k], nb);
          if (li >= 0) {
            bool lv = d == 0 ? X.live(li, k) : X.live(k, li);
            if (lane == 0) D[d].loc[k] = lv ? li : -1;
            continue;
          }
          // fallback candidate
          int cand = -1;
          const bool other = d == 0 ? has_r : has_c;
          if (other && nfc == 1 && nfr == 1) {
            cand = d == 0 ? sh->fr0 : sh->fc0;
          } else {
            int nnf = 0, nfidx = nb;
            double best = -1.0;
            int bidx = nb;
            for (int r = lane; r < nb; r += 32) {
              T v = d == 0 ? X.x(r, k) : X.x(k, r);
              double av = fabs((double)v);
              if (!isfinite((double)v)) {
                ++nnf;
                nfidx = min(nfidx, r);
              } else if (av > best || (av == best && r < bidx)) {
                best = av;
                bidx = r;
              }
            }
#pragma unroll
            for (int m = 16; m >= 1; m >>= 1) {
              nnf += __shfl_xor_sync(0xffffffffu, nnf, m);
              nfidx = min(nfidx, __shfl_xor_sync(0xffffffffu, nfidx, m));
              double ob = __shfl_xor_sync(0xffffffffu, best, m);
              int oi = __shfl_xor_sync(0xffffffffu, bidx, m);
              if (ob > best || (ob == best && oi < bidx)) {
                best = ob;
                bidx = oi;
              }
            }
            if (nnf == 1)
              cand = nfidx;
            else if (nnf > 1)
              cand = -1;
            else
              cand = bidx < nb ? bidx : -1;
          }
          bool ok = cand >= 0 && (d == 0 ? X.live(cand, k) : X.live(k, cand));
          if (ok) {
            // confirm: tentative c-4 correction, then both residuals within tau
            T ce = d == 0 ? X.colchk_e(k)[0] : X.rowchk_e(k)[0];
            T cw = d == 0 ? X.colchk_e(k)[1] : X.rowchk_e(k)[p.ldr];
            T rest = T(0);
            for (int r = lane; r < nb; r += 32)
              if (r != cand) rest = fadd(rest, d == 0 ? X.x(r, k) : X.x(k, r));
            rest = warp_sum(rest);
            T nv = ce - rest;
            T e = T(0), w = T(0), a = T(0);
            for (int r = lane; r < nb; r += 32) {
              T v = (r == cand) ? nv : (d == 0 ? X.x(r, k) : X.x(k, r));
              e = fadd(e, v);
              w = ffma(T(r + 1), v, w);
              a = fadd(a, fabs(v));
            }
            e = warp_sum(e);
            w = warp_sum(w);
            a = warp_sum(a);
            double m;
            if (p.use_mag)
              m = d == 0 ? (double)*X.colmag_at(k) : (double)*X.rowmag_at(k);
            else
              m = (double)a;
            double tau = p.tau_fac * m;
            double de = (double)(ce - e), dw = (double)(cw - w);
            ok = isfinite(de) && isfinite(dw) && fabs(de) <= tau && fabs(dw) <= (double)nb * tau;
          }
          if (lane == 0) D[d].loc[k] = ok ? cand : -1;
        }
      }
      loc_sync();
      // ---- classify (thread 0), c-11 -----------------------------------
      if (tid == 0) {
        int na = 0, cls = ABFT_CLS_2D;
        auto push = [&](int kind, int i, int j, int c) {
          if (na < max_act) acts[na++] = Action{(short)kind, (short)c, i, j};
        };
        bool decided = false;
        // step 3: columns locate one row
        if (!decided && has_c && nfc) {
          int i0 = -2;
          bool ok = true;
          for (int j = 0; j < nb && ok; ++j)
            if (D[0].fl[j] & 3) {
              int l = D[0].loc[j];
              if (l < 0 || (i0 != -2 && l != i0)) ok = false;
              i0 = l;
            }
          if (ok && has_r)
            for (int i = 0; i < nb && ok; ++i)
              if ((D[1].fl[i] & 3) && i != i0) ok = false;
          if (ok) {
            cls = nfc == 1 ? ABFT_CLS_0D : ABFT_CLS_1D_ROW;
            for (int j = 0; j < nb; ++j)
              if (D[0].fl[j] & 3) push(ACT_FIX_COL, i0, j, cls);
            decided = true;
          }
        }
        // step 4: rows locate one column
        if (!decided && has_r && nfr) {
          int j0 = -2;
          bool ok = true;
          for (int i = 0; i < nb && ok; ++i)
            if (D[1].fl[i] & 3) {
              int l = D[1].loc[i];
              if (l < 0 || (j0 != -2 && l != j0)) ok = false;
              j0 = l;
            }
          if (ok && has_c)
            for (int j = 0; j < nb && ok; ++j)
              if ((D[0].fl[j] & 3) && j != j0) ok = false;
          if (ok) {
            cls = nfr == 1 ? ABFT_CLS_0D : ABFT_CLS_1D_COL;
            for (int i = 0; i < nb; ++i)
              if (D[1].fl[i] & 3) push(ACT_FIX_ROW, i, j0, cls);
            decided = true;
          }
        }
        // step 2 (after steps 3-4, reading c-11b): a lone e- or w-flag that no
        // consistent data location explains => the checksum entry is corrupt
        bool rep = false;
        if (!decided && has_c && nfc && (!has_r || !nfr))
          for (int j = 0; j < nb; ++j) {
            unsigned f = D[0].fl[j];
            if ((f & 3) && ((f & 1) != 0) != ((f & 2) != 0)) {
              push(ACT_REENC_COL, -1, j, ABFT_CLS_CHK_CORRUPT);
              rep = true;
            }
          }
        if (!decided && has_r && nfr && (!has_c || !nfc))
          for (int i = 0; i < nb; ++i) {
            unsigned f = D[1].fl[i];
            if ((f & 3) && ((f & 1) != 0) != ((f & 2) != 0)) {
              push(ACT_REENC_ROW, i, -1, ABFT_CLS_CHK_CORRUPT);
              rep = true;
            }
          }
        if (rep) {
          cls = ABFT_CLS_CHK_CORRUPT;
          decided = true;
        }
        if (!decided && sym && has_c) {
          // step 5: mirrored pair
          if (nfc == 2) {
            int pcol = -1, qcol = -1;
            for (int j = 0; j < nb; ++j)
              if (D[0].fl[j] & 3) {
                if (pcol < 0) pcol = j; else qcol = j;
              }
            if (D[0].loc[qcol] == pcol && D[0].loc[pcol] == qcol) {
              push(ACT_FIX_COL, pcol, qcol, ABFT_CLS_0D);
              cls = ABFT_CLS_0D;
              decided = true;
            }
          }
          // step 6: SYM_CROSS
          if (!decided && nfc >= 2) {
            for (int r = 0; r < nb && !decided; ++r) {
              if (!(D[0].fl[r] & 3)) continue;
              bool ok = true;
              for (int j = 0; j < nb && ok; ++j)
                if (j != r && (D[0].fl[j] & 3) && D[0].loc[j] != r) ok = false;
              if (ok) {
                for (int j = 0; j < nb; ++j)
                  if (j != r && (D[0].fl[j] & 3)) push(ACT_FIX_COL, r, j, ABFT_CLS_SYM_CROSS);
                cls = ABFT_CLS_SYM_CROSS;
                decided = true;
              }
            }
          }
        }
        // step 5b: stale side (after steps 3-6, so a genuine 1D error seen by
        // one side is always corrected first)
        if (!decided && has_c && has_r) {
          if (nfr && !nfc) {
            for (int i = 0; i < nb; ++i)
              if (D[1].fl[i] & 3) push(ACT_REENC_ROW, i, -1, ABFT_CLS_STALE_R);
            cls = ABFT_CLS_STALE_R;
            decided = true;
          } else if (nfc && !nfr) {
            for (int j = 0; j < nb; ++j)
              if (D[0].fl[j] & 3) push(ACT_REENC_COL, -1, j, ABFT_CLS_STALE_C);
            cls = ABFT_CLS_STALE_C;
            decided = true;
          }
        }
        sh->nact = decided ? na : 0;
        sh->cls = decided ? cls : ABFT_CLS_2D;
      }
      loc_sync();
      if (sh->cls == ABFT_CLS_2D) {
        if (tid == 0) sh->final = ABFT_CLS_2D;
        break;
      }
      // ---- execute actions (warp per action) ---------------------------
      for (int a = warp; a < sh->nact; a += kLWarps) {
        Action ac = acts[a];
        if (ac.kind == ACT_FIX_COL || ac.kind == ACT_FIX_ROW) {
          const bool viacol = ac.kind == ACT_FIX_COL;
          const int line = viacol ? ac.j : ac.i;  // the column / row used
          const int skip = viacol ? ac.i : ac.j;
          T rest = T(0);
          for (int r = lane; r < nb; r += 32)
            if (r != skip) rest = fadd(rest, viacol ? X.x(r, line) : X.x(line, r));
          rest = warp_sum(rest);
          if (lane == 0) {
            T ce = viacol ? X.colchk_e(line)[0] : X.rowchk_e(line)[0];
            T nv = ce - rest;
            T* ptr = X.addr(ac.i, ac.j);
            T before = *ptr;
            *ptr = nv;
            int si, sj;
            X.stored(ac.i, ac.j, si, sj);
            if (p.ckpt)
              reinterpret_cast<T*>(p.ckpt)[((int64_t)(I - p.tiles.I0) * nb + si) +
                                           ((int64_t)(J - p.tiles.J0) * nb + sj) * p.ldk] = nv;
            int slot = atomicAdd(p.n_fixes, 1);
            if (slot < p.max_fixes && p.fixes) {
              abft_fix_t f;
              f.gi = (int64_t)I * nb + si;
              f.gj = (int64_t)J * nb + sj;
              f.before = (double)before;
              f.after = (double)nv;
              f.cls = ac.cls;
              f.kind = ABFT_FIX_DATA;
              p.fixes[slot] = f;
            }
            atomicAdd(&sh->data_fixes, 1);
          }
        } else {
          const bool col = ac.kind == ACT_REENC_COL;
          const int k = col ? ac.j : ac.i;
          T e = T(0), w = T(0), aa = T(0);
          for (int r = lane; r < nb; r += 32) {
            T v = col ? X.x(r, k) : X.x(k, r);
            e = fadd(e, v);
            w = ffma(T(r + 1), v, w);
            aa = fadd(aa, fabs(v));
          }
          e = warp_sum(e);
          w = warp_sum(w);
          aa = warp_sum(aa);
          if (lane == 0) {
            T before;
            if (col) {
              T* c = X.colchk_e(k);
              before = c[0];
              c[0] = e;
              c[1] = w;
              if (p.colmag) *X.colmag_at(k) = aa;
            } else {
              T* r = X.rowchk_e(k);
              before = r[0];
              r[0] = e;
              r[p.ldr] = w;
              if (p.rowmag) *X.rowmag_at(k) = aa;
            }
            int slot = atomicAdd(p.n_fixes, 1);
            if (slot < p.max_fixes && p.fixes) {
              abft_fix_t f;
              f.gi = col ? I : (int64_t)I * nb + k;
              f.gj = col ? (int64_t)J * nb + k : J;
              f.before = (double)before;
              f.after = (double)e;
              f.cls = ac.cls;
              f.kind = col ? ABFT_FIX_COLCHK : ABFT_FIX_ROWCHK;
              p.fixes[slot] = f;
            }
            atomicAdd(&sh->chk_fixes, 1);
          }
        }
      }
      __threadfence_block();
      loc_sync();
    }
    loc_sync();
    if (tid == 0) {
      if (sh->final == ABFT_CLS_CLEAN) {
        *stp = 0;
        atomicAdd(&p.counts[ABFT_CNT_TILES_FIXED], 1);
      } else {
        *stp = ABFT_ST_UNCORRECTABLE;
        atomicAdd(&p.counts[ABFT_CNT_UNCORRECTABLE], 1);
      }
      if (sh->data_fixes) atomicAdd(&p.counts[ABFT_CNT_ELEMS_FIXED], sh->data_fixes);
      if (sh->chk_fixes) atomicAdd(&p.counts[ABFT_CNT_CHK_REPAIRED], sh->chk_fixes);
    }
    loc_sync();
  loc_sync();
}

// LocArgs of one locate call (validation as abft_locate_correct's); the
// standalone launch of it (abft_locate.cu).
int fill_loc_args(LocArgs& a, const abft_mat_t* m, const abft_tiles_t* t, int32_t which, const abft_tol_t* tol,
                  const abft_report_t* rep, abft_fix_t* fixes, int32_t max_fixes, int32_t* n_fixes);
int launch_locate_args(LocArgs& a, int32_t dtype, cudaStream_t s);

}  // namespace abft
