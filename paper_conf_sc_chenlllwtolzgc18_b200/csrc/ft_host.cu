// ft_host.cu — pd_location = FT_PD_HOST: Alg. 2 lines 3-7 as the paper runs
// them (L364-L372; MAGMA's CPU panel, L61).  Per iteration the panel goes to
// pinned host memory, is factored there by the host LAPACK, and comes back.
//
// Transfer protection (reading c-28): each direction carries a
// fresh column-checksum guard c(X) = [v1 v2]^T X per nb-row tile (L111/L446)
// encoded by the sender right before the copy.
//   D2H: abft_encode on the device -> copy -> host recomputes and compares
//        (tau = 2 gamma_nb e^T|x|), locates each flagged column by the ratio
//        rule (c-5) or the c-7 candidate, corrects by c-4 and re-checks the
//        column; anything left -> fetch again (the device copy is intact),
//        at most 2 repeats.
//   H2D: host guard of the factored panel -> copy -> abft_verify +
//        abft_locate_correct on the device (GENERAL, COL, posteriori tau);
//        an uncorrectable tile -> send again, at most 2 repeats.
// The maintained checksums were checked on the device before line 3 (the
// pre-PD check) and the PD checksum rule + post-PD check follow on the
// device, so the guard covers exactly the two transfers.
#include <dlfcn.h>
#include <math.h>
#include <sched.h>

#include <thread>

#include "ft_driver.cuh"

namespace abft {
namespace {

typedef void (*potrf_d_t)(const char*, const int*, double*, const int*, int*, size_t);
typedef void (*potrf_s_t)(const char*, const int*, float*, const int*, int*, size_t);
typedef void (*getrf_d_t)(const int*, const int*, double*, const int*, int*, int*);
typedef void (*getrf_s_t)(const int*, const int*, float*, const int*, int*, int*);
typedef void (*geqrf_d_t)(const int*, const int*, double*, const int*, double*, double*, const int*, int*);
typedef void (*geqrf_s_t)(const int*, const int*, float*, const int*, float*, float*, const int*, int*);

// Host cores for the guard / check loops: the half of the process's cores
// that ft_ctx_set_host_lapack leaves to us (OpenBLAS gets the other half: its
// idle threads spin, so sharing all cores slows both sides down).
int64_t g_host_threads = 8;

// Columns of a panel split over the host's cores (plain threads: the process
// already hosts torch's OpenMP runtime, a second one is not linked in).
template <typename F>
void parallel_cols(int64_t w, int64_t rows, F f) {
  // one thread per >= 256K elements, at most 16 (thread start-up is ~20 us)
  const int64_t by_work = (w * rows) >> 18;
  const int64_t cap = g_host_threads;
  const int64_t nth =
      std::max<int64_t>(1, std::min<int64_t>({(int64_t)std::thread::hardware_concurrency(), cap, by_work, w}));
  if (nth == 1) {
    f(0, w);
    return;
  }
  std::vector<std::thread> th;
  const int64_t per = (w + nth - 1) / nth;
  for (int64_t t = 0; t < nth; ++t) {
    const int64_t a = t * per, b = std::min<int64_t>(w, a + per);
    if (a < b) th.emplace_back([=] { f(a, b); });
  }
  for (auto& x : th) x.join();
}

__global__ void add_counter_kernel(int32_t* p, int32_t v) { *p += v; }

// Fix records of a guard check are relative to the panel; make them global.
__global__ void offset_fixes_kernel(abft_fix_t* fixes, int cap, const int32_t* from, const int32_t* to, int64_t row0,
                                    int64_t col0, int64_t nb) {
  const int n0 = *from, n1 = min(*to, cap);
  for (int f = n0 + (int)threadIdx.x; f < n1; f += blockDim.x) {
    abft_fix_t& x = fixes[f];
    if (x.kind == ABFT_FIX_COLCHK) {
      x.gi += row0 / nb;
      x.gj += col0;
    } else if (x.kind == ABFT_FIX_ROWCHK) {
      x.gi += row0;
      x.gj += col0 / nb;
    } else {
      x.gi += row0;
      x.gj += col0;
    }
  }
}

// sum x, sum (i+1) x, sum |x| of one nb-element column segment: four
// interleaved partial sums per quantity (fixed order, so deterministic; nb is
// a power of two >= 32), added pairwise at the end.
template <typename T>
inline void col_sums(const T* x, int64_t nb, double& se, double& sw, double& sa) {
  double e[4] = {0, 0, 0, 0}, w[4] = {0, 0, 0, 0}, a[4] = {0, 0, 0, 0};
  for (int64_t i = 0; i < nb; i += 4)
    for (int q = 0; q < 4; ++q) {
      const double v = (double)x[i + q];
      e[q] += v;
      w[q] += (double)(i + q + 1) * v;
      a[q] += fabs(v);
    }
  se = (e[0] + e[1]) + (e[2] + e[3]);
  sw = (w[0] + w[1]) + (w[2] + w[3]);
  sa = (a[0] + a[1]) + (a[2] + a[3]);
}

// Host guard: G[2I + 2mt*j] = sum_i x, G[2I+1 + 2mt*j] = sum_i (i+1) x of
// every nb-row tile I of column j (column-major panel, ld = rows).
template <typename T>
void host_guard(const T* P, int64_t rows, int64_t nb, int64_t w, T* G) {
  const int64_t mt = rows / nb;
  parallel_cols(w, rows, [=](int64_t j0, int64_t j1) {
    for (int64_t j = j0; j < j1; ++j)
      for (int64_t I = 0; I < mt; ++I) {
        double se, sw, sa;
        col_sums(P + I * nb + j * rows, nb, se, sw, sa);
        G[2 * I + j * 2 * mt] = (T)se;
        G[2 * I + 1 + j * 2 * mt] = (T)sw;
      }
  });
}

struct ColResid {
  double de, dw, te;
  bool bad;
};

template <typename T>
ColResid col_resid(const T* x, int64_t nb, double ge, double gw, double gam) {
  double se, sw, sa;
  col_sums(x, nb, se, sw, sa);
  ColResid r;
  r.de = ge - se;
  r.dw = gw - sw;
  r.te = 2.0 * gam * sa;
  r.bad = !isfinite(r.de) || !isfinite(r.dw) || fabs(r.de) > r.te || fabs(r.dw) > (double)nb * r.te;
  return r;
}

// c-5: q = dw/de, j = rint(q) accepted iff finite, |q-j| <= 0.25, 1 <= j <= nb,
// |dw - j de| <= tw + j te.  Returns the 0-based row or -1.
int locate_ratio(double de, double dw, double te, double tw, int64_t nb) {
  if (!isfinite(de) || !isfinite(dw) || de == 0.0) return -1;
  const double q = dw / de;
  if (!isfinite(q)) return -1;
  const double j = rint(q);
  if (fabs(q - j) > 0.25 || j < 1.0 || j > (double)nb) return -1;
  if (!(fabs(dw - j * de) <= tw + j * te)) return -1;
  return (int)j - 1;
}

// Line 4 (host check of the received panel, in place) over the nb-row tiles
// [I0, I1).  Returns 1 if every flagged column was located and corrected, 0
// if the panel must be fetched again; accumulates flagged columns / fixed
// elements.
template <typename T>
int host_check(T* P, int64_t rows, int64_t nb, int64_t w, const T* G, int64_t I0, int64_t I1, int* flagged,
               int* fixed) {
  const int64_t mt = rows / nb;
  const double gam = (double)nb * Prec<T>::u / (1.0 - (double)nb * Prec<T>::u);
  std::vector<int> fl_c(w, 0), fx_c(w, 0), ok_c(w, 1);
  parallel_cols(w, (I1 - I0) * nb, [&](int64_t j0, int64_t j1) {
  for (int64_t j = j0; j < j1; ++j) {
    int& fl = fl_c[j];
    int& fx = fx_c[j];
    int& ok = ok_c[j];
    for (int64_t I = I0; I < I1; ++I) {
      T* x = P + I * nb + j * rows;
      const double ge = (double)G[2 * I + j * 2 * mt], gw = (double)G[2 * I + 1 + j * 2 * mt];
      ColResid r = col_resid(x, nb, ge, gw, gam);
      if (!r.bad) continue;
      ++fl;
      int i = locate_ratio(r.de, r.dw, r.te, (double)nb * r.te, nb);
      if (i < 0) {  // c-7 candidate: the unique non-finite element, else the largest |x|
        int nf = 0, inf_at = -1, big_at = -1;
        double big = -1.0;
        for (int64_t a = 0; a < nb; ++a) {
          const double v = (double)x[a];
          if (!isfinite(v)) {
            ++nf;
            inf_at = (int)a;
          } else if (fabs(v) > big) {
            big = fabs(v);
            big_at = (int)a;
          }
        }
        i = nf == 1 ? inf_at : big_at;
      }
      if (i < 0) {
        ok = 0;
        continue;
      }
      double rest = 0.0;  // c-4: x_i <- c_e - sum_{r != i} x_r
      for (int64_t a = 0; a < nb; ++a)
        if (a != i) rest += (double)x[a];
      const T before = x[i];
      x[i] = (T)(ge - rest);
      if (col_resid(x, nb, ge, gw, gam).bad) {
        x[i] = before;
        ok = 0;
        continue;
      }
      ++fx;
    }
  }
  });
  int ok = 1;
  for (int64_t j = 0; j < w; ++j) {
    *flagged += fl_c[j];
    *fixed += fx_c[j];
    ok &= ok_c[j];
  }
  return ok;
}

int lapack_info_potrf(ft_ctx* c, int dt, int n, void* a, int lda) {
  int info = 0;
  if (dt == ABFT_F64)
    ((potrf_d_t)c->lp[0])("L", &n, (double*)a, &lda, &info, 1);
  else
    ((potrf_s_t)c->lp[1])("L", &n, (float*)a, &lda, &info, 1);
  return info;
}

}  // namespace

template <typename T>
static int host_pd_t(Driver& d, int k, int kind, int64_t row0, int64_t col0, int64_t rows, int32_t* piv_dev,
                     T* tau_dev, int32_t* info_dev) {
  ft_ctx* c = d.c;
  cudaStream_t s = d.s;
  const abft_stream_t as = (abft_stream_t)s;
  const int64_t nb = d.nb, mt = rows / nb, es = sizeof(T);
  const bool ft = d.o->abft != 0;
  const auto t0 = std::chrono::steady_clock::now();
  // staging: panel | guard | tau | ipiv | counts | work
  int lwork = 0;
  if (kind == HOST_GEQRF) {
    int m = (int)rows, n = (int)nb, ld = (int)rows, q = -1, info = 0;
    T wq = 0;
    if (sizeof(T) == 8)
      ((geqrf_d_t)c->lp[4])(&m, &n, nullptr, &ld, nullptr, (double*)&wq, &q, &info);
    else
      ((geqrf_s_t)c->lp[5])(&m, &n, nullptr, &ld, nullptr, (float*)&wq, &q, &info);
    lwork = std::max<int>((int)wq, (int)nb);
  }
  const size_t off_guard = ((size_t)rows * nb * es + 255) / 256 * 256;
  const size_t off_tau = off_guard + ((size_t)2 * mt * nb * es + 255) / 256 * 256;
  const size_t off_piv = off_tau + ((size_t)nb * es + 255) / 256 * 256;
  const size_t off_cnt = off_piv + ((size_t)nb * 4 + 255) / 256 * 256;
  const size_t off_work = off_cnt + 256;
  const size_t need = off_work + (size_t)(lwork + 1) * es;
  if (c->hstage_bytes < need) {
    if (c->hstage) cudaFreeHost(c->hstage);
    c->hstage = nullptr;
    c->hstage_bytes = 0;
    if (cudaHostAlloc((void**)&c->hstage, need, cudaHostAllocDefault) != cudaSuccess) return ABFT_E_NOMEM;
    c->hstage_bytes = need;
  }
  FT_TRY(grow_buffer(c->dguard, c->dguard_bytes, (size_t)2 * mt * nb * es));
  T* hp = reinterpret_cast<T*>(c->hstage);
  T* hg = reinterpret_cast<T*>(c->hstage + off_guard);
  T* htau = reinterpret_cast<T*>(c->hstage + off_tau);
  int* hpiv = reinterpret_cast<int*>(c->hstage + off_piv);
  int32_t* hcnt = reinterpret_cast<int32_t*>(c->hstage + off_cnt);
  T* hwork = reinterpret_cast<T*>(c->hstage + off_work);
  T* panel = reinterpret_cast<T*>(d.a_at(row0, col0));

  abft_mat_t P{};
  P.dtype = d.dtype;
  P.m = rows;
  P.n = nb;
  P.nb = nb;
  P.A = panel;
  P.lda = d.lda;
  P.colchk = c->dguard;
  P.ldc = 2 * mt;
  abft_tiles_t all{0, (int)mt, 0, 1, 0, ABFT_GENERAL};
  auto faults = [&](int point) {
    std::vector<ft_inject_t> v;
    for (auto& u : d.xfer_used)
      if (u.first == k && u.second == point) return v;
    d.xfer_used.push_back({k, point});
    for (int t = 0; t < d.o->n_inject; ++t) {
      const ft_inject_t& f = d.o->inject[t];
      if (f.iter == k && f.point == point && f.target == 0) v.push_back(f);
    }
    return v;
  };

  // lines 3-4: guarded D2H + host check.  The panel comes over in up to
  // four tile-row chunks; the host checks each chunk as soon as it has
  // arrived, so the check overlaps the rest of the copy.
  if (ft) FT_TRY(abft_encode(&P, &all, ABFT_COL, as));
  const auto d2h_faults = faults(FT_AT_D2H);
  const int nch = ft ? (int)std::min<int64_t>(4, mt) : 1;
  for (int ch = 0; ch < nch; ++ch)
    if (!c->hchunk[ch]) ABFT_CUDA_TRY(cudaEventCreateWithFlags(&c->hchunk[ch], cudaEventDisableTiming));
  auto inject_d2h = [&](int64_t r0, int64_t r1) {  // faults in panel rows [r0, r1)
    for (auto& f : d2h_faults) {
      if (f.gi - row0 < r0 || f.gi - row0 >= r1) continue;
      T* e = hp + (f.gi - row0) + (f.gj - col0) * rows;
      if (sizeof(T) == 8) {
        uint64_t b;
        memcpy(&b, e, 8);
        b ^= f.xor_mask;
        memcpy(e, &b, 8);
      } else {
        uint32_t b;
        memcpy(&b, e, 4);
        b ^= (uint32_t)f.xor_mask;
        memcpy(e, &b, 4);
      }
    }
  };
  for (int attempt = 0; attempt < 3; ++attempt) {
    if (!ft) {
      ABFT_CUDA_TRY(cudaMemcpy2DAsync(hp, rows * es, panel, d.lda * es, rows * es, nb, cudaMemcpyDeviceToHost, s));
      ABFT_CUDA_TRY(cudaStreamSynchronize(s));
      if (attempt == 0) inject_d2h(0, rows);
      break;
    }
    ABFT_CUDA_TRY(cudaMemcpyAsync(hg, c->dguard, (size_t)2 * mt * nb * es, cudaMemcpyDeviceToHost, s));
    for (int ch = 0; ch < nch; ++ch) {
      const int64_t I0 = mt * ch / nch, I1 = mt * (ch + 1) / nch;
      ABFT_CUDA_TRY(cudaMemcpy2DAsync(hp + I0 * nb, rows * es, panel + I0 * nb, d.lda * es, (I1 - I0) * nb * es, nb,
                                      cudaMemcpyDeviceToHost, s));
      ABFT_CUDA_TRY(cudaEventRecord(c->hchunk[ch], s));
    }
    int ok = 1;
    for (int ch = 0; ch < nch; ++ch) {
      const int64_t I0 = mt * ch / nch, I1 = mt * (ch + 1) / nch;
      ABFT_CUDA_TRY(cudaEventSynchronize(c->hchunk[ch]));
      if (attempt == 0) inject_d2h(I0 * nb, I1 * nb);
      ok &= host_check<T>(hp, rows, nb, nb, hg, I0, I1, &d.xs[0], &d.xs[1]);
    }
    if (ok) break;
    if (attempt < 2) {
      ++d.xs[2];
    } else {
      ++d.xs[6];
      add_counter_kernel<<<1, 1, 0, s>>>(d.counts + ABFT_CNT_UNCORRECTABLE, 1);
    }
  }

  const auto t1 = std::chrono::steady_clock::now();
  // line 5: host PD
  int info = 0;
  {
    int m = (int)rows, n = (int)nb, ld = (int)rows;
    if (kind == HOST_POTRF) {
      info = lapack_info_potrf(c, d.dtype, n, hp, ld);
    } else if (kind == HOST_GETRF) {
      if (sizeof(T) == 8)
        ((getrf_d_t)c->lp[2])(&m, &n, (double*)hp, &ld, hpiv, &info);
      else
        ((getrf_s_t)c->lp[3])(&m, &n, (float*)hp, &ld, hpiv, &info);
    } else {
      if (sizeof(T) == 8)
        ((geqrf_d_t)c->lp[4])(&m, &n, (double*)hp, &ld, (double*)htau, (double*)hwork, &lwork, &info);
      else
        ((geqrf_s_t)c->lp[5])(&m, &n, (float*)hp, &ld, (float*)htau, (float*)hwork, &lwork, &info);
    }
  }
  hcnt[8] = info > 0 ? info : 0;
  auto t2 = std::chrono::steady_clock::now(), t3 = t2;

  // lines 6-7: guarded H2D + device check.  The panel goes out first and the
  // host encodes its guard while the DMA reads the same pinned buffer.
  const auto h2d_faults = faults(FT_AT_H2D);
  for (int attempt = 0; attempt < 3; ++attempt) {
    ABFT_CUDA_TRY(cudaMemcpy2DAsync(panel, d.lda * es, hp, rows * es, rows * es, nb, cudaMemcpyHostToDevice, s));
    if (attempt == 0) {
      ABFT_CUDA_TRY(cudaMemcpyAsync(info_dev, hcnt + 8, 4, cudaMemcpyHostToDevice, s));
      if (kind == HOST_GETRF) ABFT_CUDA_TRY(cudaMemcpyAsync(piv_dev, hpiv, nb * 4, cudaMemcpyHostToDevice, s));
      if (kind == HOST_GEQRF) ABFT_CUDA_TRY(cudaMemcpyAsync(tau_dev, htau, nb * es, cudaMemcpyHostToDevice, s));
      for (auto& f : h2d_faults) FT_TRY(d.inject_at_elem(f));
    }
    if (!ft) break;
    if (attempt == 0) {
      t2 = std::chrono::steady_clock::now();
      host_guard<T>(hp, rows, nb, nb, hg);
      t3 = std::chrono::steady_clock::now();
    }
    ABFT_CUDA_TRY(cudaMemcpyAsync(c->dguard, hg, (size_t)2 * mt * nb * es, cudaMemcpyHostToDevice, s));
    ABFT_CUDA_TRY(cudaMemsetAsync(d.xcounts, 0, 8 * sizeof(int32_t), s));
    ABFT_CUDA_TRY(cudaMemcpyAsync(d.mark2, d.nfix, sizeof(int32_t), cudaMemcpyDeviceToDevice, s));
    abft_tol_t tol{ABFT_TOL_POSTERIORI, 1.0, 0};
    abft_report_t R{d.status, d.nt, nullptr, nullptr, d.xcounts};
    FT_TRY(abft_check(&P, &all, ABFT_COL, &tol, &R, c->fixlog, c->fixcap, d.nfix, as));
    offset_fixes_kernel<<<1, 128, 0, s>>>(c->fixlog, c->fixcap, d.mark2, d.nfix, row0, col0, nb);
    ABFT_CUDA_TRY(cudaMemcpyAsync(hcnt, d.xcounts, 8 * sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    ABFT_CUDA_TRY(cudaStreamSynchronize(s));
    d.xs[3] += hcnt[ABFT_CNT_COLS_FLAGGED];
    d.xs[4] += hcnt[ABFT_CNT_ELEMS_FIXED];
    if (hcnt[ABFT_CNT_UNCORRECTABLE] == 0) break;
    if (attempt < 2) {
      ++d.xs[5];
    } else {
      ++d.xs[6];
      add_counter_kernel<<<1, 1, 0, s>>>(d.counts + ABFT_CNT_UNCORRECTABLE, 1);
    }
  }
  ABFT_CUDA_TRY(cudaGetLastError());
  const auto t4 = std::chrono::steady_clock::now();
  auto ms = [](std::chrono::steady_clock::time_point a, std::chrono::steady_clock::time_point b) {
    return std::chrono::duration<double, std::milli>(b - a).count();
  };
  d.ms_host += ms(t0, t4);
  d.host_phase[0] += ms(t0, t1);  // guard encode + D2H (+ waiting for the device) + host check
  d.host_phase[1] += ms(t1, t2);  // host LAPACK
  d.host_phase[2] += ms(t2, t3);  // host guard
  d.host_phase[3] += ms(t3, t4);  // H2D + device check + read-back
  return 0;
}

int host_panel_pd(Driver& d, int k, int kind, int64_t row0, int64_t col0, int64_t rows, int32_t* piv_dev,
                  void* tau_dev, int32_t* info_dev) {
  if (!d.c->lapack) return ABFT_E_UNSUPPORTED;
  return d.dtype == ABFT_F64
             ? host_pd_t<double>(d, k, kind, row0, col0, rows, piv_dev, (double*)tau_dev, info_dev)
             : host_pd_t<float>(d, k, kind, row0, col0, rows, piv_dev, (float*)tau_dev, info_dev);
}

}  // namespace abft

extern "C" int ft_ctx_set_host_lapack(ft_ctx_t* c, const char* path) {
  if (!c) return -1;
  if (!path) return -2;
  void* h = dlopen(path, RTLD_NOW | RTLD_LOCAL);
  if (!h) {
    fprintf(stderr, "[abft] dlopen(%s): %s\n", path, dlerror());
    return ABFT_E_UNSUPPORTED;
  }
  static const char* names[6] = {"dpotrf_", "spotrf_", "dgetrf_", "sgetrf_", "dgeqrf_", "sgeqrf_"};
  void* f[6];
  for (int i = 0; i < 6; ++i) {
    std::string scipy = std::string("scipy_") + names[i];
    f[i] = dlsym(h, scipy.c_str());
    if (!f[i]) f[i] = dlsym(h, names[i]);
    if (!f[i]) {
      fprintf(stderr, "[abft] %s: no %s\n", path, names[i]);
      dlclose(h);
      return ABFT_E_UNSUPPORTED;
    }
  }
  // split the cores between OpenBLAS and the guard loops (see g_host_threads)
  cpu_set_t cs;
  int cores = 16;
  if (sched_getaffinity(0, sizeof(cs), &cs) == 0) cores = CPU_COUNT(&cs);
  const int half = cores > 1 ? cores / 2 : 1;
  typedef void (*set_threads_t)(int);
  set_threads_t st = (set_threads_t)dlsym(h, "scipy_openblas_set_num_threads");
  if (!st) st = (set_threads_t)dlsym(h, "openblas_set_num_threads");
  if (st) st(half);
  abft::g_host_threads = st ? std::max(1, cores - half) : std::max(1, cores);
  if (getenv("ABFT_HOST_THREADS")) abft::g_host_threads = atoi(getenv("ABFT_HOST_THREADS"));
  if (c->lapack) dlclose(c->lapack);
  c->lapack = h;
  for (int i = 0; i < 6; ++i) c->lp[i] = f[i];
  return 0;
}
