// Shared plumbing of the fault-tolerant drivers (ft_potrf, ft_getrf):
// context buffers, the checksum state of the matrix, Alg. 2 check helper,
// fault-injection hooks (reading c-8) and the final statistics read-back.
#pragma once
#include <cublas_v2.h>
#include <cusolverDn.h>

#include <algorithm>
#include <chrono>
#include <cstring>
#include <mutex>
#include <string>
#include <initializer_list>
#include <tuple>
#include <vector>

#include "abft_common.cuh"

namespace abft {
cublasHandle_t blas_handle(cudaStream_t s, std::unique_lock<std::mutex>& lk);
cusolverDnHandle_t solver_handle(cudaStream_t s, std::unique_lock<std::mutex>& lk);
int scratch(cudaStream_t s, int slot, size_t bytes, void** out);
}  // namespace abft

#define FT_TRY(expr)     \
  do {                   \
    int _rc = (expr);    \
    if (_rc) return _rc; \
  } while (0)

struct ft_ctx {
  int device = 0;
  cudaStream_t stream = nullptr;
  void* state = nullptr;  // colchk | rowchk | colmag | rowmag
  size_t state_bytes = 0;
  int32_t* ints = nullptr;  // status | counts[8] | n_fixes | mark | info | rep[2] | info_total | spare
  size_t ints_n = 0;
  abft_fix_t* fixlog = nullptr;
  int fixcap = 0;
  void* linv = nullptr;  // nb x nb inverse of the current L_kk
  size_t linv_bytes = 0;
  void* uinv = nullptr;  // nb x nb inverse of the current U_kk (LU)
  size_t uinv_bytes = 0;
  void* putmp = nullptr;  // n x nb panel scratch (GEMM-based PU, LU panel copy)
  size_t putmp_bytes = 0;
  void* aux = nullptr;  // driver-specific device scratch (LU pivots / swap rows)
  size_t aux_bytes = 0;
  void* rsv = nullptr;  // local-restart copies (f1): PD tile + PU panel with checksums
  size_t rsv_bytes = 0;
  int32_t* hpin = nullptr;  // pinned host words (read-backs), mapped into the device address space
  int32_t* hpin_dev = nullptr;  // device alias of hpin (a kernel writes read-back words straight to the host)
  cudaEvent_t ev = nullptr;  // marks the PD-check read-back (restart decision)
  // The drivers run on a private non-blocking stream joined to `stream` at
  // entry and exit (the look-ahead's side and rule streams fork from and join
  // back into it; library handles and scratch are per stream).
  cudaStream_t drv = nullptr;
  cudaEvent_t join = nullptr;
  // look-ahead (the next panel's PD / PU next to the current TMU): a second
  // private stream (high priority) and its events
  cudaStream_t side = nullptr;
  cudaEvent_t ev_col = nullptr, ev_side = nullptr;
  // ft_potrf look-ahead: the TMU checksum rule of the trailing rest on its own
  // stream, next to the DSYRK it does not depend on (ft_opts_t.rule_stream)
  cudaStream_t rule = nullptr;
  cudaEvent_t ev_rule = nullptr;
  void* putmp2 = nullptr;  // PU scratch of the side stream
  size_t putmp2_bytes = 0;
  std::vector<cudaEvent_t> evpool;  // opts->timing: per-phase span events (reused across calls)
  // FT_PD_HOST (ft_host.cu): host LAPACK, pinned panel staging, device guard
  void* lapack = nullptr;  // dlopen handle
  void* lp[6] = {};        // dpotrf spotrf dgetrf sgetrf dgeqrf sgeqrf
  char* hstage = nullptr;  // pinned: panel | guard | tau | ipiv | counts | work
  size_t hstage_bytes = 0;
  void* dguard = nullptr;  // device transfer guard
  size_t dguard_bytes = 0;
  cudaEvent_t hchunk[4] = {};  // D2H chunk arrivals (the host checks a chunk while the next is in flight)
};

namespace abft {

inline int grow_buffer(void*& p, size_t& have, size_t need) {
  if (have >= need) return 0;
  if (p) cudaFree(p);
  p = nullptr;
  have = 0;
  if (cudaMalloc(&p, need) != cudaSuccess) return ABFT_E_NOMEM;
  have = need;
  return 0;
}

// LAPACK info of the whole factorization: first failing panel's local value
// offset by the panel origin.
static __global__ void drv_add_i32_kernel(int32_t* p, int32_t v) { *p += v; }

// Restart read-back (f1): the uncorrectable errors a check added, written to
// mapped host memory by one thread (replaces two device-to-host copies on
// the stream's critical path).
static __global__ void drv_delta_to_host_kernel(const int32_t* now, const int32_t* snap, volatile int32_t* host) {
  *host = *now - *snap;
}
static __global__ void drv_word_to_host_kernel(const int32_t* src, volatile int32_t* host) { *host = *src; }

// Device-decided local restart (f1, L430): did the post-op check add
// uncorrectable errors?  Then take them back (the redo re-checks), count the
// restart and the redo's checks, and open the gate of the redo's launches.
static __global__ void drv_restart_gate_kernel(int32_t* uncorrectable, const int32_t* snap, int32_t* gate,
                                               int32_t* restarts, int32_t* runs, int32_t nchk) {
  const int32_t delta = *uncorrectable - *snap;
  *gate = delta > 0;
  if (delta > 0) {
    *uncorrectable = *snap;
    atomicAdd(restarts, 1);  // shared with the other stream's gate kernels (look-ahead)
    atomicAdd(runs, nchk);
  }
}

// Fig. 4b gate: did the fixes logged since the start of the iteration include
// a 1D pattern (class 1D_ROW / 1D_COL)?  Counts the gated checks that run.
static __global__ void fig4b_gate_kernel(const abft_fix_t* fixes, int cap, const int32_t* from, const int32_t* to,
                                         int32_t* gate, int32_t* runs) {
  const int n0 = *from, n1 = min(*to, cap);
  int hit = 0;
  for (int f = n0 + (int)threadIdx.x; f < n1; f += blockDim.x)
    hit |= fixes[f].kind == ABFT_FIX_DATA && (fixes[f].cls == ABFT_CLS_1D_ROW || fixes[f].cls == ABFT_CLS_1D_COL);
  hit = __any_sync(0xffffffffu, hit);
  if (threadIdx.x == 0) {
    *gate = hit;
    if (hit) atomicAdd(runs, 1);
  }
}

static __global__ void accum_info_kernel(int32_t* tile_info, int32_t* total, int64_t offset) {
  if (*tile_info != 0 && *total == 0) *total = (int32_t)(*tile_info + offset);
  *tile_info = 0;
}

struct Driver {
  ft_ctx* c = nullptr;
  cudaStream_t s = nullptr;
  int32_t dtype = ABFT_F64;
  int64_t n = 0, nb = 0, nt = 0, lda = 0;
  size_t es = 8;
  void* A = nullptr;
  const ft_opts_t* o = nullptr;
  bool lu = false;
  bool qr = false;
  abft_mat_t M{};
  abft_report_t R{};
  abft_tol_t tol{};
  int32_t *status = nullptr, *counts = nullptr, *nfix = nullptr, *mark = nullptr, *info = nullptr, *rep = nullptr,
          *info_total = nullptr, *snap = nullptr;
  int restarts = 0;
  std::vector<ft_inject_t> onchip_pending;
  int n_checks = 0;
  // FT_PD_HOST bookkeeping (ft_host.cu)
  int32_t* xcounts = nullptr;          // device int32[8]: counts of one H2D guard check
  int32_t* mark2 = nullptr;            // device: fix-log position before an H2D guard check
  int xs[7] = {};                      // ft_stats_t.xfer_* accumulators
  double ms_host = 0.0;
  double host_phase[4] = {};           // ABFT_HOST_TIMING=1: per-phase host ms (stderr at the end)
  int32_t* ctf_cnt = nullptr;          // device: flagged entries of one CTF check (QR, f2)
  int32_t* gate4b = nullptr;           // device: Fig. 4b gate of this iteration
  int32_t* gated_runs = nullptr;       // device: gated checks that ran
  int32_t* iter_mark = nullptr;        // device: fix-log position at the start of the iteration
  int32_t* gate_rs = nullptr;          // device: gate of the device-decided restart's redo
  int32_t* restarts_dev = nullptr;     // device: restarts decided on the device
  int32_t* f4b_end = nullptr;          // device: fix-log position where a deferred Fig. 4b gate stops
  // Look-ahead (reading c-35): the next panel's PD / PU run on the context's
  // side stream with their own report counters (so that a restart decision
  // there never sees the main stream's checks); on_side() switches both.
  cudaStream_t s_main = nullptr;
  int32_t *counts_main = nullptr, *counts_side = nullptr;
  void on_side(bool side) {
    s = side ? c->side : s_main;
    counts = side ? counts_side : counts_main;
    R.counts = counts;
  }
  int side_setup() {
    if (c->side) return 0;
    int lo = 0, hi = 0;
    ABFT_CUDA_TRY(cudaDeviceGetStreamPriorityRange(&lo, &hi));
    // high priority: at the default priority the whole chain waits behind the
    // DSYRK and look-ahead is lost (measured: plain 295 -> 310 ms at n=30720)
    ABFT_CUDA_TRY(cudaStreamCreateWithPriority(&c->side, cudaStreamNonBlocking, hi));
    ABFT_CUDA_TRY(cudaEventCreateWithFlags(&c->ev_col, cudaEventDisableTiming));
    ABFT_CUDA_TRY(cudaEventCreateWithFlags(&c->ev_side, cudaEventDisableTiming));
    return 0;
  }
  int rule_setup() {
    if (c->rule) return 0;
    ABFT_CUDA_TRY(cudaStreamCreateWithFlags(&c->rule, cudaStreamNonBlocking));
    ABFT_CUDA_TRY(cudaEventCreateWithFlags(&c->ev_rule, cudaEventDisableTiming));
    return 0;
  }
  int ctf_flagged = 0, ctf_recomputed = 0;
  std::vector<std::pair<int, int>> xfer_used;  // (iter, point) transfer faults already applied

  // opts->timing: spans (phase, start, end) recorded on the stream each phase runs on
  struct Span {
    int ph;
    cudaEvent_t a, b;
  };
  std::vector<Span> spans;
  // ABFT_ITER_EVENTS=1 (diagnostics): an event on the main stream at each
  // iteration start; per-iteration ms printed to stderr by finish()
  std::vector<cudaEvent_t> iter_ev;
  void iter_event() {
    static const bool on = getenv("ABFT_ITER_EVENTS") != nullptr;
    if (!on) return;
    cudaEvent_t e = ev_take();
    if (e && cudaEventRecord(e, s_main) == cudaSuccess) iter_ev.push_back(e);
  }
  size_t ev_used = 0;
  cudaEvent_t ev_take() {
    if (ev_used == c->evpool.size()) {
      cudaEvent_t e = nullptr;
      if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
      c->evpool.push_back(e);
    }
    return c->evpool[ev_used++];
  }

  Driver() = default;
  Driver(const Driver&) = delete;
  Driver& operator=(const Driver&) = delete;
  // Every exit (error returns included) orders the caller's stream after the
  // work queued on the private one.
  ~Driver() {
    if (c && c->drv && s == c->drv && cudaEventRecord(c->join, s) == cudaSuccess)
      cudaStreamWaitEvent(c->stream, c->join, 0);
  }

  int setup(ft_ctx* ctx, int32_t dt, int64_t n_, int64_t nb_, void* dA, int64_t lda_, const ft_opts_t* opts,
            bool is_lu) {
    c = ctx;
    if (!c->drv) {
      ABFT_CUDA_TRY(cudaStreamCreateWithFlags(&c->drv, cudaStreamNonBlocking));
      ABFT_CUDA_TRY(cudaEventCreateWithFlags(&c->join, cudaEventDisableTiming));
    }
    ABFT_CUDA_TRY(cudaEventRecord(c->join, c->stream));
    ABFT_CUDA_TRY(cudaStreamWaitEvent(c->drv, c->join, 0));
    s = c->drv;
    dtype = dt;
    n = n_;
    nb = nb_;
    nt = n_ / nb_;
    lda = lda_;
    es = dt == ABFT_F64 ? 8 : 4;
    A = dA;
    o = opts;
    lu = is_lu;
    const bool ft = o->abft != 0;
    size_t need = ft ? (size_t)(2 * nt * n + n * 2 * nt + nt * n + n * nt) * es : 0;
    FT_TRY(grow_buffer(c->state, c->state_bytes, need));
    if (o->pd_location == FT_PD_HOST && !c->lapack) return ABFT_E_UNSUPPORTED;
    if (o->pd_location != FT_PD_DEVICE && o->pd_location != FT_PD_HOST) return ABFT_E_UNSUPPORTED;
    size_t ints_need = (size_t)nt * nt + 48;  // status | counts[32] | side counts[8] | spare
    void* ip = c->ints;
    FT_TRY(grow_buffer(ip, c->ints_n, ints_need * sizeof(int32_t)));
    c->ints = reinterpret_cast<int32_t*>(ip);
    FT_TRY(grow_buffer(c->linv, c->linv_bytes, (size_t)nb * nb * es));
    if (lu) FT_TRY(grow_buffer(c->uinv, c->uinv_bytes, (size_t)nb * nb * es));
    if (o->pu_gemm || lu) FT_TRY(grow_buffer(c->putmp, c->putmp_bytes, (size_t)n * nb * es));
    status = c->ints;
    counts = status + nt * nt;
    nfix = counts + 8;
    mark = nfix + 1;
    info = mark + 1;
    rep = info + 1;
    info_total = rep + 2;
    snap = info_total + 1;
    mark2 = snap + 1;
    xcounts = counts + 16;
    ctf_cnt = counts + 24;
    gate4b = counts + 25;
    gated_runs = counts + 26;
    iter_mark = counts + 27;
    gate_rs = counts + 29;
    restarts_dev = counts + 28;
    f4b_end = counts + 30;
    counts_main = counts;
    counts_side = counts + 32;
    s_main = s;
    if (o->abft && o->restart)
      FT_TRY(grow_buffer(c->rsv, c->rsv_bytes,
                         ((size_t)n * nb + (size_t)nb * nb + 3 * (size_t)nt * nb + 4 * nb + 3 * (size_t)n) * es));
    ABFT_CUDA_TRY(cudaMemsetAsync(c->ints, 0, ints_need * sizeof(int32_t), s));
    char* st = (char*)c->state;
    M.dtype = dtype;
    M.m = n;
    M.n = n;
    M.nb = nb;
    M.A = dA;
    M.lda = lda;
    if (ft) {
      M.colchk = st;
      M.ldc = 2 * nt;
      st += 2 * nt * n * es;
      M.rowchk = st;
      M.ldr = n;
      st += n * 2 * nt * es;
      M.colmag = st;
      M.ldcm = nt;
      st += nt * n * es;
      M.rowmag = st;
      M.ldrm = n;
    }
    R.status = status;
    R.ld_status = nt;
    R.counts = counts;
    tol.kind = o->tol_kind;
    tol.scale = o->tol_scale > 0 ? o->tol_scale : 1.0;
    tol.refresh = o->refresh;
    return 0;
  }

  char* elem(int target, int64_t gi, int64_t gj) {
    if (target == 1) return (char*)M.colchk + (gi + gj * M.ldc) * es;
    if (target == 2) return (char*)M.rowchk + (gi + gj * M.ldr) * es;
    if (target == 3) return (char*)c->linv + (gi + gj * nb) * es;  // ft_geqrf: the CTF T (nb x nb)
    return (char*)A + (gi + gj * lda) * es;
  }
  // Elements the op after `point` overwrites: an on-chip flip there cannot be
  // changed back, so it stays (reading c-8).
  bool in_update_region(int point, int k, int64_t gi, int64_t gj) const {
    const int64_t r0 = k * nb, r1 = (k + 1) * nb;
    if (!lu) {
      if (point == FT_AT_PRE_PD) return gi >= r0 && gi < r1 && gj >= r0 && gj < r1;
      if (point == FT_AT_PRE_PU) return gi >= r1 && gj >= r0 && gj < r1;
    } else {
      if (point == FT_AT_PRE_PD) return gi >= r0 && gj >= r0 && gj < r1;
      if (point == FT_AT_PRE_PU) return gi >= r0 && gi < r1 && gj >= r1;
    }
    if (point == FT_AT_PRE_TMU) return gi >= (qr ? r0 : r1) && gj >= r1;
    return false;
  }
  int inject_at(int k, int point) {
    for (int t = 0; t < o->n_inject; ++t) {
      const ft_inject_t& f = o->inject[t];
      if (f.iter != k || f.point != point) continue;
      FT_TRY(abft_inject(elem(f.target, f.gi, f.gj), dtype, 0, f.xor_mask, (abft_stream_t)s));
      bool op_point = point == FT_AT_PRE_PD || point == FT_AT_PRE_PU || point == FT_AT_PRE_TMU;
      if (f.kind == FT_KIND_ONCHIP && op_point && f.target == 0 && !in_update_region(point, k, f.gi, f.gj))
        onchip_pending.push_back(f);
    }
    return 0;
  }
  bool has_inject(int k, int point) const {
    for (int t = 0; t < o->n_inject; ++t)
      if (o->inject[t].iter == k && o->inject[t].point == point) return true;
    return false;
  }
  // Fault-injection runs only: does the plan touch the diagonal tile between
  // the PD (which produced the inverse the GEMM-based PU reads) and the PU?
  // Then the PU must see the flipped tile, as an in-place TRSM would (c-8).
  bool diag_touched_before_pu(int k) const {
    for (int t = 0; t < o->n_inject; ++t) {
      const ft_inject_t& f = o->inject[t];
      if (f.iter != k || f.target != 0) continue;
      if (f.point != FT_AT_PRE_PU_CHECK && f.point != FT_AT_PRE_PU) continue;
      if (f.gi >= k * nb && f.gi < (k + 1) * nb && f.gj >= k * nb && f.gj < (k + 1) * nb) return true;
    }
    return false;
  }
  int inject_at_elem(const ft_inject_t& f) {  // one planned flip, now (transfer hooks)
    return abft_inject(elem(f.target, f.gi, f.gj), dtype, 0, f.xor_mask, (abft_stream_t)s);
  }
  int restore_onchip() {  // after the op's data step: undo on-chip flips (the stored value was never wrong)
    for (auto& f : onchip_pending)
      FT_TRY(abft_inject(elem(f.target, f.gi, f.gj), dtype, 0, f.xor_mask, (abft_stream_t)s));
    onchip_pending.clear();
    return 0;
  }
  // ckpt (nullable): also leave a copy of the checked range's data, as
  // corrected by the check, at ckpt (ld ldk) — the local-restart copy of the
  // next op's input (f1), written by the check's own pass when it can be
  int check(int I0, int I1, int J0, int J1, int view, int which, bool lower_only = false,
            cudaStream_t on = nullptr, void* ckpt = nullptr, int64_t ldk = 0);
  // ABFT_DIAG_SKIP (timing diagnostics only; results are then unprotected):
  // bit 0 skips the checks issued on the main stream, bit 1 those on the
  // look-ahead side stream, bit 2 the TMU checksum rule, bit 3 the PD / PU rules
  static int diag_skip() {
    static const int v = getenv("ABFT_DIAG_SKIP") ? atoi(getenv("ABFT_DIAG_SKIP")) : 0;
    return v;
  }
  int check_impl(int I0, int I1, int J0, int J1, int view, int which, bool lower_only, cudaStream_t on, void* ckpt,
                 int64_t ldk) {
    abft_tiles_t t{I0, I1, J0, J1, lower_only ? 1 : 0, view};
    const abft_stream_t st = (abft_stream_t)(on ? on : s);
    auto plain_copy = [&]() -> int {
      if (!ckpt) return 0;
      return abft::copy2d(ckpt, ldk * es, a_at((int64_t)I0 * nb, (int64_t)J0 * nb), lda * es,
                          (size_t)(I1 - I0) * nb * es, (size_t)(J1 - J0) * nb, (cudaStream_t)st);
    };
    if (diag_skip() & (s == s_main && !on ? 1 : 2)) return plain_copy();
    if (o->checksum_gemm) {  // prior-art GEMM recalculation (f3 baseline)
      FT_TRY(abft_verify_gemm(&M, &t, which, &tol, &R, st));
      FT_TRY(abft_locate_correct(&M, &t, which, &tol, &R, c->fixlog, c->fixcap, nfix, st));
      FT_TRY(plain_copy());
    } else if (ckpt) {  // verify + locate + checkpoint in one pass
      FT_TRY(check_ckpt(&M, &t, which, &tol, &R, c->fixlog, c->fixcap, nfix, ckpt, ldk, (cudaStream_t)st));
    } else {  // verify + locate in one launch
      FT_TRY(abft_check(&M, &t, which, &tol, &R, c->fixlog, c->fixcap, nfix, st));
    }
    ++n_checks;
    return 0;
  }
  // Local restart (f1, L430) bookkeeping: snapshot the uncorrectable counter
  // before a post-op check, read back how many 2D errors that check added
  // (one host wait), and take them back when the op is redone.
  int snap_uncorrectable() {
    ABFT_CUDA_TRY(cudaMemcpyAsync(snap, counts + ABFT_CNT_UNCORRECTABLE, 4, cudaMemcpyDeviceToDevice, s));
    return 0;
  }
  int post_delta(int slot) {  // queue the read-back of the check just issued into hpin[slot]
    drv_delta_to_host_kernel<<<1, 1, 0, s>>>(counts + ABFT_CNT_UNCORRECTABLE, snap, c->hpin_dev + slot);
    ABFT_CUDA_TRY(cudaGetLastError());
    ABFT_CUDA_TRY(cudaEventRecord(c->ev, s));
    return 0;
  }
  int post_word(const int32_t* src, int slot) {  // queue the read-back of one device word into hpin[slot]
    drv_word_to_host_kernel<<<1, 1, 0, s>>>(src, c->hpin_dev + slot);
    ABFT_CUDA_TRY(cudaGetLastError());
    ABFT_CUDA_TRY(cudaEventRecord(c->ev, s));
    return 0;
  }
  int32_t host_word(int slot) const { return ((volatile int32_t*)c->hpin)[slot]; }
  int wait_delta(int slot, int* delta) {
    ABFT_CUDA_TRY(cudaEventSynchronize(c->ev));
    *delta = ((volatile int32_t*)c->hpin)[slot];
    return 0;
  }
  int uncorrectable_added(int* delta) {
    FT_TRY(post_delta(0));
    return wait_delta(0, delta);
  }
  // The same decision without a host wait (the PU restarts): `redo` queues
  // the restore / redo / re-check as gated launches (copy2d, gemm_gated,
  // verify and locate all return at once while the gate is closed) after
  // drv_restart_gate_kernel has compared the counter with the snapshot.  The
  // redo's `nchk` checks and the restart are counted on the device
  // (counts[26], counts[28]) when the gate opens.
  template <typename F>
  int gated_restart(int nchk, F&& redo) {
    drv_restart_gate_kernel<<<1, 1, 0, s>>>(counts + ABFT_CNT_UNCORRECTABLE, snap, gate_rs, restarts_dev, gated_runs,
                                            nchk);
    ABFT_CUDA_TRY(cudaGetLastError());
    GateScope g(gate_rs);
    const int c0 = n_checks;
    FT_TRY(redo(gate_rs));
    n_checks = c0;  // counted on the device when the redo runs
    return 0;
  }
  int take_back_uncorrectable(int delta) {
    ++restarts;
    drv_add_i32_kernel<<<1, 1, 0, s>>>(counts + ABFT_CNT_UNCORRECTABLE, -delta);
    ABFT_CUDA_TRY(cudaGetLastError());
    return 0;
  }
  // 2-D copy of rows x cols elements between column-major arrays (SM kernel)
  int copy(void* dst, int64_t ldd, const void* src, int64_t lds, int64_t rows, int64_t cols) {
    if (rows <= 0 || cols <= 0) return 0;
    return abft::copy2d(dst, ldd * es, src, lds * es, rows * es, cols, s);
  }
  // up to 6 such copies as one launch: (dst, ldd, src, lds, rows, cols) in elements
  using CopySpec = std::tuple<void*, int64_t, const void*, int64_t, int64_t, int64_t>;
  int copies(std::initializer_list<CopySpec> l) {
    Copy2D cs[6];
    int n = 0;
    for (const CopySpec& t : l) {
      if (n == 6) return ABFT_E_UNSUPPORTED;
      cs[n++] = Copy2D{std::get<0>(t), (size_t)std::get<1>(t) * es, std::get<2>(t), (size_t)std::get<3>(t) * es,
                       (size_t)std::get<4>(t) * es, (size_t)std::get<5>(t)};
    }
    return copy2d_multi(cs, n, s);
  }
  // f1 hooks: the fix-log position at the start of iteration k; the Fig. 4b
  // check (gated on a 1D fix since then); the periodic trailing check.
  int begin_iteration() {
    ABFT_CUDA_TRY(cudaMemcpyAsync(iter_mark, nfix, 4, cudaMemcpyDeviceToDevice, s));
    return 0;
  }
  // mark_fig4b_end: under look-ahead the Fig. 4b check of an iteration runs
  // after its PU (on the main stream); the gate must then see only the fixes
  // up to where Alg. 2 puts the check (before the PU), recorded here.
  int mark_fig4b_end() {
    ABFT_CUDA_TRY(cudaMemcpyAsync(f4b_end, nfix, 4, cudaMemcpyDeviceToDevice, s));
    return 0;
  }
  int fig4b_check(int I0, int I1, int J0, int J1, int view, int which, bool lower_only, bool deferred = false) {
    if (!o->fig4b || o->checksum_gemm || I0 >= I1) return 0;  // GEMMs cannot honour the device gate
    fig4b_gate_kernel<<<1, 32, 0, s>>>(c->fixlog, c->fixcap, iter_mark, deferred ? f4b_end : nfix, gate4b,
                                       gated_runs);
    ABFT_CUDA_TRY(cudaGetLastError());
    GateScope g(gate4b);
    FT_TRY(check(I0, I1, J0, J1, view, which, lower_only));
    --n_checks;  // counted on the device when it runs
    return 0;
  }
  int periodic_check(int k, int I0, int I1, int J0, int J1, int view, bool lower_only) {
    const int P = o->trailing_check_period;
    if (P <= 0 || (k + 1) % P != 0 || I0 >= I1) return 0;
    return check(I0, I1, J0, J1, view, ABFT_BOTH, lower_only);
  }
  void* colchk_at(int64_t r, int64_t col) { return (char*)M.colchk + (r + col * M.ldc) * es; }
  void* colmag_at(int64_t r, int64_t col) { return (char*)M.colmag + (r + col * M.ldcm) * es; }
  void* rowchk_at(int64_t r, int64_t col) { return (char*)M.rowchk + (r + col * M.ldr) * es; }
  void* rowmag_at(int64_t r, int64_t col) { return (char*)M.rowmag + (r + col * M.ldrm) * es; }
  void* a_at(int64_t r, int64_t col) { return (char*)A + (r + col * lda) * es; }

  // The single host synchronisation: counters, info and the fix log.
  int finish(std::chrono::steady_clock::time_point t0, ft_stats_t* stats, int64_t* info_out) {
    int32_t h[40];
    ABFT_CUDA_TRY(cudaMemcpyAsync(h, counts_main, sizeof(h), cudaMemcpyDeviceToHost, s));
    if (o->fix_log && o->fix_log_cap > 0)
      ABFT_CUDA_TRY(cudaMemcpyAsync(o->fix_log, c->fixlog, sizeof(abft_fix_t) * std::min(o->fix_log_cap, c->fixcap),
                                    cudaMemcpyDeviceToDevice, s));
    ABFT_CUDA_TRY(cudaEventRecord(c->join, s));
    ABFT_CUDA_TRY(cudaStreamWaitEvent(c->stream, c->join, 0));
    ABFT_CUDA_TRY(cudaStreamSynchronize(s));
    auto t1 = std::chrono::steady_clock::now();
    if (iter_ev.size() > 1) {
      fprintf(stderr, "[abft] iteration ms:");
      for (size_t i = 1; i < iter_ev.size(); ++i) {
        float ms = 0.f;
        cudaEventElapsedTime(&ms, iter_ev[i - 1], iter_ev[i]);
        fprintf(stderr, " %.3f", ms);
      }
      fprintf(stderr, "\n");
    }
    // layout after counts: nfix(8) mark(9) info(10) rep(11,12) info_total(13); side counts at 32
    for (int i = 0; i < 8; ++i) h[i] += h[32 + i];
    if (info_out) *info_out = h[13];
    if (stats) {
      for (int i = 0; i < 8; ++i) stats->counts[i] = h[i];
      stats->n_fixes = h[8];
      stats->repairs_applied = h[11];
      stats->repairs_skipped = h[12];
      stats->uncorrectable = h[ABFT_CNT_UNCORRECTABLE];
      stats->n_checks = n_checks + h[26];
      stats->restarts = restarts + h[28];
      stats->ms_total = std::chrono::duration<double, std::milli>(t1 - t0).count();
      int32_t* x = &stats->xfer_d2h_flagged;
      for (int i = 0; i < 7; ++i) x[i] = xs[i];
      stats->ms_host_pd = ms_host;
      if (ms_host > 0 && getenv("ABFT_HOST_TIMING"))
        fprintf(stderr, "[abft] host PD ms: d2h+check %.1f lapack %.1f guard %.1f h2d+check %.1f\n", host_phase[0],
                host_phase[1], host_phase[2], host_phase[3]);
      stats->ctf_flagged = ctf_flagged;
      stats->ctf_recomputed = ctf_recomputed;
      // outcomes by class from the fix log
      stats->detected = h[ABFT_CNT_TILES_FLAGGED];
      stats->corrected_0d = stats->corrected_1d = stats->checksum_repaired = 0;
      const int nf = std::min(h[8], c->fixcap);
      if (nf > 0) {
        std::vector<abft_fix_t> fx(nf);
        ABFT_CUDA_TRY(cudaMemcpy(fx.data(), c->fixlog, sizeof(abft_fix_t) * nf, cudaMemcpyDeviceToHost));
        for (const abft_fix_t& f : fx) {
          if (f.kind != ABFT_FIX_DATA)
            ++stats->checksum_repaired;
          else if (f.cls == ABFT_CLS_0D)
            ++stats->corrected_0d;
          else
            ++stats->corrected_1d;
        }
      }
      stats->comm_errors = xs[1] + xs[2] + xs[4] + xs[5];  // d2h fixed, retransfers, h2d fixed, resends
      for (int i = 0; i < FT_NPHASE; ++i) stats->ms_phase[i] = 0.0;
      for (const Span& sp : spans) {
        float ms = 0.f;
        if (cudaEventElapsedTime(&ms, sp.a, sp.b) == cudaSuccess) stats->ms_phase[sp.ph] += ms;
      }
    }
    return h[ABFT_CNT_UNCORRECTABLE] ? ABFT_E_UNCORRECTABLE : 0;
  }
};

// opts->timing: one span of phase `ph` on the driver's current stream
// (start recorded now, end when the scope closes).  Scopes do not nest.
struct PhaseScope {
  Driver& d;
  cudaEvent_t b = nullptr;
  cudaStream_t st = nullptr;
  PhaseScope(Driver& dd, int ph) : d(dd) {
    if (!dd.o->timing) return;
    st = dd.s;
    cudaEvent_t a = dd.ev_take();
    b = dd.ev_take();
    if (!a || !b || cudaEventRecord(a, st) != cudaSuccess) {
      b = nullptr;
      return;
    }
    dd.spans.push_back({ph, a, b});
  }
  ~PhaseScope() {
    if (b) cudaEventRecord(b, st);
  }
};

inline int Driver::check(int I0, int I1, int J0, int J1, int view, int which, bool lower_only, cudaStream_t on,
                          void* ckpt, int64_t ldk) {
  PhaseScope ps(*this, FT_PH_CHECKS);
  return check_impl(I0, I1, J0, J1, view, which, lower_only, on, ckpt, ldk);
}

// FT_PD_HOST (ft_host.cu): Alg. 2 lines 3-7 for the panel of iteration k,
// rows x nb at (row0, col0) of A: guarded D2H, host check, host LAPACK
// factorization (kind), guarded H2D, device check.  Writes the LAPACK info to
// info_dev (device int32), the 1-based local pivots to piv_dev (GETRF) and
// tau to tau_dev (GEQRF).
enum { HOST_POTRF = 0, HOST_GETRF = 1, HOST_GEQRF = 2 };
int host_panel_pd(Driver& d, int k, int kind, int64_t row0, int64_t col0, int64_t rows, int32_t* piv_dev,
                  void* tau_dev, int32_t* info_dev);

}  // namespace abft
