// abft_locate.cu — a3: locate / classify / correct flagged tiles in place.
//
// Paper: detect |delta_1| > e_c, locate j = round(delta_2/delta_1), correct
// with the magnitude delta_1 (L122, §III.B); full checksums tolerate an
// erroneous row or column checksum (L145); 0D/1D/2D propagation classes
// (L330-L334); "same row => 1D, otherwise 2D" (L432-L434, §VII.D).
// Readings: c-4 correction x <- c_e - sum_{r!=i} X[r][j];
// c-5 acceptance of the rounded ratio; c-7 non-finite fallback with
// confirmation; c-11 class order 0D/1D_ROW -> 0D/1D_COL -> CHK_CORRUPT (c-11b) ->
// SYM pair -> SYM_CROSS -> STALE -> 2D, at most 3 rounds.
//
// This is the rare path (only tiles whose verify status is non-zero do any
// work), so it favours clarity: one 256-thread CTA per flagged tile, warp-per-
// column sums, thread-per-row sums, the class decision by thread 0 on
// shared-memory flag tables, corrections executed warp-parallel.
#include "abft_locate.cuh"

namespace abft {

template <typename T>
__global__ void __launch_bounds__(kLThreads) locate_correct_kernel(const __grid_constant__ LocArgs p) {
  if (p.gate && *p.gate == 0) return;
  extern __shared__ __align__(16) unsigned char sm[];
  for (int64_t t = blockIdx.x; t < p.ntiles; t += gridDim.x) {
    int I, J;
    tile_of(p.tiles, t, I, J);
    int32_t* stp = p.status + I + (int64_t)J * p.ld_status;
    if ((*stp & (ABFT_ST_COL | ABFT_ST_ROW)) == 0) continue;  // uniform across the CTA
    locate_tile<T>(p, I, J, stp, sm);
  }
}

int validate_mat(const abft_mat_t* m, const abft_tiles_t* t, int which);

template <typename T>
static int launch_locate(LocArgs& a, cudaStream_t s) {
  const size_t smem = locate_smem_bytes(a.nb, (int)sizeof(T));
  auto k = locate_correct_kernel<T>;
  ABFT_CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int64_t grid = a.ntiles < 592 ? a.ntiles : 592;
  k<<<(unsigned)grid, kLThreads, smem, s>>>(a);
  ABFT_CUDA_TRY(cudaGetLastError());
  return 0;
}

int fill_loc_args(LocArgs& a, const abft_mat_t* m, const abft_tiles_t* t, int32_t which, const abft_tol_t* tol,
                  const abft_report_t* rep, abft_fix_t* fixes, int32_t max_fixes, int32_t* n_fixes) {
  int rc = validate_mat(m, t, which);
  if (rc) return rc;
  if (!tol) return -4;
  if (!rep || !rep->status || !rep->counts || rep->ld_status < m->m / m->nb) return -5;
  if (max_fixes < 0 || (max_fixes > 0 && !fixes)) return -7;
  if (!n_fixes) return -8;
  a = LocArgs{};
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
  a.nb = (int)m->nb;
  a.which = which;
  a.use_mag = tol->kind == ABFT_TOL_MAGNITUDE && (!(which & ABFT_COL) || m->colmag) &&
              (!(which & ABFT_ROW) || m->rowmag);
  a.tau_fac = m->dtype == ABFT_F64 ? tau_factor<double>((int)m->nb, tol->scale)
                                   : tau_factor<float>((int)m->nb, tol->scale);
  a.status = rep->status;
  a.ld_status = rep->ld_status;
  a.counts = rep->counts;
  a.fixes = fixes;
  a.max_fixes = max_fixes;
  a.n_fixes = n_fixes;
  a.ntiles = tiles_count(*t);
  a.gate = launch_gate();
  return 0;
}

int launch_locate_args(LocArgs& a, int32_t dtype, cudaStream_t s) {
  if (a.ntiles == 0) return 0;
  return dtype == ABFT_F64 ? launch_locate<double>(a, s) : launch_locate<float>(a, s);
}

}  // namespace abft

extern "C" int abft_locate_correct(const abft_mat_t* m, const abft_tiles_t* t, int32_t which, const abft_tol_t* tol,
                                   const abft_report_t* rep, abft_fix_t* fixes, int32_t max_fixes, int32_t* n_fixes,
                                   abft_stream_t stream) {
  abft::LocArgs a;
  const int rc = abft::fill_loc_args(a, m, t, which, tol, rep, fixes, max_fixes, n_fixes);
  if (rc) return rc;
  return abft::launch_locate_args(a, m->dtype, (cudaStream_t)stream);
}
