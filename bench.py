#!/usr/bin/env python
"""Benchmark of the 2D weighted-checksum hot path (BASELINE.json metric:
"checksum encode+verify GB/s vs HBM peak; ft_potrf overhead % at n=30720").

One timed STEP = abft_encode + abft_check (verify with the locate / correct
rounds fused into the same launch; they do nothing when no tile is flagged)
over the whole fp64 n=30720, nb=512 matrix
(7.55 GB per pass, larger than the 126 MB L2, so no flush is needed).  The
ft_potrf overhead half of the metric is measured in the same run: the
fault-tolerant driver (all §8(a) rows, Alg. 2 order) vs the same driver with
ABFT disabled, at n=30720 nb=512.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

N>1 is launched by torchrun: every rank owns its own n=30720 block-cyclic
share (weak scaling), encodes/verifies it, and the per-step error flags are
all-reduced over NCCL (the paper's error-report exchange, L361-L363).
`--impl reference` times the CPU oracle (oracle/, the plain implementation
written from the paper) on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

N_MAT, NB = 30720, 512
METRIC = "checksum encode+verify GB/s vs HBM peak; ft_potrf overhead % at n=30720"


def alg_bytes(n, nb, es):
    """Algorithmic bytes of one pass over an n x n matrix:
    n^2 s read + 4 n^2/nb s checksum write (encode) or read (verify)."""
    return n * n * es * (1.0 + 4.0 / nb)


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def ncu_traffic(n=None, nb=None, kernel=None):
    """dram read+write bytes per launch of the dominant kernel (`kernel`, the
    name bench.py reports) from the committed `ncu --set full` summary
    (profiles/) of the same (n, nb), or None."""
    p = os.path.join(ROOT, "profiles", "ncu_verify_summary.json")
    try:
        with open(p) as f:
            d = json.load(f)
        if d.get("n") == (n or N_MAT) and d.get("nb") == (nb or NB):
            return float(d["kernels"][kernel]["dram_bytes_per_launch"])
    except Exception:
        pass
    return None


class Clocks:
    """SM clock and clock-event (throttle) reasons sampled DURING the timed
    region (B200_PROFILING.md clocks line) by an NVML polling thread (1 ms),
    so even a ~20 ms timed region yields a few dozen samples; falls back to
    one nvidia-smi query if NVML is unavailable."""

    REASONS = {0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown", 0x4: "sw_power_cap"}

    def __init__(self, dev):
        self.dev = dev
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = False
        self._t = None

    def _nvml_index(self):
        vis = os.environ.get("CUDA_VISIBLE_DEVICES")
        if vis:
            ids = [v.strip() for v in vis.split(",") if v.strip()]
            if self.dev < len(ids) and ids[self.dev].isdigit():
                return int(ids[self.dev])
        return self.dev

    def _run(self):
        import pynvml

        h = pynvml.nvmlDeviceGetHandleByIndex(self._nvml_index())
        self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
        get_reasons = getattr(pynvml, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
            pynvml.nvmlDeviceGetCurrentClocksThrottleReasons
        while not self._stop:
            self.samples.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
            r = get_reasons(h)
            for bit, name in self.REASONS.items():
                if r & bit:
                    self.reasons.add(name)
            time.sleep(0.001)

    def __enter__(self):
        import threading

        try:
            import pynvml

            pynvml.nvmlInit()
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
            t0 = time.time()
            while not self.samples and time.time() - t0 < 2.0:  # sampler live before timing starts
                time.sleep(0.001)
        except Exception:
            self._t = None
        return self

    def __exit__(self, *a):
        self._stop = True
        if self._t:
            self._t.join(timeout=2)

    def summary(self):
        if not self.samples:
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.dev), "--query-gpu=clocks.sm,clocks.max.sm",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True, timeout=10)
                sm, mx = [float(x) for x in out.stdout.strip().split(",")[:2]]
                return {"sm_mhz": sm, "sm_max_mhz": mx, "reasons": [], "samples": 1, "source": "nvidia-smi after"}
            except Exception:
                return None
        sm = sorted(self.samples)
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                "samples": len(sm), "source": "nvml 1 ms during the timed region"}


# ------------------------------------------------------------- reference --
def workload_config(n, nb, world, potrf_n):
    """The `config` object of both arms' JSON lines (same workload named)."""
    try:
        import torch

        l2 = torch.cuda.get_device_properties(0).L2_cache_size if torch.cuda.is_available() else 126 * 2 ** 20
    except Exception:
        l2 = 126 * 2 ** 20
    return {"workload": f"encode+verify(+locate) fp64 n={n} nb={nb} per GPU, U(-1,1), full matrix "
                        f"(BASELINE configs[3] shape at the n={N_MAT} metric size)",
            "n": n, "nb": nb, "tiles_per_gpu": (n // nb) ** 2,
            "l2": f"inputs larger than L2 ({alg_bytes(n, nb, 8) / 1e9:.2f} GB/pass vs {l2 / 1e6:.0f} MB L2)",
            "parallelism": f"tiles block-cyclic, dp{world}", "ft_potrf_n": potrf_n}


def run_reference(args):
    """The oracle on the host cores: each step = encode + verify of a bounded
    sample (8 tiles) of nb x nb tiles drawn across an 8192^2 fp64 U(-1,1)
    matrix (not cache resident), same byte formula; host BLAS on all cores."""
    import synth_inputs as si
    from oracle import checksum as ck

    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    cores = len(os.sched_getaffinity(0))
    nb, m = NB, 8192
    n_tiles_sample = 8  # tiles per step sample
    st = ck.State.alloc(si.general(m, seed=0), nb)
    mt = m // nb
    g = si.rng(6)
    step_t = []
    for s in range(args.warmup + args.steps):
        picks = [(int(g.integers(0, mt)), int(g.integers(0, mt))) for _ in range(n_tiles_sample)]
        t0 = time.perf_counter()
        for I, J in picks:
            t = ck.Tiles(I, I + 1, J, J + 1)
            ck.encode(st, t)
            ck.verify(st, t)
        dt = time.perf_counter() - t0
        if s >= args.warmup:
            step_t.append(dt)
    bytes_step = 2 * n_tiles_sample * alg_bytes(nb, nb, 8)
    t = sum(step_t) / len(step_t)
    val = bytes_step / t / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": val, "unit": "GB/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": workload_config(args.n, nb, int(os.environ.get("WORLD_SIZE", "1")), args.potrf_n),
        "cpu_baseline": {"value": val, "unit": "GB/s", "cores": cores, "kind": "oracle", "cpu": _cpu_model(),
                         "sample": f"{n_tiles_sample} tiles of {nb}x{nb} fp64 per step drawn across an 8192^2 "
                                   f"matrix (not cache resident; a bounded sample of the n={args.n} workload, "
                                   f"GB/s with the same per-tile byte formula); host BLAS threads = {cores}"},
        "e2e": {"value": val, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def _oracle_ev_rate(seconds, threads):
    """Oracle encode+verify GB/s (the same per-tile byte formula as the GPU)
    over tiles spread across an 8192 x 8192 fp64 matrix (512 MB, larger than
    the host caches, so every tile comes from DRAM), with the host BLAS
    limited to `threads` threads; returns (GB/s, tiles, seconds)."""
    import threadpoolctl

    import synth_inputs as si
    from oracle import checksum as ck

    nb, m = NB, 8192
    st = ck.State.alloc(si.general(m, seed=1), nb)
    mt = m // nb
    order = [(I, J) for J in range(mt) for I in range(mt)]
    g = si.rng(5)
    g.shuffle(order)
    done, k = 0, 0
    with threadpoolctl.threadpool_limits(limits=threads, user_api="blas"):
        t0 = time.perf_counter()
        while time.perf_counter() - t0 < seconds:
            I, J = order[k % len(order)]
            t = ck.Tiles(I, I + 1, J, J + 1)
            ck.encode(st, t)
            ck.verify(st, t)
            done += 1
            k += 1
        dt = time.perf_counter() - t0
    return 2 * done * alg_bytes(nb, nb, 8) / dt / 1e9, done, dt


def cpu_baseline_sample(seconds=10.0, potrf_n=10240):
    """The oracle (oracle/, numpy + the host BLAS, untuned) on this box's host
    cores: encode+verify GB/s with the host BLAS on all
    affinity cores and on 1 core (non-cache-resident tiles), and the oracle's
    ft_potrf wall time at n=10240 nb=512 (Alg. 2, all cores).  `cores` is the
    BLAS thread count of the all-cores run; numpy's elementwise steps are
    single-threaded, so that is an upper bound on the threads used."""
    import threadpoolctl

    import synth_inputs as si
    from oracle import drivers as dr

    all_cores = len(os.sched_getaffinity(0))
    v_all, n_all, t_all = _oracle_ev_rate(seconds / 2, all_cores)
    v_one, n_one, t_one = _oracle_ev_rate(seconds / 2, 1)
    potrf_s = None
    if potrf_n:
        A = si.spd(potrf_n, seed=7)
        with threadpoolctl.threadpool_limits(limits=all_cores, user_api="blas"):
            t0 = time.perf_counter()
            dr.ft_potrf(A, NB)
            potrf_s = time.perf_counter() - t0
    return {"value": v_all, "unit": "GB/s", "cores": all_cores, "kind": "oracle",
            "value_1core": v_one, "cores_1core": 1,
            "ft_potrf_s": potrf_s, "ft_potrf_n": potrf_n, "ft_potrf_cores": all_cores,
            "cpu": _cpu_model(),
            "sample": f"encode+verify of {n_all} (all cores, {t_all:.1f} s) / {n_one} (1 core, {t_one:.1f} s) "
                      f"{NB}x{NB} fp64 tiles drawn across an 8192^2 matrix (512 MB, not cache resident); "
                      f"oracle ft_potrf n={potrf_n} nb={NB} once (Alg. 2, error free)"}


def _cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


# ------------------------------------------------------------------ ours --
def run_ours(args):
    import torch
    import torch.distributed as dist

    import synth_inputs as si
    from paper_conf_sc_chenlllwtolzgc18_b200 import abft
    from paper_conf_sc_chenlllwtolzgc18_b200 import dist as D

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # BENCH_SHARED_GPU=1 (tests only): every rank on cuda:0 over gloo, so the
    # N>1 code path can be exercised on a one-GPU box; numbers are not valid
    shared = os.environ.get("BENCH_SHARED_GPU") == "1"
    if shared:
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    n, nb = args.n, NB
    es = 8
    # ---- workload: each rank holds its own n x n block-cyclic share (weak) ----
    A = si.general_device(n, seed=1000 + rank)
    mat = abft.Mat.alloc(A, nb, mags=False)
    t_all = abft.tiles(0, n // nb, 0, n // nb)
    rep = abft.Report.alloc(mat)
    tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, 1.0)
    fixbuf = torch.zeros(1024 * abft.FIX_BYTES, dtype=torch.uint8, device="cuda")
    nfix = torch.zeros(1, dtype=torch.int32, device="cuda")
    stream = torch.cuda.current_stream()

    def step(ev=None):
        if ev:
            ev[0].record()
        abft.abft_encode(mat, t_all)
        if ev:
            ev[1].record()
        abft.abft_check(mat, t_all, abft.BOTH, tol, rep, fixbuf, nfix)  # verify + fused locate
        if ev:
            ev[2].record()
        if world > 1:
            D.reduce_counts(rep.counts)  # error-report exchange (L361-L363)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.steps)]
    t0e, t1e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with Clocks(local) as clk:
        torch.cuda.synchronize()
        t0e.record()
        for s in range(args.steps):
            step(evs[s])
        t1e.record()
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ms = t0e.elapsed_time(t1e)
    enc_ms = sum(e[0].elapsed_time(e[1]) for e in evs) / args.steps
    ver_ms = sum(e[1].elapsed_time(e[2]) for e in evs) / args.steps
    assert int(rep.counts.sum().item()) == 0, "error-free input flagged"
    if world > 1:
        tt = torch.tensor([ms], device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms = float(tt.item())
    pass_bytes = alg_bytes(n, nb, es)
    total_bytes = 2 * pass_bytes * args.steps * world
    value = total_bytes / (ms / 1e3) / 1e9
    peak, peak_src = peaks()
    dom_ms = max(enc_ms, ver_ms)
    dom = "checksum_pass_kernel<double,512,VERIFY=true>" if ver_ms >= enc_ms else "checksum_pass_kernel<double,512,VERIFY=false>"
    achieved = pass_bytes / (dom_ms / 1e3) / 1e9

    # ---- e2e: through the C ABI with host buffers (pinned H2D + result D2H) ----
    e2e = None
    if not args.no_e2e:
        hostA = torch.empty((n, n), dtype=torch.float64, pin_memory=True)
        hostA.copy_(A.t())  # row-major host image of the column-major matrix
        status_h = torch.empty_like(rep.status.t().contiguous(), device="cpu").pin_memory()
        counts_h = torch.empty(abft.NCOUNTS, dtype=torch.int32).pin_memory()
        e_steps = max(2, min(args.steps, 3))

        def e2e_step():
            A.t().copy_(hostA, non_blocking=True)  # H2D of the step's input
            step()
            counts_h.copy_(rep.counts, non_blocking=True)  # D2H of the result
            status_h.copy_(rep.status.t(), non_blocking=True)

        e2e_step()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(e_steps):
            e2e_step()
        b.record()
        torch.cuda.synchronize()
        ems = a.elapsed_time(b) / e_steps
        if world > 1:
            tt = torch.tensor([ems], device="cuda")
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            ems = float(tt.item())
        e2e = {"value": 2 * pass_bytes * world / (ems / 1e3) / 1e9, "unit": "GB/s",
               "h2d_bytes_per_step": n * n * es,
               "d2h_bytes_per_step": int(counts_h.numel() * 4 + status_h.numel() * 4), "ms_per_step": ems}
        del hostA

    # ---- context for the roofline: torch's own read-only reduction (sum) of
    # the same matrix, timed in the same run next to the copy peak of
    # MEASURED_PEAKS.json (the checksum pass is read-dominated) ----
    ro_ms = []
    for r in range(4):
        a_, b_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a_.record()
        A.sum()
        b_.record()
        torch.cuda.synchronize()
        if r:
            ro_ms.append(a_.elapsed_time(b_))
    read_only_gbs = n * n * es / (min(ro_ms) / 1e3) / 1e9
    del A, mat
    torch.cuda.empty_cache()
    # ---- BASELINE configs[4]: distributed ft_potrf on all ranks (row e) ----
    mg = None
    if not args.no_mgpu:
        mg = mgpu_overhead(si, args.mgpu_n, nb, args.mgpu_reps, world, rank)

    # ---- ft_potrf overhead at n=30720 (the metric's second half) ----
    ftp = lq = None
    if not args.no_potrf and rank == 0:
        ftp = potrf_overhead(abft, si, args.potrf_n, nb, args.potrf_reps, host_pd=not args.no_host_pd)
    if not args.no_lu_qr and rank == 0:
        lq = lu_qr_overhead(abft, si, args.lu_qr_n, nb, args.lu_qr_reps, host_pd=not args.no_host_pd)

    cpu = cpu_baseline_sample(args.cpu_seconds) if (rank == 0 and world == 1 and not args.no_cpu) else None
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": workload_config(n, nb, world, args.potrf_n),
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": ncu_traffic(n, nb, dom), "kernel": dom,
                         "bytes_per_launch": pass_bytes, "ms_per_launch": dom_ms, "peak_source": peak_src,
                         "encode_GBs": pass_bytes / (enc_ms / 1e3) / 1e9,
                         "verify_GBs": pass_bytes / (ver_ms / 1e3) / 1e9,
                         "torch_sum_GBs": read_only_gbs},
            "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": 2 * args.steps, "clocks": clk.summary(),
            "ft_potrf": ftp, "ft_getrf_geqrf": lq, "ft_potrf_mgpu": mg,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def potrf_overhead(abft, si, n, nb, reps, host_pd=True):
    """T_ft vs T_plain of the same blocked driver, plus cuSOLVER
    potrf as context; ms are CUDA-event times on the driver's stream."""
    import torch

    A0 = si.spd_device(n, seed=7)
    A = torch.empty_like(A0.t()).t()
    ctx = abft.Context()

    def run(ft, restart=True, pd=abft.PD_DEVICE, scheme=abft.SCHEME_NEW, gemm=False, la=True, timing=False):
        A.copy_(A0)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        rc, info, st = abft.ft_potrf(ctx, A, nb, abft=ft, restart=restart, pd_location=pd, scheme=scheme,
                                     checksum_gemm=gemm, lookahead=la, timing=timing)
        b.record()
        torch.cuda.synchronize()
        assert rc == 0 and info == 0
        return a.elapsed_time(b), st

    run(True)
    run(False)
    t_ft, t_plain, t_nors = [], [], []
    # one run of each without look-ahead (the Alg. 2 order of round 1) for context
    run(True, la=False)
    nola_ft, nola_plain = run(True, la=False)[0], run(False, la=False)[0]
    for _ in range(reps):
        t_plain.append(run(False)[0])
        t, st = run(True)
        t_ft.append(t)
        assert sum(st.counts) == 0
        t_nors.append(run(True, restart=False)[0])
    t_ft.sort()
    t_plain.sort()
    t_nors.sort()
    ft_ms, plain_ms = t_ft[len(t_ft) // 2], t_plain[len(t_plain) // 2]
    nors_ms = t_nors[len(t_nors) // 2]
    # the checking schemes the paper compares (L542, L653 Figs. 12-14; c-34),
    # same driver, same plain baseline, no restart (so that every scheme is
    # timed alike: SINGLE_PRE has no post-op check to restart from)
    schemes = {}
    # ("new_gemm_checks": the new scheme with the checks' recalculation done by
    # cuBLAS GEMMs, the paper's "without the optimized kernel", L653-L657)
    for name, sc, gm in (("new", abft.SCHEME_NEW, False), ("new_gemm_checks", abft.SCHEME_NEW, True),
                         ("full_post", abft.SCHEME_FULL_POST, False),
                         ("single_post", abft.SCHEME_SINGLE_POST, False),
                         ("single_pre", abft.SCHEME_SINGLE_PRE, False)):
        # all schemes in Alg. 2's sequential order (look-ahead applies to the
        # new scheme only), against the sequential unprotected driver
        run(True, restart=False, scheme=sc, gemm=gm, la=False)
        ts = sorted(run(True, restart=False, scheme=sc, gemm=gm, la=False)[0] for _ in range(max(1, reps - 1)))
        tm = ts[len(ts) // 2]
        schemes[name] = {"ms_ft": tm, "overhead_pct": 100.0 * (tm - nola_plain) / nola_plain}
    host = None
    if host_pd:  # Alg. 2 lines 3-7 with the PD on the host (FT_PD_HOST)
        import os

        ctx.set_host_lapack()
        run(True, pd=abft.PD_HOST)
        hf, hst = run(True, pd=abft.PD_HOST)
        hp = run(False, pd=abft.PD_HOST)[0]
        host = {"ms_ft": hf, "ms_plain": hp, "overhead_pct": 100.0 * (hf - hp) / hp, "ms_host_pd": hst.ms_host_pd,
                "host_cores": len(os.sched_getaffinity(0)), "lapack": os.path.basename(ctx.host_lapack)}
    # cuSOLVER dpotrf of the whole matrix (context)
    S = A0.t().contiguous()
    torch.backends.cuda.preferred_linalg_library("cusolver")
    torch.linalg.cholesky(S)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    torch.linalg.cholesky(S)
    b.record()
    torch.cuda.synchronize()
    cus = a.elapsed_time(b)
    phases = dict(zip(abft.PHASES, run(True, timing=True)[1].ms_phase))
    del S, A, A0
    torch.cuda.empty_cache()
    return {"n": n, "nb": nb, "ms_ft": ft_ms, "ms_plain": plain_ms,
            "overhead_pct": 100.0 * (ft_ms - plain_ms) / plain_ms, "cusolver_potrf_ms": cus,
            "overhead_vs_cusolver_pct": 100.0 * (ft_ms - cus) / cus,
            "lookahead": True, "phases_ms": phases,
            "phases_note": "device spans per phase on the stream each phase runs on; side-stream and rule-stream "
                           "spans overlap the main stream (the trailing checksum rule interleaves with the DSYRK, "
                           "so its span is about the DSYRK's)",
            "no_lookahead": {"ms_ft": nola_ft, "ms_plain": nola_plain,
                             "overhead_pct": 100.0 * (nola_ft - nola_plain) / nola_plain},
            "ms_ft_no_restart": nors_ms, "overhead_pct_no_restart": 100.0 * (nors_ms - plain_ms) / plain_ms,
            "tflops_ft": n ** 3 / 3 / (ft_ms / 1e3) / 1e12, "reps": reps, "host_pd": host,
            "schemes_no_restart": schemes}


def mgpu_overhead(si, n, nb, reps, world, rank):
    """BASELINE configs[4]: ft_potrf_mgpu (2D block-cyclic over the ranks,
    NCCL panel broadcasts + error-report all-reduce) at n=61440, ABFT on vs
    off; device time per rank between barriers, max over ranks."""
    import torch
    import torch.distributed as dist

    from paper_conf_sc_chenlllwtolzgc18_b200 import dist as D
    from paper_conf_sc_chenlllwtolzgc18_b200 import mgpu

    P, Q = D.grid_shape(world)
    lay = mgpu.Layout(n, nb, P, Q, rank)
    groups = D.Groups(P, Q)  # the broadcast communicators, created once (collective)
    A0 = si.spd_block_cyclic_device(n, nb, P, Q, rank, seed=61440)
    A = torch.empty_like(A0.t()).t()

    def run(ft):
        A.copy_(A0)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        rc, st = mgpu.ft_potrf_mgpu(A, lay, abft_on=ft, groups=groups)
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b)
        if world > 1:
            t = torch.tensor([ms], device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
        assert rc == 0 and st.info == 0 and sum(st.counts) == 0 and sum(st.bcast_counts) == 0
        return ms

    run(True)  # warm-up (allocator, cuBLAS / cuSOLVER handles, NCCL)
    t_ft, t_plain = [], []
    for _ in range(reps):
        t_plain.append(run(False))
        t_ft.append(run(True))
    del A, A0
    torch.cuda.empty_cache()
    ft_ms, plain_ms = min(t_ft), min(t_plain)
    return {"n": n, "nb": nb, "grid": [P, Q], "ms_ft": ft_ms, "ms_plain": plain_ms,
            "overhead_pct": 100.0 * (ft_ms - plain_ms) / plain_ms,
            "tflops_ft": n ** 3 / 3 / (ft_ms / 1e3) / 1e12, "reps": reps, "timing": "min over reps, max over ranks",
            "comm": "NCCL broadcast of L_kk inside its process column and of each panel piece to the ranks "
                    "that need it (dist.Groups); int32 decision all-reduce per round and report all-reduce"}


def lu_qr_overhead(abft, si, n, nb, reps, host_pd=True):
    """BASELINE configs[2]: ft_getrf / ft_geqrf at n=20480 nb=512, ABFT on vs
    the same driver with ABFT off; cuSOLVER getrf / geqrf as context.  With
    host_pd, also the FT_PD_HOST drivers (Alg. 2 lines 3-7: guarded panel
    round trip through pinned host memory around the host LAPACK, the
    configuration's 'panel/PCIe-transfer verification'), ABFT on vs off."""
    import torch

    A0 = si.general_device(n, seed=21)
    A = torch.empty_like(A0.t()).t()
    ctx = abft.Context()
    if host_pd:
        ctx.set_host_lapack()
    ipiv = torch.zeros(n, dtype=torch.int64, device="cuda")
    tau = torch.zeros(n, dtype=torch.float64, device="cuda")
    out = {"n": n, "nb": nb, "reps": reps}

    def run(fn, ft):
        A.copy_(A0)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        rc, info, st = fn(ft)
        b.record()
        torch.cuda.synchronize()
        assert rc == 0 and sum(st.counts) == 0, (rc, list(st.counts))
        return a.elapsed_time(b)

    for name, fn, flops in [("getrf", lambda ft: abft.ft_getrf(ctx, A, nb, ipiv, abft=ft), 2 * n ** 3 / 3),
                            ("geqrf", lambda ft: abft.ft_geqrf(ctx, A, nb, tau, abft=ft), 4 * n ** 3 / 3)]:
        run(fn, True)
        run(fn, False)
        tf = sorted(run(fn, True) for _ in range(reps))[reps // 2]
        tp = sorted(run(fn, False) for _ in range(reps))[reps // 2]
        out[name] = {"ms_ft": tf, "ms_plain": tp, "overhead_pct": 100.0 * (tf - tp) / tp,
                     "tflops_ft": flops / (tf / 1e3) / 1e12}
    if host_pd:
        import os

        for name, fn in [("getrf", lambda ft: abft.ft_getrf(ctx, A, nb, ipiv, abft=ft, pd_location=abft.PD_HOST)),
                         ("geqrf", lambda ft: abft.ft_geqrf(ctx, A, nb, tau, abft=ft, pd_location=abft.PD_HOST))]:
            run(fn, True)
            tf = run(fn, True)
            tp = run(fn, False)
            out[name]["host_pd"] = {"ms_ft": tf, "ms_plain": tp, "overhead_pct": 100.0 * (tf - tp) / tp,
                                    "host_cores": len(os.sched_getaffinity(0)),
                                    "lapack": os.path.basename(ctx.host_lapack)}
    torch.backends.cuda.preferred_linalg_library("cusolver")
    G = A0.t().contiguous()
    for name, fn in [("getrf", lambda: torch.linalg.lu_factor(G)), ("geqrf", lambda: torch.geqrf(G))]:
        fn()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        out[name]["cusolver_ms"] = a.elapsed_time(b)
    del G, A, A0
    torch.cuda.empty_cache()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--matrix-n", dest="n", type=int, default=N_MAT)  # not "--n": torchrun would take it
    ap.add_argument("--potrf-n", type=int, default=N_MAT)
    ap.add_argument("--potrf-reps", type=int, default=3)
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-potrf", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--lu-qr-n", type=int, default=20480)
    ap.add_argument("--lu-qr-reps", type=int, default=1)
    ap.add_argument("--no-lu-qr", action="store_true")
    ap.add_argument("--no-host-pd", action="store_true")
    ap.add_argument("--mgpu-n", type=int, default=61440)
    ap.add_argument("--mgpu-reps", type=int, default=1)
    ap.add_argument("--no-mgpu", action="store_true")
    args = ap.parse_args()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
