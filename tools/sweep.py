"""BASELINE configs[3]: standalone checksum encode+verify bandwidth sweep,
n = 4096..65536 x nb in {256, 512, 1024} x {fp32, fp64}, GENERAL view, plus
the Cholesky lower-only variant and the paper's prior-art GEMM-based checksum
([11],[12]; L35, L442) timed on the same matrices (the B200 analogue of the
paper's 1.7x claim, NEXT row f3).  CUDA events, 3 warm-ups, median of reps;
inputs below 16x L2 are re-read after an L2 flush (write a buffer larger than
L2, then read another one, so that no dirty line is written back inside the
timed pass).  Writes
gpurun_out/sweep.json.
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft

L2 = torch.cuda.get_device_properties(0).L2_cache_size
try:  # SM clock right after each timed set (a record, not a filter)
    import pynvml

    pynvml.nvmlInit()
    _nvh = pynvml.nvmlDeviceGetHandleByIndex(torch.cuda.current_device())

    def sm_clock():
        return pynvml.nvmlDeviceGetClockInfo(_nvh, pynvml.NVML_CLOCK_SM)
except Exception:  # noqa: BLE001
    def sm_clock():
        return None
flush = torch.empty(4 * L2, dtype=torch.uint8, device="cuda")
evict = torch.empty(4 * L2 // 8, dtype=torch.float64, device="cuda")


def flush_l2():
    # write a buffer larger than L2, then read another one: the dirty lines the
    # write leaves are written back during the read, not inside the timed pass
    # (a write-only flush added ~126 MB of write-backs to a 512 MB pass)
    flush.add_(1)
    evict.sum()


def timed(fn, reps, need_flush):
    for _ in range(3):
        fn()
    ts = []
    for _ in range(reps):
        if need_flush:
            flush_l2()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


def main():
    sizes = [int(x) for x in os.environ.get("SWEEP_N", "4096,8192,16384,32768,65536").split(",")]
    out = []
    mem = torch.cuda.get_device_properties(0).total_memory
    for dt, es in ((torch.float64, 8), (torch.float32, 4)):
        for n in sizes:
            if n * n * es * 2.2 > mem:
                continue
            A = si.general_device(n, seed=n, dtype=dt)
            for nb in (256, 512, 1024):
                for lower in (False, True):
                    mat = abft.Mat.alloc(A, nb, mags=False)
                    t = abft.tiles(0, n // nb, 0, n // nb, lower, abft.SYM_LOWER if lower else abft.GENERAL)
                    rep = abft.Report.alloc(mat)
                    tol = abft.abft_tol_t(abft.TOL_MAGNITUDE, 1.0, 0)
                    ntiles = (n // nb) * (n // nb + 1) // 2 if lower else (n // nb) ** 2
                    bytes_pass = ntiles * nb * nb * es * (1 + 4 / nb)
                    small = bytes_pass < 16 * L2  # re-read after a (clean) flush below 2 GB
                    reps = 20 if n <= 16384 else 8
                    te = timed(lambda: abft.abft_encode(mat, t), reps, small)
                    clk_e = sm_clock()
                    tv = timed(lambda: abft.abft_verify(mat, t, abft.BOTH, tol, rep), reps, small)
                    clk_v = sm_clock()
                    assert int(rep.counts.sum().item()) == 0
                    rec = {"dtype": str(dt).split(".")[-1], "n": n, "nb": nb, "lower_only": lower,
                           "encode_GBs": bytes_pass / te / 1e6, "verify_GBs": bytes_pass / tv / 1e6,
                           "encode_verify_GBs": 2 * bytes_pass / (te + tv) / 1e6, "l2_flushed": small,
                           "sm_mhz_after_encode": clk_e, "sm_mhz_after_verify": clk_v}
                    if not lower:
                        V = torch.stack([torch.ones(nb, dtype=dt, device="cuda"),
                                         torch.arange(1, nb + 1, dtype=dt, device="cuda")], 1)
                        nt = n // nb
                        At = A.t()  # row-major (n, n) storage of the column-major matrix

                        def gemm_chk():
                            # prior art: column checksums V^T X and row checksums X V per tile as GEMMs
                            torch.matmul(At.reshape(n, nt, nb), V)  # per tile column block: A^T rows . V
                            torch.matmul(V.t(), At.reshape(nt, nb, n))

                        tg = timed(gemm_chk, reps, small)
                        rec["gemm_prior_art_GBs"] = bytes_pass / tg / 1e6
                        rec["speedup_vs_gemm"] = tg / te
                    out.append(rec)
                    print(json.dumps(rec), flush=True)
                    del mat, rep
            del A
            torch.cuda.empty_cache()
    os.makedirs("gpurun_out", exist_ok=True)
    with open("gpurun_out/sweep.json", "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
