"""Box calibration: device props, read-only HBM GB/s, DGEMM,
cuSOLVER potrf/getrf/geqrf context timings, GEMM-based checksum (prior art,
paper L35/L442) GB/s. Torch only; writes gpurun_out/calibration.json."""
import json, os, platform, time
import torch

def timeit(fn, reps=10, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); fn(); e.record(); torch.cuda.synchronize()
        ts.append(s.elapsed_time(e))
    ts.sort()
    return ts[len(ts) // 2]

out = {}
p = torch.cuda.get_device_properties(0)
out["device"] = {"name": p.name, "sms": p.multi_processor_count, "mem": p.total_memory,
                 "l2": getattr(p, "L2_cache_size", None)}
out["host"] = {"cores": len(os.sched_getaffinity(0)), "cpu": platform.processor()}
try:
    with open("/proc/cpuinfo") as f:
        for line in f:
            if line.startswith("model name"):
                out["host"]["cpu"] = line.split(":", 1)[1].strip(); break
    with open("/proc/meminfo") as f:
        out["host"]["mem"] = f.readline().strip()
except Exception:
    pass
flush = torch.empty(512 * 1024 * 1024, dtype=torch.uint8, device="cuda")
for dt in (torch.float64, torch.float32):
    x = torch.rand(8 * 1024**3 // torch.tensor([], dtype=dt).element_size(), dtype=dt, device="cuda")
    t = timeit(lambda: x.sum())
    out[f"read_sum_{dt}"] = x.numel() * x.element_size() / t / 1e6
    y = torch.empty_like(x)
    t = timeit(lambda: y.copy_(x))
    out[f"copy_{dt}"] = 2 * x.numel() * x.element_size() / t / 1e6
    del x, y
torch.cuda.empty_cache()
for n in (8192,):
    a = torch.rand(n, n, dtype=torch.float64, device="cuda"); b = torch.rand_like(a)
    t = timeit(lambda: a @ b)
    out[f"dgemm_{n}_tflops"] = 2 * n**3 / t / 1e9
n, k = 30720, 512
a = torch.rand(n, k, dtype=torch.float64, device="cuda"); c = torch.rand(n, n, dtype=torch.float64, device="cuda")
t = timeit(lambda: c.addmm_(a, a.T, alpha=-1.0), reps=5)
out["dgemm_tmu_30720x30720x512_tflops"] = 2 * n * n * k / t / 1e9
s = torch.rand(120, k, dtype=torch.float64, device="cuda"); o = torch.empty(120, n, dtype=torch.float64, device="cuda")
t = timeit(lambda: torch.mm(s, a.T, out=o))
out["dgemm_skinny_120x30720x512_tflops"] = 2 * 120 * n * k / t / 1e9
del a, c, s, o
torch.cuda.empty_cache()
# prior art: GEMM-based checksum encoding (batched V^T X and X V per tile)
for dt in (torch.float64, torch.float32):
    for n in (16384, 32768):
        for nb in (256, 512, 1024):
            A = torch.rand(n, n, dtype=dt, device="cuda")  # row-major view: treat as A^T col-major; symmetric cost
            V = torch.stack([torch.ones(nb, dtype=dt, device="cuda"), torch.arange(1, nb + 1, dtype=dt, device="cuda")], 1)
            nt = n // nb
            def enc():
                # column checksums: V^T (nb x n) per tile row
                cc = torch.matmul(V.T, A.view(nt, nb, n))
                rc = torch.matmul(A.view(n, nt, nb), V)
                return cc, rc
            t = timeit(enc, reps=5)
            out[f"gemm_checksum_{dt}_{n}_{nb}_GBs"] = n * n * A.element_size() * (1 + 4 / nb) / t / 1e6
            del A
            torch.cuda.empty_cache()
# cuSOLVER context
torch.backends.cuda.preferred_linalg_library("cusolver")
for n in (10240, 30720):
    M = torch.rand(n, n, dtype=torch.float64, device="cuda"); S = (M + M.T) / 2 + n * torch.eye(n, dtype=torch.float64, device="cuda")
    del M
    t = timeit(lambda: torch.linalg.cholesky(S), reps=3, warm=1)
    out[f"cusolver_potrf_{n}_ms"] = t
    out[f"cusolver_potrf_{n}_tflops"] = n**3 / 3 / t / 1e9
    del S; torch.cuda.empty_cache()
n = 20480
G = torch.rand(n, n, dtype=torch.float64, device="cuda")
t = timeit(lambda: torch.linalg.lu_factor(G), reps=3, warm=1); out["cusolver_getrf_20480_ms"] = t
t = timeit(lambda: torch.geqrf(G), reps=3, warm=1); out["cusolver_geqrf_20480_ms"] = t
print(json.dumps(out, indent=1))
os.makedirs("gpurun_out", exist_ok=True)
with open("gpurun_out/calibration.json", "w") as f:
    json.dump(out, f, indent=1)
