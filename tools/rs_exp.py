import os, sys, time
sys.path.insert(0, os.getcwd())
import torch, synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import abft
n, nb = 30720, 512
A0 = si.spd_device(n, seed=7); A = torch.empty_like(A0.t()).t(); ctx = abft.Context()
def run(ft, rs):
    A.copy_(A0); torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0=time.perf_counter(); a.record(); abft.ft_potrf(ctx, A, nb, abft=ft, restart=rs); t1=time.perf_counter(); b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b), (t1-t0)*1e3
for cfg in [(False,False),(True,False),(True,True)]:
    run(*cfg)
    r=[run(*cfg) for _ in range(3)]
    print(os.environ.get("ABFT_DBG_RESTART_NOSYNC","sync"), cfg, ["%.1f/%.1f"%x for x in r], flush=True)
