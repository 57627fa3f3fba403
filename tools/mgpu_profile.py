"""Time ft_potrf_mgpu (ABFT on / off) on the ranks of a torchrun launch
(or one process): python tools/mgpu_profile.py N NB [reps]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import torch.distributed as dist

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import dist as D
from paper_conf_sc_chenlllwtolzgc18_b200 import mgpu

n, nb = int(sys.argv[1]), int(sys.argv[2])
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
world = int(os.environ.get("WORLD_SIZE", 1))
rank = int(os.environ.get("RANK", 0))
torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", 0)))
if world > 1:
    dist.init_process_group("nccl")
P, Q = D.grid_shape(world)
lay = mgpu.Layout(n, nb, P, Q, rank)
A0 = si.spd_block_cyclic_device(n, nb, P, Q, rank, seed=5)
A = torch.empty_like(A0.t()).t()
for ft in (False, True, False, True):
    ts = []
    for _ in range(reps):
        A.copy_(A0)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        a.record()
        rc, st = mgpu.ft_potrf_mgpu(A, lay, abft_on=ft)
        b.record()
        torch.cuda.synchronize()
        ts.append((a.elapsed_time(b), (time.perf_counter() - t0) * 1e3, rc, st.counts[0], st.info))
    if rank == 0:
        print(f"n={n} nb={nb} grid={P}x{Q} abft={ft} " + " ".join(f"{d:.1f}/{h:.1f}ms rc={r} flg={f} info={i}"
                                                            for d, h, r, f, i in ts), flush=True)
if world > 1:
    dist.destroy_process_group()
