"""Process body of the multi-rank ft_potrf_mgpu tests (spawned by
tests/test_gpu_mgpu.py): every rank shares cuda:0 and talks gloo over
127.0.0.1; rank 0 writes the gathered factor and the stats to out_path."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def run(rank, world, port, n, nb, grid, inject, out_path, abft_on, seed, restart=True):
    import torch
    import torch.distributed as dist

    import synth_inputs as si
    from paper_conf_sc_chenlllwtolzgc18_b200 import mgpu

    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        P, Q = grid
        lay = mgpu.Layout(n, nb, P, Q, rank)
        A = torch.from_numpy(si.spd(n, seed=seed))
        A_loc = mgpu.scatter_tiles(A, lay)
        rc, st = mgpu.ft_potrf_mgpu(A_loc, lay, abft_on=abft_on, inject=inject, restart=restart)
        torch.cuda.synchronize()
        L = mgpu.gather_tiles(A_loc, lay)
        if rank == 0:
            torch.save({"L": torch.tril(L), "rc": rc, "counts": st.counts, "bcast_counts": st.bcast_counts,
                        "bcast_events": st.bcast_events, "tmu_consumed": st.tmu_consumed, "info": st.info,
                        "uncorrectable": st.uncorrectable, "restarts": st.restarts}, out_path)
    finally:
        dist.destroy_process_group()
