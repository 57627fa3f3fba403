"""One ft_potrf_mgpu run on one GPU for an ncu launch list: python tools/mgpu_once.py N NB ABFT"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import synth_inputs as si
from paper_conf_sc_chenlllwtolzgc18_b200 import mgpu

n, nb, ft = int(sys.argv[1]), int(sys.argv[2]), bool(int(sys.argv[3]))
lay = mgpu.Layout(n, nb, 1, 1, 0)
A = si.spd_block_cyclic_device(n, nb, 1, 1, 0, seed=5)
rc, st = mgpu.ft_potrf_mgpu(A, lay, abft_on=ft)
torch.cuda.synchronize()
print(rc, st.counts)
