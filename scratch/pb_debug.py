import sys, numpy as np
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
from helpers import make_cell_case, run_gpu_cell
cell, T, B, H = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
p, inp, dY, dhT, dcT = make_cell_case(cell, T, B, 64, H, 97, bf16=True)
o0, g0, _ = run_gpu_cell(cell, p, inp, dY, dhT, dcT, "bf16", "bwd=0")
o1, g1, _ = run_gpu_cell(cell, p, inp, dY, dhT, dcT, "bf16", "bwd=2")
for k in g0:
    d = np.abs(g0[k] - g1[k]).max()
    print(k, "equal" if np.array_equal(g0[k], g1[k]) else f"maxdiff {d:.3e} ref max {np.abs(g0[k]).max():.3e}")
