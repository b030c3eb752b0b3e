import sys, numpy as np, torch
sys.path.insert(0, '.'); sys.path.insert(0, 'tests')
from helpers import make_cell_case, run_gpu_cell
from oracle import cells as C
def go(T,B,I,H,L,variant=None):
    p, inp, dY, dhT, dcT = make_cell_case("rhn", T, B, I, H, 123, bf16=True, L=L)
    o, g = C.cell_fwd_bwd("rhn", p, inp, dY, dhT, dcT)
    out, gg, c = run_gpu_cell("rhn", p, inp, dY, dhT, dcT, "bf16", variant, depth=L)
    W, Wo = gg["W"], g["W"]
    zr = int((np.abs(W).sum(1)==0).sum())
    print(T,B,I,H,L,variant, "W", np.linalg.norm(W-Wo)/np.linalg.norm(Wo), "zero rows", zr, "R", np.linalg.norm(gg["R"]-g["R"])/np.linalg.norm(g["R"]))
go(4,4,32,64,1)
go(4,4,32,64,3,"du=128,dw=128")
go(4,4,32,64,3,"du=64,dw=64")
go(4,16,32,64,1)
go(4,32,32,64,1)
go(4,4,64,64,1)
go(4,4,128,128,1)
go(8,16,128,128,2)
