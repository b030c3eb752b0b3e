import sys, numpy as np, torch
sys.path.insert(0, '.'); sys.path.insert(0, 'tests')
from helpers import make_cell_case, run_gpu_cell
import synth
from oracle import cells as C
T,B,I,H,L = 4,4,32,64,3
p, inp, dY, dhT, dcT = make_cell_case("rhn", T, B, I, H, 123, bf16=True, L=L)
o, g = C.cell_fwd_bwd("rhn", p, inp, dY, dhT, dcT)
for dt in ["fp32","bf16"]:
    out, gg, c = run_gpu_cell("rhn", p, inp, dY, dhT, dcT, dt, None, depth=L)
    for k in ["W","R","b","dx","dh0"]:
        a, r = gg[k], g[k]
        print(dt, k, np.linalg.norm(a-r)/np.linalg.norm(r))
    R = gg["R"]; Ro = g["R"]
    for l in range(L):
        for half in range(2):
            a = R[l][:, half*H:(half+1)*H]; r = Ro[l][:, half*H:(half+1)*H]
            print(dt, "R", l, half, np.linalg.norm(a-r)/np.linalg.norm(r), np.abs(a).max(), np.abs(r).max())
    W = gg["W"]; Wo = g["W"]
    print(dt, "W halves", [np.linalg.norm(W[:, h*H:(h+1)*H]-Wo[:, h*H:(h+1)*H])/np.linalg.norm(Wo[:, h*H:(h+1)*H]) for h in range(2)])
    print(W[:3,:4], Wo[:3,:4])
