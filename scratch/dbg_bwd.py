import sys, numpy as np
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
from helpers import make_cell_case, run_gpu_cell, rel_err
from oracle import cells as C
for (T, B, H) in [(3, 128, 64), (4, 128, 64)]:
    p, inp, dY, dhT, dcT = make_cell_case("lstm", T, B, 64, H, 91, bf16=True)
    oo, go = C.cell_fwd_bwd("lstm", p, inp, dY, dhT, dcT)
    r = {}
    for v in ("bwd=0", "bwd=1"):
        out, g, _ = run_gpu_cell("lstm", p, inp, dY, dhT, dcT, "bf16", v)
        r[v] = {k: rel_err(g[k], go[k]) for k in go}
    print(T, B, H, {k: (round(r["bwd=0"][k], 5), round(r["bwd=1"][k], 5)) for k in go})
