"""Tiny invocations of the flag-barrier / persistent / peer kernels for compute-sanitizer
(memcheck, racecheck, synccheck): one case per argv[1]."""
import sys
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
import numpy as np, torch
from helpers import make_cell_case, run_gpu_cell

case = sys.argv[1]
if case == "rec_fused":        # K2 fused per step (1) and persistent (2), LSTM family
    p, inp, dY, dhT, dcT = make_cell_case("milstm", 3, 130, 64, 128, 5, bf16=True)
    for v in ("fwd=1", "fwd=2"):
        run_gpu_cell("milstm", p, inp, dY, dhT, dcT, "bf16", v)
elif case == "rec_persist":    # small-batch persistent forward (fwd=3)
    p, inp, dY, dhT, dcT = make_cell_case("milstm", 3, 16, 64, 128, 5, bf16=True)
    run_gpu_cell("milstm", p, inp, dY, dhT, dcT, "bf16", "fwd=3")
elif case == "bptt_fused":     # fused BPTT step (bwd=1)
    p, inp, dY, dhT, dcT = make_cell_case("lstm", 3, 130, 64, 128, 5, bf16=True)
    run_gpu_cell("lstm", p, inp, dY, dhT, dcT, "bf16", "bwd=1")
elif case == "rhn_fused":      # persistent RHN forward (fwd=1)
    p, inp, dY, dhT, dcT = make_cell_case("rhn", 2, 16, 64, 64, 5, bf16=True, L=2)
    run_gpu_cell("rhn", p, inp, dY, dhT, dcT, "bf16", "fwd=1", depth=2)
elif case == "bptt_persist":   # small-batch persistent BPTT (bwd=3)
    p, inp, dY, dhT, dcT = make_cell_case("milstm", 3, 16, 64, 128, 5, bf16=True)
    run_gpu_cell("milstm", p, inp, dY, dhT, dcT, "bf16", "bwd=3")
else:
    raise SystemExit(f"unknown case {case}")
torch.cuda.synchronize()
print("ok", case)
