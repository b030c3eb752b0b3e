"""bptt_chain_ms of the persistent BPTT (bwd=2) at cfg5 B=64 for the ASTRA_PB_* knobs in the env."""
import os, sys, json, numpy as np, torch
sys.path.insert(0, "/root/repo")
import synth
import paper_conf_asplos_sivathanucsz19_b200 as A
import bench
H = I = 2048; B = int(os.environ.get("SB_B", "64")); T = 100
c = A.Cell("milstm", H, I, B, T, dtype="bf16")
shapes = {k: (r, cc) if r > 1 else (cc,) for k, (off, r, cc) in c.param_info.items()}
c.load(synth.weights(7, shapes, H, {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)}))
x = (torch.rand(T, B, I, device="cuda") * 2 - 1).to(torch.bfloat16)
y = torch.empty(T, B, H, dtype=torch.bfloat16, device="cuda")
dy = (torch.randn(T, B, H, device="cuda") * 0.01).to(torch.bfloat16)
dx = torch.empty(T, B, I, dtype=torch.bfloat16, device="cuda")
v = os.environ.get("PB_VARIANT", "bwd=2,fwd=3")
c.tune_mode(A.TUNE_FROZEN, v)
for _ in range(3):
    c.forward(x, None, None, y); c.backward(dy, None, None, dx, None, None)
torch.cuda.synchronize()
ts = []
for _ in range(5):
    c.forward(x, None, None, y); c.backward(dy, None, None, dx, None, None)
    torch.cuda.synchronize()
    ts.append(bench.region_times(c)["bptt_chain_ms"])
print(json.dumps({"env": {k: vv for k, vv in os.environ.items() if k.startswith("ASTRA_PB")}, "variant": v,
                  "bptt_chain_ms": round(float(np.median(ts)), 4)}), flush=True)
