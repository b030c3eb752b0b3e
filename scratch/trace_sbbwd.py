"""Phase trace + timing of the small-batch persistent BPTT (bwd=2) at cfg5 shapes, B=64 (cell API)."""
import os, sys, json, numpy as np, torch
sys.path.insert(0, "/root/repo")
import synth
import paper_conf_asplos_sivathanucsz19_b200 as A
H = I = 2048; B = int(os.environ.get("SB_B", "64")); T = 100
c = A.Cell("milstm", H, I, B, T, dtype="bf16")
shapes = {k: (r, cc) if r > 1 else (cc,) for k, (off, r, cc) in c.param_info.items()}
c.load(synth.weights(7, shapes, H, {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)}))
x = (torch.rand(T, B, I, device="cuda") * 2 - 1).to(torch.bfloat16)
y = torch.empty(T, B, H, dtype=torch.bfloat16, device="cuda")
dy = (torch.randn(T, B, H, device="cuda") * 0.01).to(torch.bfloat16)
dx = torch.empty(T, B, I, dtype=torch.bfloat16, device="cuda")
res = {}
import bench
for v in ("bwd=0,bptt=128.1.1,bpw=1", "bwd=0,bptt=64.1.1,bpw=1", "bwd=2"):
    c.tune_mode(A.TUNE_FROZEN, v + ",fwd=3")
    for _ in range(3):
        c.forward(x, None, None, y); c.backward(dy, None, None, dx, None, None)
    torch.cuda.synchronize()
    ts = []
    for _ in range(5):
        c.forward(x, None, None, y); c.backward(dy, None, None, dx, None, None)
        torch.cuda.synchronize()
        ts.append(bench.region_times(c)["bptt_chain_ms"])
    res[v] = {"bptt_chain_ms": float(np.median(ts))}
NC = 2048 // 16
tr = torch.zeros(NC * T * 8, dtype=torch.int64, device="cuda")
c.forward(x, None, None, y)
A._check(A.lib().astra_debug_set_trace(3, A._ptr(tr)))
c.backward(dy, None, None, dx, None, None)
torch.cuda.synchronize()
A._check(A.lib().astra_debug_set_trace(3, None))
t = tr.cpu().numpy().reshape(NC, T, 8).astype(np.float64) / 1e3
st = slice(1, T - 2)   # GEMM steps t = T-2 .. 0 (skip the edges)
q = {}
q["step (cta0 flag->flag)"] = -np.diff(t[0, 1:T - 1, 0])
q["flag -> first A landed"] = (t[:, st, 1] - t[:, st, 0]).ravel()
q["first A -> MMAs issued"] = (t[:, st, 2] - t[:, st, 1]).ravel()
q["MMAs issued -> epi tfull"] = (t[:, st, 3] - t[:, st, 2]).ravel()
q["tfull -> xbuf arrive"] = (t[:, st, 4] - t[:, st, 3]).ravel()
q["arrive -> xready"] = (t[:, st, 5] - t[:, st, 4]).ravel()
q["xready -> stores done"] = (t[:, st, 6] - t[:, st, 5]).ravel()
q["stores -> published"] = (t[:, st, 7] - t[:, st, 6]).ravel()
# chunk c's producers: CTAs of groups 8c..8c+7; consumers wait for all of them
last_pub = np.zeros((4, T))
for cch in range(4):
    last_pub[cch] = t[cch * 32:(cch + 1) * 32, :, 7].max(0)
lat = []
for cta in range(NC):
    cch = cta % 4
    for tt in range(1, T - 2):
        lat.append(t[cta, tt, 0] - last_pub[cch, tt + 1])
q["last producer publish -> flag seen"] = np.array(lat)
q["publish spread within chunk"] = np.array([last_pub[c2, tt] - t[c2 * 32:(c2 + 1) * 32, tt, 7].min() for c2 in range(4) for tt in range(2, T - 1)])
out = {"B": B, "timing": res, "phases_us": {k: [round(float(np.median(v)), 3), round(float(np.percentile(v, 90)), 3)] for k, v in q.items()}}
print(json.dumps(out))
