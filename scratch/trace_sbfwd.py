"""Phase trace + timing of the small-batch persistent forward (fwd=3) at cfg5 shapes, B=64 (cell API)."""
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
res = {}
for v in ("fwd=0,rec=64.1.1", "fwd=3"):
    c.tune_mode(A.TUNE_FROZEN, v)
    for _ in range(3): c.forward(x, None, None, y)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10): c.forward(x, None, None, y)
    e1.record(); torch.cuda.synchronize()
    import bench
    res[v] = {"fwd_call_ms": e0.elapsed_time(e1) / 10, "fwd_chain_ms": bench.region_times(c)["fwd_chain_ms"]}
NC = 2048 // 16
tr = torch.zeros(NC * T * 6 + 128, dtype=torch.int64, device="cuda")
A._check(A.lib().astra_debug_set_trace(2, A._ptr(tr)))
c.forward(x, None, None, y)
torch.cuda.synchronize()
A._check(A.lib().astra_debug_set_trace(2, None))
trn = tr.cpu().numpy()
t = trn[:NC * T * 6].reshape(NC, T, 6).astype(np.float64) / 1e3
kbs = trn[NC * T * 6:].astype(np.float64) / 1e3
c0 = kbs[64] * 1e3
cyc = lambda v: [int(x * 1e3 - c0) if x else None for x in v]
issue = {"A": cyc(kbs[0:8]), "B": cyc(kbs[32:44]), "mma_ready": cyc(kbs[64:96]), "mma_issued": cyc(kbs[96:128])}
land = None
q = {}
q["step (cta0 flag->flag)"] = np.diff(t[0, :, 0])
q["flag acquired -> first A landed"] = (t[:, :, 1] - t[:, :, 0]).ravel()
q["first A -> last MMA issued"] = (t[:, :, 2] - t[:, :, 1]).ravel()
q["last MMA issued -> epi sees tfull"] = (t[:, :, 3] - t[:, :, 2]).ravel()
q["epi tfull -> stores issued"] = (t[:, :, 3:5] @ [-1, 1]).ravel()
q["stores -> published"] = (t[:, :-1, 5] - t[:, :-1, 4]).ravel()
last_pub = t[:, :-1, 5].max(0)
q["last publish -> flag seen"] = (t[:, 1:, 0] - last_pub[None, :]).ravel()
q["publish spread (max-min)"] = t[:, :-1, 5].max(0) - t[:, :-1, 5].min(0)
out = {"env": {k: v for k, v in os.environ.items() if k.startswith("ASTRA_SB")}, "B": B, "timing": res,
       "kb_issue_us": issue, "kb_mma_us": land, "phases_us": {k: [round(float(np.median(v)), 3), round(float(np.percentile(v, 90)), 3)] for k, v in q.items()}}
print(json.dumps(out))
