"""A/B helper: median per-region times over N synced steps of the cfg5 LM (one config per process)."""
import json, os, sys, statistics, torch
sys.path.insert(0, "/root/repo")
import bench
import paper_conf_asplos_sivathanucsz19_b200 as A
T, B, H, I, V = 100, 512, 2048, 2048, 256
cell = A.Cell("milstm", H, I, B, T, dtype="bf16", device=0)
lm = A.LM(cell, V)
lm.load(bench.make_params(I, H, V))
tok = torch.as_tensor(bench.make_inputs(B, T, V, 205, 0, 1), dtype=torch.int32).cuda()
var = os.environ.get("ASTRA_VARIANT", "a1=256.1.1.2,rec=256.1.1.2,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=0,bwd=0")
cell.tune_mode(A.TUNE_FROZEN, var)
n = int(sys.argv[1]) if len(sys.argv) > 1 else 8
for _ in range(3): lm.train_step(tok, 0.05)
torch.cuda.synchronize()
rs = []
for _ in range(n):
    lm.train_step(tok, 0.05)
    torch.cuda.synchronize()
    rs.append(bench.region_times(cell))
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(n): lm.train_step(tok, 0.05)
e1.record(); torch.cuda.synchronize()
med = {k: round(statistics.median(r[k] for r in rs), 3) for k in rs[0]}
med["b2b_ms"] = round(e0.elapsed_time(e1) / n, 3)
print(os.environ.get("AB_TAG", ""), json.dumps(med))
