import sys, time, json, torch
sys.path.insert(0, "/root/repo")
import bench
import paper_conf_asplos_sivathanucsz19_b200 as A
T, B, H, I, V = 100, 512, 2048, 2048, 256
cell = A.Cell("milstm", H, I, B, T, dtype="bf16", device=0)
lm = A.LM(cell, V)
lm.load(bench.make_params(I, H, V))
tok = torch.as_tensor(bench.make_inputs(B, T, V, 205, 0, 1), dtype=torch.int32).cuda()
V0 = sys.argv[1] if len(sys.argv) > 1 else ""
if V0: cell.tune_mode(A.TUNE_FROZEN, V0)
for _ in range(3): lm.train_step(tok, 0.05)
torch.cuda.synchronize()
# host enqueue time per step with the GPU far behind (no sync)
t0 = time.perf_counter()
for _ in range(10): lm.train_step(tok, 0.05)
t1 = time.perf_counter()
torch.cuda.synchronize()
t2 = time.perf_counter()
print(json.dumps({"host_enqueue_ms_per_step": (t1 - t0) * 100, "wall_ms_per_step": (t2 - t0) * 100}))
