"""Phase trace of the forward pointwise kernel inside the cfg5 chain (last launch of a step)."""
import os, sys, numpy as np, torch
sys.path.insert(0, "/root/repo")
tr = None
def main():
    import bench
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, H, I, V = 100, 512, 2048, 2048, 256
    buf = torch.zeros(600 * 34, dtype=torch.int64, device="cuda")
    A._check(A.lib().astra_debug_set_trace(0, A._ptr(buf)))
    cell = A.Cell("milstm", H, I, B, T, dtype="bf16")
    lm = A.LM(cell, V)
    lm.load(bench.make_params(I, H, V))
    tok = torch.as_tensor(bench.make_inputs(B, T, V, 205, 0, 1), dtype=torch.int32).cuda()
    cell.tune_mode(A.TUNE_FROZEN, "a1=256.1.1.2,rec=256.1.1.2,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,wg_side=1,fwd=0")
    for _ in range(3): lm.train_step(tok, 0.01)
    torch.cuda.synchronize()
    t = buf.cpu().numpy().reshape(600, 34).astype(np.float64)
    g = 444   # 3 CTAs per SM since session 5 (was 296)
    t = t[:g] / 1e3
    t0 = t[:, 0].min()
    print("kernel span (first entry -> last row done) us:", round(t[:, 3::2].max() - t0, 2))
    print("entry spread us:", round(t[:, 0].max() - t0, 2), " pdl_wait done (median rel. to first entry):", round(np.median(t[:, 1] - t0), 2))
    for k in range(8):
        ready = t[:, 2 + 2 * k] - t0
        done = t[:, 3 + 2 * k] - t0
        ok = t[:, 2 + 2 * k] > 0
        print(f"row {k}: ready median {np.median(ready[ok]):6.2f}  done median {np.median(done[ok]):6.2f}  (n={ok.sum()})")
main()
