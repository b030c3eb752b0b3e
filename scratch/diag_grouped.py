"""Diagnose the full-size grouped cfg5 LM parity failure: per-variant l2 errors vs the oracle."""
import sys, json, time
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
import numpy as np, torch, synth
from oracle import lm as OLM
from helpers import bf16_round, cell_shapes, rel_l2
import paper_conf_asplos_sivathanucsz19_b200 as A

T = int(sys.argv[1]) if len(sys.argv) > 1 else 100
B, I, H, V, G = 512, 2048, 2048, 256, 8
seed = synth.config_seed(5) + 200
shapes = cell_shapes("milstm", I, H); shapes.update({"E": (V, I), "W_o": (H, V), "b_o": (V,)})
p = synth.weights(seed, shapes, H, {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)})
for k in ("W", "U", "E", "W_o"): p[k] = bf16_round(p[k])
distinct = synth.zipf_tokens(seed, "tok", (T + 1, G), V, 205)
group = synth.rng(seed, "groups").permutation(np.repeat(np.arange(G), B // G))
t0 = time.time()
lo, go, _ = OLM.lm_forward_backward("milstm", p, distinct, np.zeros((G, H)), np.zeros((G, H)))
print("oracle", time.time() - t0, "s loss", lo, flush=True)
BV = "a1=256.1.1.2,rec=256.1.1.2,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=0,bwd=0"
for name, bsz, var in [("b512-bench-hov1", B, BV + ",hov=1"), ("b512-bench-hov0", B, BV + ",hov=0"),
                       ("b512-default", B, None), ("b8-default", G, None), ("b64-default", 64, None)]:
    if bsz == B:
        tok = distinct[:, group]
    elif bsz == G:
        tok = distinct
    else:
        tok = distinct[:, np.arange(bsz) % G]
    c = A.Cell("milstm", H, I, bsz, T, dtype="bf16")
    if var: c.tune_mode(A.TUNE_FROZEN, var)
    m = A.LM(c, V); m.load(p)
    m.set_state(torch.zeros(bsz, H, device="cuda"), torch.zeros(bsz, H, device="cuda"))
    loss = float(m.fwd_bwd(torch.as_tensor(tok, dtype=torch.int32, device="cuda")).item())
    torch.cuda.synchronize()
    g = {k: m.view(k, m.grads).cpu().numpy().reshape(np.shape(p[k])) for k in p}
    print(name, "loss", loss, {k: round(rel_l2(g[k], go[k]), 5) for k in go}, flush=True)
    del m, c; torch.cuda.empty_cache()
