"""Batch-size consistency: an LM batch of duplicated sequences must give the same mean loss /
gradients as the distinct sequences alone."""
import sys
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
import numpy as np, torch, synth
from oracle import lm as OLM
from helpers import bf16_round, cell_shapes, rel_l2
import paper_conf_asplos_sivathanucsz19_b200 as A

def run(dtype, T, H, I, V, tok, p):
    B = tok.shape[1]
    c = A.Cell("milstm", H, I, B, T, dtype=dtype)
    m = A.LM(c, V); m.load(p)
    m.set_state(torch.zeros(B, H, device="cuda"), torch.zeros(B, H, device="cuda"))
    loss = float(m.fwd_bwd(torch.as_tensor(tok, dtype=torch.int32, device="cuda")).item())
    torch.cuda.synchronize()
    return loss, {k: m.view(k, m.grads).cpu().numpy().reshape(np.shape(p[k])) for k in p}

for dtype in ("fp32", "bf16"):
    for (T, H, I, V) in [(2, 64, 64, 48), (8, 256, 128, 256)]:
        seed = 99
        shapes = cell_shapes("milstm", I, H); shapes.update({"E": (V, I), "W_o": (H, V), "b_o": (V,)})
        p = synth.weights(seed, shapes, H, {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)})
        for k in ("W", "U", "E", "W_o"): p[k] = bf16_round(p[k])
        d8 = synth.zipf_tokens(seed, "tok", (T + 1, 8), V, V - 5)
        l8, g8 = run(dtype, T, H, I, V, d8, p)
        lo, go, _ = OLM.lm_forward_backward("milstm", p, d8, np.zeros((8, H)), np.zeros((8, H)))
        print(dtype, T, H, "B8 vs oracle", l8, lo, {k: round(rel_l2(g8[k], go[k]), 6) for k in go}, flush=True)
        for name, idx in [("dup16-interleave", np.arange(16) % 8), ("dup16-blocks", np.repeat(np.arange(8), 2)),
                          ("dup64", np.arange(64) % 8)]:
            l, g = run(dtype, T, H, I, V, d8[:, idx], p)
            print(dtype, T, H, name, "loss", l, "vs B8", l8, {k: round(rel_l2(g[k], g8[k]), 6) for k in go}, flush=True)
