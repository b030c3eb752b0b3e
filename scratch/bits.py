"""Save the params after 3 LM steps of a small cfg3-like RHN and cfg2-like SCRN LM (A/B bitwise checks across builds)."""
import sys, numpy as np, torch
sys.path.insert(0, "/root/repo")
import synth
import paper_conf_asplos_sivathanucsz19_b200 as A
out = []
for cell, kw, H in (("rhn", {"depth": 10}, 830), ("scrn", {"context": 1024, "scrn_alpha": 0.95}, 1024)):
    T, B, V = 6, 64, 1000
    c = A.Cell(cell, H, H, B, T, dtype="bf16", **kw)
    m = A.LM(c, V)
    shapes = {k: (r, cc) if r > 1 else (cc,) for k, (off, r, cc) in m.param_info.items()}
    m.load(synth.weights(5, shapes, H))
    tok = torch.as_tensor(synth.zipf_tokens(5, "tok", (T + 1, B), V, None), dtype=torch.int32).cuda()
    for _ in range(3): m.train_step(tok, 0.1)
    torch.cuda.synchronize()
    out.append(m.params.cpu().numpy())
np.save(sys.argv[1], np.concatenate(out))
