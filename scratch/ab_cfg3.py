"""cfg3 RHN LM (L=10, H=830, B=64, T=35, V=10k): median region times per frozen variant (argv)."""
import json, sys, statistics, torch
sys.path.insert(0, "/root/repo")
import synth, bench
import paper_conf_asplos_sivathanucsz19_b200 as A
H, I, B, T, V = 830, 830, 64, 35, 10000
c = A.Cell("rhn", H, I, B, T, dtype="bf16", depth=10)
m = A.LM(c, V)
shapes = {k: (r, cc) if r > 1 else (cc,) for k, (off, r, cc) in m.param_info.items()}
m.load(synth.weights(777, shapes, H))
tok = torch.as_tensor(synth.zipf_tokens(777, "tok", (T + 1, B), V, None), dtype=torch.int32).cuda()
for v in sys.argv[1:]:
    c.tune_mode(A.TUNE_FROZEN, v)
    for _ in range(3): m.train_step(tok, 0.01)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10): m.train_step(tok, 0.01)
    e1.record(); torch.cuda.synchronize()
    m.set_graph(False); m.train_step(tok, 0.01); torch.cuda.synchronize()
    r = {k: round(x, 3) for k, x in bench.region_times(c).items()}
    m.set_graph(True)
    print(v, round(e0.elapsed_time(e1) / 10, 3), "ms/step", json.dumps(r))
