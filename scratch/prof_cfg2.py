"""One cfg2 (SC-RNN LM) training step in a fixed variant, for an ncu launch list."""
import sys, torch
sys.path.insert(0, "/root/repo")
import synth
import paper_conf_asplos_sivathanucsz19_b200 as A
H, I, B, T, V = 1024, 1024, 64, 35, 10000
c = A.Cell("scrn", H, I, B, T, dtype="bf16", context=1024, scrn_alpha=0.95)
m = A.LM(c, V)
shapes = {k: (r, cc) if r > 1 else (cc,) for k, (off, r, cc) in m.param_info.items()}
m.load(synth.weights(777, shapes, H))
tok = torch.as_tensor(synth.zipf_tokens(777, "tok", (T + 1, B), V, None), dtype=torch.int32).cuda()
c.tune_mode(A.TUNE_FROZEN, sys.argv[1] if len(sys.argv) > 1 else
            "a1=128.1.1,rec=64.1.1,bptt=64.1.1,du=64.1.1,dw=64.1.1,dx=128.1.1,head=256.1.1.2,wg_side=0,fwd=1,bwd=1,pf=0,hov=1")
m.set_graph(False)
for _ in range(3): m.train_step(tok, 0.01)
torch.cuda.synchronize()
