import sys, torch, numpy as np
sys.path.insert(0, "/root/repo")
import paper_conf_asplos_sivathanucsz19_b200 as A
H = I = A_ = 1024; B = 128; Ts = Tt = 50
c = A.Cell("attn", H, I, B, Tt, dtype="bf16", src_seq=Ts, attn_dim=A_)
rng = np.random.default_rng(779)
p = {k: (rng.uniform(-1, 1, (r, cc) if r > 1 else (cc,)) / np.sqrt(H)).astype(np.float32) for k, (off, r, cc) in c.param_info.items()}
c.load(p)
x = (torch.rand((Ts + Tt) * B * I, device="cuda") * 2 - 1).to(torch.bfloat16)
y = torch.empty(Tt, B, 2 * H, dtype=torch.bfloat16, device="cuda")
dY = (torch.randn(Tt, B, 2 * H, device="cuda") * 0.01).to(torch.bfloat16)
h0, c0 = torch.zeros(B, H, device="cuda"), torch.zeros(B, H, device="cuda")
dx = torch.empty((Ts + Tt) * B * I, dtype=torch.bfloat16, device="cuda")
if len(sys.argv) > 1:
    c.tune_mode(A.TUNE_FROZEN, sys.argv[1])
for _ in range(2):
    c.forward(x, h0, c0, y, None, None); c.backward(dY, None, None, dx, None, None); c.sgd(0.01)
torch.cuda.synchronize()
