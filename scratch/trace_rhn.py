"""Phase trace of the persistent fused RHN forward at cfg3 shapes (cell API, forward only)."""
import os, sys, numpy as np, torch
sys.path.insert(0, "/root/repo")
import synth
import paper_conf_asplos_sivathanucsz19_b200 as A
H, I, B, T, L = 830, 830, 64, 35, 10
c = A.Cell("rhn", H, I, B, T, dtype="bf16", depth=L)
shapes = {k: (r, cc) if r > 1 else (cc,) for k, (off, r, cc) in c.param_info.items()}
c.load(synth.weights(7, shapes, H))
c.tune_mode(A.TUNE_FROZEN, "fwd=1")
x = (torch.rand(T, B, I, device="cuda") * 2 - 1).to(torch.bfloat16)
y = torch.empty(T, B, H, dtype=torch.bfloat16, device="cuda")
Hp = 832; G = Hp // 32; N = T * L
tr = torch.zeros(G * N * 12, dtype=torch.int64, device="cuda")
for _ in range(2): c.forward(x, None, None, y)
torch.cuda.synchronize()
A._check(A.lib().astra_debug_set_trace(1, A._ptr(tr)))
c.forward(x, None, None, y)
torch.cuda.synchronize()
t = tr.cpu().numpy().reshape(G, N, 12).astype(np.float64) / 1e3   # us
q = np.arange(1, N)
flag = t[:, 1:, 0] - t[:, :-1, 4]            # own release -> flag observed for the next step
a_lat = t[:, :, 1] - t[:, :, 0]              # flag observed -> first A+B stage landed
kloop = t[:, :, 2] - t[:, :, 1]              # first -> last stage landed (MMA issue)
mma_tail = t[:, :, 3] - t[:, :, 2]           # last stage landed -> epilogue sees tfull
epi = t[:, :, 4] - t[:, :, 3]                # epilogue (incl. publish)
lastrel = t[:, :-1, 4].max(0)
prop = t[:, 1:, 0] - lastrel[None, :]        # last CTA's release -> this CTA sees the flag
step = np.diff(t[0, :, 0])
tm = t[:, :-1, :]
extra = [("epi: tfull->tmem chunk0", tm[:, :, 5] - tm[:, :, 3]), ("epi: chunk0 tmem -> loop end", tm[:, :, 6] - tm[:, :, 5]),
         ("epi: chunk0 compute", tm[:, :, 9] - tm[:, :, 5]), ("epi: chunk0 so stores", tm[:, :, 10] - tm[:, :, 9]),
         ("epi: chunk1 tmem", tm[:, :, 11] - tm[:, :, 10]), ("epi: chunk1 rest", tm[:, :, 6] - tm[:, :, 11]),
         ("epi: fence.proxy.async", tm[:, :, 7] - tm[:, :, 6]), ("epi: bar.sync", tm[:, :, 8] - tm[:, :, 7]),
         ("epi: red.release", tm[:, :, 4] - tm[:, :, 8])]
for name, v in extra:
    print(f"{name:32s} median {np.median(v):7.2f} us  p90 {np.percentile(v, 90):7.2f}")
for name, v in [("step", step), ("flag_wait_after_own_release", flag), ("propagation_after_last_release", prop),
                ("A_latency", a_lat), ("k_loop", kloop), ("mma_tail", mma_tail), ("epilogue+publish", epi)]:
    print(f"{name:32s} median {np.median(v):7.2f} us  p90 {np.percentile(v, 90):7.2f}")
