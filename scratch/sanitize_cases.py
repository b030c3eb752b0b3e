"""Tiny invocations of the flag-barrier / persistent / peer kernels for compute-sanitizer
(memcheck, racecheck, synccheck): one case per argv[1]."""
import sys
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
import numpy as np, torch
from helpers import make_cell_case, run_gpu_cell

case = sys.argv[1]
if case == "rec_fused":        # K2 fused per step (1) and persistent (2), LSTM family
    p, inp, dY, dhT, dcT = make_cell_case("milstm", 3, 130, 64, 128, 5, bf16=True)
    for v in ("fwd=1", "fwd=2"):
        run_gpu_cell("milstm", p, inp, dY, dhT, dcT, "bf16", v)
elif case == "rec_persist":    # small-batch persistent forward (fwd=3)
    p, inp, dY, dhT, dcT = make_cell_case("milstm", 3, 16, 64, 128, 5, bf16=True)
    run_gpu_cell("milstm", p, inp, dY, dhT, dcT, "bf16", "fwd=3")
elif case == "bptt_fused":     # fused BPTT step (bwd=1)
    p, inp, dY, dhT, dcT = make_cell_case("lstm", 3, 130, 64, 128, 5, bf16=True)
    run_gpu_cell("lstm", p, inp, dY, dhT, dcT, "bf16", "bwd=1")
elif case == "rhn_fused":      # persistent RHN forward (fwd=1)
    p, inp, dY, dhT, dcT = make_cell_case("rhn", 2, 16, 64, 64, 5, bf16=True, L=2)
    run_gpu_cell("rhn", p, inp, dY, dhT, dcT, "bf16", "fwd=1", depth=2)
elif case == "bptt_persist":   # small-batch persistent BPTT (bwd=2: clusters of 4, needs 4 K chunks: H >= 2048)
    p, inp, dY, dhT, dcT = make_cell_case("milstm", 2, 16, 64, 2048, 5, bf16=True)
    run_gpu_cell("milstm", p, inp, dY, dhT, dcT, "bf16", "bwd=2")
elif case == "scrn_persist":   # SC-RNN persistent forward + BPTT (fwd=1, bwd=1)
    p, inp, dY, dhT, dcT = make_cell_case("scrn", 3, 16, 64, 128, 5, bf16=True, S=128)
    run_gpu_cell("scrn", p, inp, dY, dhT, dcT, "bf16", "fwd=1,bwd=1", context=128, scrn_alpha=0.95)
elif case == "gemm_kb":        # K1 with multi-k-block stages (K-major and MN-major, partial last stage)
    import paper_conf_asplos_sivathanucsz19_b200 as A
    for (M, N, K, amn, bmn, ks) in ((64, 256, 512, 0, 0, 1), (64, 256, 448, 0, 1, 1), (128, 128, 1792, 1, 1, 4)):
        a = (torch.randn(K, M) if amn else torch.randn(M, K)).cuda().to(torch.bfloat16)
        b = (torch.randn(K, N) if bmn else torch.randn(N, K)).cuda().to(torch.bfloat16)
        A.gemm_bf16_ex(a, b, M, N, K, a_mn=bool(amn), b_mn=bool(bmn), bn=64, ksplit=ks)
elif case == "rhn_bptt":       # persistent RHN BPTT (bwd=1: clusters of 4, R33 split of 4)
    p, inp, dY, dhT, dcT = make_cell_case("rhn", 2, 16, 64, 512, 5, bf16=True, L=2)   # Hp 512: split of 4
    run_gpu_cell("rhn", p, inp, dY, dhT, dcT, "bf16", "bwd=1", depth=2)
elif case == "bwd_pw3":        # TMA-tiled backward pointwise (bpw=2, LM mode: fp32 dY, 2-way split at H = 1024)
    import paper_conf_asplos_sivathanucsz19_b200 as A
    sys.path.insert(0, "/root/repo/tests")
    from test_gpu_lm import _lm_case
    import synth
    for H in (130, 1024):
        pa, tok, h0, c0 = _lm_case("milstm", 3, 40, 64, H, 64, synth.config_seed(5) + 31, True)
        c = A.Cell("milstm", H, 64, 40, 3, dtype="bf16")
        m = A.LM(c, 64)
        m.load(pa)
        c.tune_mode(A.TUNE_FROZEN, "bpw=2,gb=1" if H == 1024 else "bpw=2")
        m.train_step(torch.as_tensor(tok, dtype=torch.int32, device=c.device), 0.1)
elif case == "attn_dec_fused":  # attentive decoder's fused step: one-step persistent (B <= 128) and rec_fused (B > 128)
    import synth
    from test_gpu_cell import _attn_check
    from helpers import TOL_BF16
    for B in (37, 160):
        _attn_check(3, 3, B, 64, 128, 128, "bf16", synth.config_seed(4) + 7, TOL_BF16, variant="fwd=3")
elif case == "gate_blocked":   # gate-blocked layout (kperm GEMMs, per-gate a1, both pointwise forms)
    p, inp, dY, dhT, dcT = make_cell_case("milstm", 3, 72, 64, 1024, 5, bf16=True)
    for v in ("gb=1,gc=2", "gb=1,bpw=1,bptt=128.1.1.2"):
        run_gpu_cell("milstm", p, inp, dY, dhT, dcT, "bf16", v)
else:
    raise SystemExit(f"unknown case {case}")
torch.cuda.synchronize()
print("ok", case)
