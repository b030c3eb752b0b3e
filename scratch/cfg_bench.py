"""Full-size runs of BASELINE configs[1..3] (SC-RNN LM, RHN LM with exploration on, LSTM-attention
cell step): samples/s after the tuner converges.  Not the headline bench (that is cfg5)."""
import json, sys, time, torch
sys.path.insert(0, "/root/repo")
import numpy as np
import synth
import paper_conf_asplos_sivathanucsz19_b200 as A


def lm_run(name, cell, H, I, B, T, V, kw, steps=10):
    c = A.Cell(cell, H, I, B, T, dtype="bf16", **kw)
    m = A.LM(c, V)
    seed = 777
    shapes = {k: (r, cc) if r > 1 else (cc,) for k, (off, r, cc) in m.param_info.items()}
    p = synth.weights(seed, shapes, H, {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)})
    m.load(p)
    tok = torch.as_tensor(synth.zipf_tokens(seed, "tok", (T + 1, B), V, None), dtype=torch.int32).cuda()
    c.tune_mode(A.TUNE_ON)
    n = 0
    t0 = time.perf_counter()
    while True:
        m.train_step(tok, 0.01)
        n += 1
        if c.tune_next() == A.TUNE_CONVERGED or n > 1000:
            break
    torch.cuda.synchronize()
    tw = time.perf_counter() - t0
    rep = c.tune_report()
    c.tune_mode(A.TUNE_FROZEN, rep["variant"])
    for _ in range(3): m.train_step(tok, 0.01)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps): m.train_step(tok, 0.01)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    import bench
    c.set_profiling(2)   # phase regions for the diagnostic step
    m.set_graph(False)
    m.train_step(tok, 0.01); torch.cuda.synchronize()
    regions = {k: round(v, 3) for k, v in bench.region_times(c).items()}
    m.set_graph(True)
    print(json.dumps({"config": name, "samples_per_s": round(B / ms * 1e3, 1), "ms_per_step": round(ms, 3),
                      "regions_eager": regions, "loss": round(float(m.loss.item()), 4), "tuner_steps": n, "configs_explored": rep.get("configs_explored"),
                      "tuner_wall_s": round(tw, 2), "variant": rep["variant"]}), flush=True)


def attn_run(name, H, I, A_, B, Ts, Tt, steps=10):
    """cfg4: the LSTM-attention cell (encoder + attentive decoder) fwd + bwd + SGD per step through
    the cell ABI, exploration on until it converges."""
    c = A.Cell("attn", H, I, B, Tt, dtype="bf16", src_seq=Ts, attn_dim=A_)
    rng = np.random.default_rng(779)
    p = {k: (rng.uniform(-1, 1, (r, cc) if r > 1 else (cc,)) / np.sqrt(H)).astype(np.float32)
         for k, (off, r, cc) in c.param_info.items()}
    c.load(p)
    x = (torch.rand((Ts + Tt) * B * I, device="cuda") * 2 - 1).to(torch.bfloat16)
    y = torch.empty(Tt, B, 2 * H, dtype=torch.bfloat16, device="cuda")
    dY = (torch.randn(Tt, B, 2 * H, device="cuda") * 0.01).to(torch.bfloat16)
    h0, c0 = torch.zeros(B, H, device="cuda"), torch.zeros(B, H, device="cuda")
    dx = torch.empty((Ts + Tt) * B * I, dtype=torch.bfloat16, device="cuda")

    def step():
        c.forward(x, h0, c0, y, None, None)
        c.backward(dY, None, None, dx, None, None)
        c.sgd(0.01)

    import os
    n = 0
    if os.environ.get("CFG_VARIANT"):   # A/B runs: a forced variant, no exploration
        c.tune_mode(A.TUNE_FROZEN, os.environ["CFG_VARIANT"])
        rep = {"variant": os.environ["CFG_VARIANT"]}
    else:
        c.tune_mode(A.TUNE_ON)
        while True:
            step()
            n += 1
            if c.tune_next() == A.TUNE_CONVERGED or n > 1000:
                break
        rep = c.tune_report()
        c.tune_mode(A.TUNE_FROZEN, rep["variant"])
    for _ in range(3): step()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps): step()
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    import bench
    c.set_profiling(2)   # phase regions for the diagnostic step
    step(); torch.cuda.synchronize()
    regions = {k: round(v, 3) for k, v in bench.region_times(c).items()}
    print(json.dumps({"config": name, "samples_per_s": round(B / ms * 1e3, 1), "ms_per_step": round(ms, 3),
                      "regions": regions, "tuner_steps": n, "configs_explored": rep.get("configs_explored"), "variant": rep["variant"]}),
          flush=True)


which = sys.argv[1] if len(sys.argv) > 1 else "all"
if which in ("all", "cfg2"):
    lm_run("cfg2 SC-RNN word LM H=1024 B=64 T=35 V=10k", "scrn", 1024, 1024, 64, 35, 10000, {"context": 1024, "scrn_alpha": 0.95})
if which in ("all", "cfg3"):
    lm_run("cfg3 RHN depth 10 H=830 B=64 T=35 V=10k (exploration on)", "rhn", 830, 830, 64, 35, 10000, {"depth": 10})
if which in ("all", "cfg4"):
    attn_run("cfg4 LSTM-attention H=1024 B=128 Ts=Tt=50", 1024, 1024, 1024, 128, 50, 50)
