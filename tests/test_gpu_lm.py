"""LM training-step parity (embedding → cell → head → mean CE → backward → SGD) against the fp64
oracle, through the C ABI; tuner exploration is value-preserving (same loss/params tuner on/off)."""
import numpy as np
import pytest
import torch

import synth
from oracle import lm as OLM

from helpers import TOL_BF16, TOL_FP32, bf16_round, cell_shapes, rel_err

pytestmark = pytest.mark.gpu


ALPHA = 0.95
S_CTX, L_DEPTH = 24, 2


def _lm_case(cell, T, B, I, H, V, seed, bf16, n_symbols=None):
    shapes = cell_shapes(cell, I, H, S_CTX, L_DEPTH)
    Hout = H + S_CTX if cell == "scrn" else H
    shapes.update({"E": (V, I), "W_o": (Hout, V), "b_o": (V,)})
    p = synth.weights(seed, shapes, H, {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)})
    if bf16:
        for k in ("W", "U", "A", "Bm", "P", "R", "E", "W_o"):
            if k in p:
                p[k] = bf16_round(p[k])
    tok = synth.zipf_tokens(seed, "tok", (T + 1, B), V, n_symbols)
    h0 = synth.uniform(seed, "h0", (B, H), -0.5, 0.5)
    c0 = None if cell == "rhn" else synth.uniform(seed, "c0", (B, S_CTX if cell == "scrn" else H), -0.5, 0.5)
    return p, tok, h0, c0


def _cell_kw(cell):
    if cell == "scrn":
        return {"context": S_CTX, "scrn_alpha": ALPHA}, {"alpha": np.float32(ALPHA).item()}
    if cell == "rhn":
        return {"depth": L_DEPTH}, {}
    return {}, {}


def _run(cell, T, B, I, H, V, dtype, seed, n_symbols=None, lr=0.0):
    import paper_conf_asplos_sivathanucsz19_b200 as A
    p, tok, h0, c0 = _lm_case(cell, T, B, I, H, V, seed, dtype == "bf16", n_symbols)
    c = A.Cell(cell, H, I, B, T, dtype=dtype, **_cell_kw(cell)[0])
    m = A.LM(c, V)
    m.load(p)
    dev = c.device
    f32 = lambda a: None if a is None else torch.as_tensor(np.asarray(a, dtype=np.float32), device=dev)
    m.set_state(f32(h0), f32(c0))
    tokens = torch.as_tensor(tok, dtype=torch.int32, device=dev)
    loss = m.fwd_bwd(tokens)
    torch.cuda.synchronize()
    g = {k: m.view(k, m.grads).cpu().numpy().reshape(np.shape(p[k])) for k in p}
    return p, tok, h0, c0, float(loss.item()), g, m


@pytest.mark.parametrize("dtype,tol", [("fp32", TOL_FP32), ("bf16", TOL_BF16)])
@pytest.mark.parametrize("cell", ["milstm", "lstm", "sublstm", "scrn", "rhn"])
def test_lm_grads(cell, dtype, tol):
    T, B, I, H, V = 6, 8, 64, 64, 50
    p, tok, h0, c0, loss, g, _ = _run(cell, T, B, I, H, V, dtype, synth.config_seed(5) + 3, n_symbols=40)
    lo, go, _ = OLM.lm_forward_backward(cell, p, tok, h0, c0, **_cell_kw(cell)[1])
    assert abs(loss - lo) / abs(lo) <= tol
    errs = {k: rel_err(g[k], go[k]) for k in go}
    bad = {k: v for k, v in errs.items() if not v <= tol}
    assert not bad, (bad, errs)


def test_lm_cfg5_shape_reduced_bf16():
    """cfg5 shapes (H=I=2048, V=256 over 205 Zipf symbols), per-GPU batch 64, T=4."""
    T, B, I, H, V = 4, 64, 2048, 2048, 256
    p, tok, h0, c0, loss, g, _ = _run("milstm", T, B, I, H, V, "bf16", synth.config_seed(5), n_symbols=205)
    lo, go, _ = OLM.lm_forward_backward("milstm", p, tok, h0, c0)
    assert abs(loss - lo) / abs(lo) <= TOL_BF16
    errs = {k: rel_err(g[k], go[k]) for k in go}
    assert all(v <= TOL_BF16 for v in errs.values()), errs


@pytest.mark.parametrize("cell,T,B,I,H,V", [("scrn", 4, 64, 1024, 1024, 10000), ("rhn", 3, 64, 830, 830, 10000)])
def test_lm_cfg2_cfg3_shapes_reduced_bf16(cell, T, B, I, H, V):
    """cfg2 (SCRN, H=S=1024, V=10k) and cfg3 (RHN L=10 → 2 here, H=830, V=10k) shapes, short T."""
    global S_CTX
    old = S_CTX
    S_CTX = H if cell == "scrn" else S_CTX
    try:
        p, tok, h0, c0, loss, g, _ = _run(cell, T, B, I, H, V, "bf16", synth.config_seed(2), n_symbols=None)
        lo, go, _ = OLM.lm_forward_backward(cell, p, tok, h0, c0, **_cell_kw(cell)[1])
    finally:
        S_CTX = old
    assert abs(loss - lo) / abs(lo) <= TOL_BF16
    errs = {k: rel_err(g[k], go[k]) for k in go}
    assert all(v <= TOL_BF16 for v in errs.values()), errs


def test_lm_sgd_and_tuner_value_preserving():
    """20 SGD steps with the tuner exploring vs frozen at the default: bitwise-identical params."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H, V = 6, 128, 128, 128, 64
    seed = synth.config_seed(5) + 9
    results = []
    for mode in (A.TUNE_OFF, A.TUNE_ON):
        p, tok, h0, c0 = _lm_case("milstm", T, B, I, H, V, seed, True)
        c = A.Cell("milstm", H, I, B, T, dtype="bf16")
        m = A.LM(c, V)
        m.load(p)
        c.tune_mode(mode)
        tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
        for _ in range(20):
            m.train_step(tokens, 0.1)
            c.tune_next()
        torch.cuda.synchronize()
        results.append((m.params.clone(), float(m.loss.item()), c.tune_report()))
    assert torch.equal(results[0][0], results[1][0])
    assert results[0][1] == results[1][1]
    assert results[1][2]["configs_explored"] >= 2


def _steps_params(variant, graph, steps=8):
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H, V = 5, 300, 128, 192, 64
    p, tok, h0, c0 = _lm_case("milstm", T, B, I, H, V, synth.config_seed(5) + 12, True)
    c = A.Cell("milstm", H, I, B, T, dtype="bf16")
    m = A.LM(c, V)
    m.load(p)
    m.set_graph(graph)
    c.tune_mode(A.TUNE_FROZEN, variant)
    tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
    for _ in range(steps):
        m.train_step(tokens, 0.1)
    torch.cuda.synchronize()
    return m.params.clone(), float(m.loss.item())


@pytest.mark.parametrize("variant", ["fwd=0", "a1=256.1.1.2,rec=256.1.1.2,bptt=128.1.1.2,du=256.1.1.2,dw=128.1.1.2,"
                                     "dx=256.1.1.2,head=256.1.1.2,wg_side=1,fwd=1",
                                     "fwd=0,hov=1,wgs=2,gc=3,wg_side=1", "gb=1,gc=2,hov=1,bpw=1"])
def test_graph_replay_bitwise(variant):
    """CUDA-graph replay of frozen steps (the bench path) is bitwise identical to kernel-by-kernel
    enqueueing, over 8 SGD steps (state carried between steps)."""
    pa, la = _steps_params(variant, graph=True)
    pb, lb = _steps_params(variant, graph=False)
    assert torch.equal(pa, pb) and la == lb


def test_pdl_off_bitwise(tmp_path):
    """Programmatic dependent launch changes only scheduling: ASTRA_PDL=0 gives the same bits."""
    import os
    import subprocess
    import sys
    code = ("import sys, numpy as np, torch; sys.path.insert(0, 'tests'); import test_gpu_lm as t; "
            "p, l = t._steps_params('fwd=1', True, 4); np.save(sys.argv[1], p.cpu().numpy())")
    outs = []
    for pdl in ("1", "0"):
        f = str(tmp_path / f"p{pdl}.npy")
        env = dict(os.environ, ASTRA_PDL=pdl)
        subprocess.run([sys.executable, "-c", code, f], check=True, env=env, cwd=os.path.dirname(os.path.dirname(__file__)))
        outs.append(np.load(f))
    assert np.array_equal(outs[0], outs[1])


@pytest.mark.parametrize("cell", ["milstm", "scrn", "rhn"])
@pytest.mark.parametrize("hov", [1, 2])
def test_head_overlap_bitwise(cell, hov):
    """The LM head in 2 / 5 time chunks on a side stream, overlapping the forward and BPTT chains
    (AV head_ov), gives the same bits as the sequential head over 4 SGD steps (graph replay)."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H, V = 7, 64, 64, 64, 300
    out = []
    for v in (0, hov):
        p, tok, h0, c0 = _lm_case(cell, T, B, I, H, V, synth.config_seed(5) + 40, True)
        c = A.Cell(cell, H, I, B, T, dtype="bf16", **_cell_kw(cell)[0])
        m = A.LM(c, V)
        m.load(p)
        c.tune_mode(A.TUNE_FROZEN, f"hov={v}")
        tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
        for _ in range(4):
            m.train_step(tokens, 0.1)
        torch.cuda.synchronize()
        out.append((m.params.clone(), float(m.loss.item())))
    assert torch.equal(out[0][0], out[1][0]) and out[0][1] == out[1][1]


def test_head_overlap_switch_on_one_lm_bitwise():
    """One LM switches head_ov 0 → 1 → 2 → 1 (as the tuner does while exploring): each step's loss
    and gradients equal the sequential head's bit for bit.  Guards the prepared-GEMM cache: the
    2-chunk and 5-chunk head GEMMs cover different row ranges and must never share an entry."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H, V = 10, 64, 64, 64, 300
    p, tok, h0, c0 = _lm_case("milstm", T, B, I, H, V, synth.config_seed(5) + 41, True)
    c = A.Cell("milstm", H, I, B, T, dtype="bf16")
    m = A.LM(c, V)
    m.load(p)
    tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
    dev = c.device
    out = []
    for v in (0, 1, 2, 1, 0):
        c.tune_mode(A.TUNE_FROZEN, f"hov={v}")
        m.set_state(torch.zeros(B, H, device=dev), torch.zeros(B, H, device=dev))
        loss = m.fwd_bwd(tokens)
        torch.cuda.synchronize()
        out.append((m.grads.clone(), float(loss.item())))
    for g, l in out[1:]:
        assert torch.equal(g, out[0][0]) and l == out[0][1]


@pytest.mark.parametrize("cell,H", [("milstm", 192), ("milstm", 2048), ("lstm", 256)])
def test_fused_bptt_lm_bitwise(cell, H):
    """LM steps with the fused BPTT kernel (bwd=1, the LM's fp32 dY streamed by TMA) give the same
    bits as GEMM + unfused pointwise (bwd=0) over 3 SGD steps; H = 2048 uses the 4-way split-K."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, V = 4, 96, 128, 64
    out = []
    for v in ("bwd=0", "bwd=1"):
        p, tok, h0, c0 = _lm_case(cell, T, B, I, H, V, synth.config_seed(5) + 50, True)
        c = A.Cell(cell, H, I, B, T, dtype="bf16")
        m = A.LM(c, V)
        m.load(p)
        c.tune_mode(A.TUNE_FROZEN, v)
        tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
        for _ in range(3):
            m.train_step(tokens, 0.1)
        torch.cuda.synchronize()
        out.append((m.params.clone(), float(m.loss.item())))
    assert torch.equal(out[0][0], out[1][0]) and out[0][1] == out[1][1]


def test_profiling_switch():
    """Region events off changes no value (graph re-captured) and is refused while exploring."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    out = []
    for prof in (True, False):
        pa, tok, h0, c0 = _lm_case("milstm", 5, 64, 64, 64, 50, synth.config_seed(5) + 70, True)
        c = A.Cell("milstm", 64, 64, 64, 5, dtype="bf16")
        m = A.LM(c, 50)
        m.load(pa)
        c.tune_mode(A.TUNE_FROZEN, "fwd=0")
        c.set_profiling(prof)
        tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
        for _ in range(3):
            m.train_step(tokens, 0.1)
        torch.cuda.synchronize()
        out.append(m.params.clone())
        c.tune_mode(A.TUNE_ON)
        with pytest.raises(A.AstraError):
            c.set_profiling(False)
    assert torch.equal(out[0], out[1])


@pytest.mark.parametrize("variant", ["rc=1", "rc=1,fwd=1", "rc=1,fwd=2", "rc=1,bwd=1", "rc=1,wg_side=1,hov=1",
                                     "gb=1", "gb=1,rc=1,gc=2,wgs=1"])
def test_recompute_lm_bitwise(variant, monkeypatch):
    """SURVEY §8(f) rank 4, the alloc fork: recomputing UH_t = h_{t-1}·U in BPTT (ring of 2-step
    chunks on a side stream, 3 chunks at T = 5 so the ring wraps) gives the same bits as storing it,
    over 8 SGD steps, with every forward / backward fusion choice and under graph replay."""
    monkeypatch.setenv("ASTRA_RC_STEPS", "2")
    pa, la = _steps_params("fwd=0", graph=True)
    pb, lb = _steps_params(variant, graph=True)
    assert torch.equal(pa, pb) and la == lb
    if variant == "rc=1":
        pc, lc = _steps_params(variant, graph=False)
        assert torch.equal(pa, pc) and la == lc


def test_tuner_fork_explores_both_allocation_contexts():
    """The live update tree's root is the hierarchical alloc fork: all four contexts are
    explored and raced end to end; the run stays bitwise equal to the default."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H, V = 4, 64, 64, 64, 40
    res = []
    n_steps = 1500
    for mode in (A.TUNE_ON, A.TUNE_OFF):
        p, tok, h0, c0 = _lm_case("milstm", T, B, I, H, V, synth.config_seed(5) + 60, True)
        c = A.Cell("milstm", H, I, B, T, dtype="bf16")
        m = A.LM(c, V)
        m.load(p)
        c.tune_mode(mode)
        tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
        seen = set()
        for i in range(n_steps):
            m.train_step(tokens, 0.05)
            vr = c.tune_report()["variant"]
            seen.add(("rc=1" in vr, "gb=1" in vr))
            if c.tune_next() == A.TUNE_CONVERGED:
                n_steps = i + 1
                break
        torch.cuda.synchronize()
        res.append((m.params.clone(), seen))
    assert n_steps < 1500, "the tuner did not converge"
    assert torch.equal(res[0][0], res[1][0])
    # the four allocation contexts: store / recompute UH × gate-interleaved / gate-blocked layout
    assert res[0][1] == {(False, False), (True, False), (False, True), (True, True)}, res[0][1]


@pytest.mark.parametrize("hov", [0, 1])
def test_rhn_fused_forward_lm_bitwise(hov):
    """RHN LM steps with the persistent fused forward chain (fwd=1) give the same bits as the
    per-micro-step launches (fwd=0), with and without the head overlapping the chain, over 4 SGD
    steps (state carried between steps, graph replay)."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H, V = 5, 64, 128, 192, 300
    out = []
    for v in ("fwd=0", "fwd=1"):
        p, tok, h0, c0 = _lm_case("rhn", T, B, I, H, V, synth.config_seed(3) + 30, True)
        c = A.Cell("rhn", H, I, B, T, dtype="bf16", depth=L_DEPTH)
        m = A.LM(c, V)
        m.load(p)
        c.tune_mode(A.TUNE_FROZEN, f"{v},hov={hov}")
        tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
        for _ in range(4):
            m.train_step(tokens, 0.1)
        torch.cuda.synchronize()
        out.append((m.params.clone(), float(m.loss.item())))
    assert torch.equal(out[0][0], out[1][0]) and out[0][1] == out[1][1]


def test_rhn_wg_side_lm_bitwise():
    """RHN weight gradients with the L dR_ℓ GEMMs alternating between the main and a side stream
    (wg_side=1, overlapping dW / dX) give the same bits as all on the main stream, over 4 SGD steps."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H, V = 5, 64, 128, 192, 300
    out = []
    for v in ("wg_side=0", "wg_side=1"):
        p, tok, h0, c0 = _lm_case("rhn", T, B, I, H, V, synth.config_seed(3) + 31, True)
        c = A.Cell("rhn", H, I, B, T, dtype="bf16", depth=L_DEPTH)
        m = A.LM(c, V)
        m.load(p)
        c.tune_mode(A.TUNE_FROZEN, v)
        tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
        for _ in range(4):
            m.train_step(tokens, 0.1)
        torch.cuda.synchronize()
        out.append((m.params.clone(), float(m.loss.item())))
    assert torch.equal(out[0][0], out[1][0]) and out[0][1] == out[1][1]


def test_profiling_levels():
    """The always-on profiling level records the step region every step and the phase
    regions only while the tuner needs them; level 2 records every phase region (diagnostics);
    neither changes a value (the step graph is re-captured per level)."""
    import ctypes
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H, V = 5, 64, 64, 64, 50

    def regions(c):
        buf = (ctypes.c_double * 16)()
        n = ctypes.c_int()
        A._check(A.lib().astra_region_times(c.h, buf, 16, ctypes.byref(n)))
        return [buf[i] for i in range(n.value)]

    out = []
    for lvl in (1, 2, 0):
        pa, tok, h0, c0 = _lm_case("milstm", T, B, I, H, V, synth.config_seed(5) + 71, True)
        c = A.Cell("milstm", H, I, B, T, dtype="bf16")
        m = A.LM(c, V)
        m.load(pa)
        c.tune_mode(A.TUNE_FROZEN, "fwd=0")
        c.set_profiling(lvl)
        tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
        for _ in range(3):
            m.train_step(tokens, 0.1)
        torch.cuda.synchronize()
        out.append(m.params.clone())
        if lvl:
            r = regions(c)
            step = r[8]   # R_STEP
            phases = [r[0], r[1], r[3]]   # a1, forward chain, BPTT chain
            assert step > 0, r
            assert all(x > 0 for x in phases) if lvl == 2 else all(x == 0 for x in phases), (lvl, r)
    assert torch.equal(out[0], out[1]) and torch.equal(out[0], out[2])
    with pytest.raises(A.AstraError):
        c.set_profiling(3)


def test_tuner_final_race(monkeypatch):
    """Reading R41: after the wirer converges, the chain-form AVs' alternatives (here every one: the
    margin widened to 1000 %) are re-measured interleaved with the converged configuration, 5
    rounds of warm-up + measured step each; the report names the candidates, their min step times
    and the winner, the run converges, and the parameters equal an untuned run's after as many SGD
    steps (every variant is value-preserving)."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    monkeypatch.setenv("ASTRA_TUNE_RACE_MARGIN", "10")
    T, B, I, H, V = 4, 64, 64, 64, 40

    def lm():
        p, tok, h0, c0 = _lm_case("milstm", T, B, I, H, V, synth.config_seed(5) + 61, True)
        c = A.Cell("milstm", H, I, B, T, dtype="bf16")
        m = A.LM(c, V)
        m.load(p)
        return c, m, torch.as_tensor(tok, dtype=torch.int32, device=c.device)

    c, m, tokens = lm()
    c.tune_mode(A.TUNE_ON)
    n, state = 0, A.TUNE_EXPLORING
    while state != A.TUNE_CONVERGED and n < 1500:
        m.train_step(tokens, 0.05)
        n += 1
        state = c.tune_next()
    m.train_step(tokens, 0.05)
    torch.cuda.synchronize()
    rep = c.tune_report()
    assert state == A.TUNE_CONVERGED and "race" in rep, rep.keys()
    race = rep["race"]
    assert len(race["candidates"]) >= 2 and 0 <= race["winner"] < len(race["candidates"]), race
    assert all(0 < x["t_step_min"] < 1e29 for x in race["candidates"]), race
    c2, m2, tokens2 = lm()
    for _ in range(n + 1):
        m2.train_step(tokens2, 0.05)
    torch.cuda.synchronize()
    assert torch.equal(m.params, m2.params)


def test_tune_next_never_blocks():
    """astra_tune_next harvests the measured steps' events with cudaEventQuery (include/astra.h):
    right after it returns, the step just enqueued is still running on the GPU — the host keeps
    pipelining exploring steps — and the exploration still converges."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H, V = 50, 128, 2048, 2048, 256
    p, tok, h0, c0 = _lm_case("milstm", T, B, I, H, V, synth.config_seed(5) + 60, True, n_symbols=205)
    c = A.Cell("milstm", H, I, B, T, dtype="bf16")
    m = A.LM(c, V)
    m.load(p)
    tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
    st = torch.cuda.current_stream()
    c.tune_mode(A.TUNE_ON)
    busy, n, state = 0, 0, A.TUNE_EXPLORING
    while state != A.TUNE_CONVERGED and n < 1500:
        m.train_step(tokens, 0.01)
        state = c.tune_next()
        n += 1
        if 2 <= n <= 41:
            busy += not st.query()
    torch.cuda.synchronize()
    assert state == A.TUNE_CONVERGED, n
    assert busy >= 36, busy      # the GPU was still working after ≥ 90 % of the calls
    rep = c.tune_report()
    assert rep["configs_explored"] >= 10 and rep["converged"]


@pytest.mark.parametrize("cell", ["milstm", "lstm", "sublstm"])
@pytest.mark.parametrize("T,B,H", [(4, 300, 192), (3, 512, 2048), (5, 40, 130), (4, 64, 1024)])
def test_bwd_pointwise_tiled_lm_bitwise(cell, T, B, H, monkeypatch):
    """The TMA-tiled backward pointwise form (bwd_pw = 2: operand tiles landed in shared memory, the
    older ones before the grid dependency) gives the row-lane and wide forms' bits over 3 LM SGD
    steps (graph replay) — ragged row chunks (B = 300, 40), padding units (H = 130), the R25 4-way
    split at cfg5's H = 2048 and the 2-way split at H = 1024, the gate-blocked layout too.  ASTRA_BPW2_STRICT makes a fallback to the
    wide form an error, so the tiled kernel really ran at every step but the first."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    monkeypatch.setenv("ASTRA_BPW2_STRICT", "1")
    V = 64
    out = {}
    for v in ("bpw=0", "bpw=1", "bpw=2", "bpw=2,gb=1"):
        p, tok, h0, c0 = _lm_case(cell, T, B, 64, H, V, synth.config_seed(5) + 31, True)
        c = A.Cell(cell, H, 64, B, T, dtype="bf16")
        m = A.LM(c, V)
        m.load(p)
        m.set_graph(True)
        c.tune_mode(A.TUNE_FROZEN, v)
        tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
        for _ in range(3):
            m.train_step(tokens, 0.1)
        torch.cuda.synchronize()
        out[v] = (m.params.clone(), float(m.loss.item()))
    for v in out:
        assert torch.equal(out[v][0], out["bpw=0"][0]) and out[v][1] == out["bpw=0"][1], v


@pytest.mark.parametrize("variant", ["hov=1,wgs=2,gc=3,wg_side=1", "wgs=1,gc=4,fwd=3", "gc=2,wgs=2,rc=1",
                                     "rsp=1,bpw=1,gc=3", "hdy=128.1.1.2,head=128.1.1", "hdy=64.2.1"])
def test_stream_schedules_lm_bitwise(variant):
    """The stream-assignment variants together — head overlap, wgrad_schedule's dX chunks during
    BPTT, gate_chunking's projection GEMMs on two streams, the small-batch persistent forward —
    give the default variant's parameters bit for bit after 8 SGD steps (CUDA-graph replay)."""
    pa, la = _steps_params("fwd=0", graph=True)
    pb, lb = _steps_params(variant, graph=True)
    assert torch.equal(pa, pb) and la == lb


@pytest.mark.parametrize("T,B,V,nsym,I", [(100, 512, 256, 205, 64), (35, 64, 10000, None, 64), (7, 33, 50, 3, 64),
                                         (9, 40, 50, 5, 30)])
def test_embedding_backward_counting_sort(T, B, V, nsym, I):
    """The embedding backward's hand-written stable counting sort + ordered segment sums (R5) against
    the oracle's dE[v] = Σ_{(t,b): tok = v} dx[t,b] on the fp32 path (1e-4, element-wise): the cfg5
    token statistics (hot Zipf symbols, segments of many 64-row pieces), a 10k vocabulary (mostly
    empty rows, which must be exactly zero), a 3-symbol batch, and an embedding width that is not a
    multiple of 4 (the scalar column path) with a vocabulary that is not either (the scalar CE)."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    H = 64
    tok = synth.zipf_tokens(7, "tok", (T + 1, B), V, nsym)
    shapes = cell_shapes("lstm", I, H)
    shapes.update({"E": (V, I), "W_o": (H, V), "b_o": (V,)})
    p = synth.weights(7, shapes, H)
    c = A.Cell("lstm", H, I, B, T, dtype="fp32")
    m = A.LM(c, V)
    m.load(p)
    tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
    m.fwd_bwd(tokens)
    torch.cuda.synchronize()
    dE = m.view("E", m.grads).cpu().numpy()
    _, go, _ = OLM.lm_forward_backward("lstm", p, tok, np.zeros((B, H)), np.zeros((B, H)))
    used = np.zeros(V, bool)
    used[tok[:T].reshape(-1)] = True
    assert np.all(dE[~used] == 0.0), "tokens absent from the batch must get exactly zero"
    assert rel_err(dE[used], go["E"][used]) <= TOL_FP32
