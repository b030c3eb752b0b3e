"""Stacked-layer LM (the paper's PTB stacked LSTM, Table 5) through
astra_lm_create_stacked: loss and every layer's gradients against the fp64 oracle; tuner exploration
on every layer stays value-preserving; graph replay is bitwise identical."""
import numpy as np
import pytest
import torch

import synth
from oracle import lm as OLM

from helpers import TOL_BF16, TOL_FP32, bf16_round, cell_shapes, rel_err

pytestmark = pytest.mark.gpu


def _case(cells, T, B, I, H, V, seed, bf16, L=2):
    ps, h0s, c0s = [], [], []
    n_in = I
    for l, cell in enumerate(cells):
        p = synth.weights(seed + l, cell_shapes(cell, n_in, H, H, L), H,
                          {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)})
        if bf16:
            for k in ("W", "U", "R"):
                if k in p:
                    p[k] = bf16_round(p[k])
        ps.append(p)
        h0s.append(synth.uniform(seed + l, "h0", (B, H), -0.5, 0.5))
        c0s.append(None if cell == "rhn" else synth.uniform(seed + l, "c0", (B, H), -0.5, 0.5))
        n_in = H
    plm = synth.weights(seed, {"E": (V, I), "W_o": (H, V), "b_o": (V,)}, H)
    if bf16:
        plm["E"] = bf16_round(plm["E"])
        plm["W_o"] = bf16_round(plm["W_o"])
    tok = synth.zipf_tokens(seed, "tok", (T + 1, B), V, V - 5)
    return ps, plm, tok, h0s, c0s


def _build(cells, T, B, I, H, V, dtype, ps, plm, L=2):
    import paper_conf_asplos_sivathanucsz19_b200 as A
    layers = []
    n_in = I
    for cell in cells:
        layers.append(A.Cell(cell, H, n_in, B, T, dtype=dtype, **({"depth": L} if cell == "rhn" else {})))
        n_in = H
    m = A.LM(layers, V)
    named = dict(plm)
    for l, p in enumerate(ps):
        named.update({f"L{l}.{k}": v for k, v in p.items()})
    m.load(named)
    return layers, m


@pytest.mark.parametrize("dtype,tol", [("fp32", TOL_FP32), ("bf16", TOL_BF16)])
@pytest.mark.parametrize("cells", [["lstm", "lstm"], ["milstm", "milstm", "milstm"], ["rhn", "rhn"], ["sublstm", "lstm"]])
def test_stacked_lm_matches_oracle(cells, dtype, tol):
    T, B, I, H, V = 5, 24, 64, 64, 60
    ps, plm, tok, h0s, c0s = _case(cells, T, B, I, H, V, synth.config_seed(5) + 60, dtype == "bf16")
    layers, m = _build(cells, T, B, I, H, V, dtype, ps, plm)
    dev = layers[0].device
    h = torch.as_tensor(np.concatenate([x.reshape(-1) for x in h0s]), dtype=torch.float32, device=dev)
    cs = [x for x in c0s if x is not None]
    c = torch.as_tensor(np.concatenate([x.reshape(-1) for x in cs]), dtype=torch.float32, device=dev) if cs else None
    m.set_state(h, c)
    loss = float(m.fwd_bwd(torch.as_tensor(tok, dtype=torch.int32, device=dev)).item())
    torch.cuda.synchronize()
    lo, gl, glm = OLM.stacked_lm_forward_backward(cells, ps, plm, tok, h0s, c0s)
    assert abs(loss - lo) / abs(lo) <= tol
    errs = {k: rel_err(m.view(k, m.grads).cpu().numpy().reshape(np.shape(glm[k])), glm[k]) for k in glm}
    for l, g in enumerate(gl):
        for k in g:
            errs[f"L{l}.{k}"] = rel_err(m.view(f"L{l}.{k}", m.grads).cpu().numpy().reshape(np.shape(g[k])), g[k])
    assert all(v <= tol for v in errs.values()), errs


def test_stacked_tuner_and_graph_bitwise():
    """Every layer exploring vs frozen at the default, and graph replay on/off: same bits."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H, V = 6, 128, 128, 128, 64
    cells = ["milstm", "milstm"]
    out = []
    for mode, graph in ((A.TUNE_OFF, True), (A.TUNE_ON, True), (A.TUNE_OFF, False)):
        ps, plm, tok, _, _ = _case(cells, T, B, I, H, V, synth.config_seed(5) + 61, True)
        layers, m = _build(cells, T, B, I, H, V, "bf16", ps, plm)
        m.set_graph(graph)
        for c in layers:
            c.tune_mode(mode)
        tokens = torch.as_tensor(tok, dtype=torch.int32, device=layers[0].device)
        for _ in range(12):
            m.train_step(tokens, 0.1)
            for c in layers:
                c.tune_next()
        torch.cuda.synchronize()
        out.append((m.params.clone(), float(m.loss.item())))
    for o in out[1:]:
        assert torch.equal(out[0][0], o[0]) and out[0][1] == o[1]


def test_stacked_shape_mismatch_rejected():
    import paper_conf_asplos_sivathanucsz19_b200 as A
    a = A.Cell("lstm", 64, 32, 8, 4)
    b = A.Cell("lstm", 64, 48, 8, 4)   # input 48 != 64
    with pytest.raises(A.AstraError):
        A.LM([a, b], 20)
    s = A.Cell("scrn", 64, 32, 8, 4, context=64)
    u = A.Cell("lstm", 64, 128, 8, 4)
    with pytest.raises(A.AstraError):
        A.LM([s, u], 20)   # SCRN's [h|s] output is two segments


@pytest.mark.parametrize("cells", [["milstm", "milstm"], ["lstm", "sublstm", "lstm"]])
@pytest.mark.parametrize("lwf", [1, 2])
def test_layer_wavefront_bitwise(cells, lwf):
    """The layer wavefront (AV lwf: layers on their own streams in 5 / T time chunks, chunked a1 and
    dX) gives the same bits as layers one after the other, over 4 SGD steps with graph replay."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H, V = 7, 64, 128, 128, 64
    out = []
    for v in (0, lwf):
        ps, plm, tok, _, _ = _case(cells, T, B, I, H, V, synth.config_seed(5) + 62, True)
        layers, m = _build(cells, T, B, I, H, V, "bf16", ps, plm)
        layers[-1].tune_mode(A.TUNE_FROZEN, f"lwf={v}")
        tokens = torch.as_tensor(tok, dtype=torch.int32, device=layers[0].device)
        for _ in range(4):
            m.train_step(tokens, 0.1)
        torch.cuda.synchronize()
        out.append((m.params.clone(), float(m.loss.item())))
    assert torch.equal(out[0][0], out[1][0]) and out[0][1] == out[1][1]


def test_layer_wavefront_matches_oracle():
    """lwf = per-step wavefront against the stacked fp64 oracle (fp32 path)."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    cells = ["milstm", "lstm"]
    T, B, I, H, V = 5, 24, 64, 64, 60
    ps, plm, tok, h0s, c0s = _case(cells, T, B, I, H, V, synth.config_seed(5) + 63, False)
    layers, m = _build(cells, T, B, I, H, V, "fp32", ps, plm)
    layers[-1].tune_mode(A.TUNE_FROZEN, "lwf=2")
    dev = layers[0].device
    m.set_state(torch.as_tensor(np.concatenate([x.reshape(-1) for x in h0s]), dtype=torch.float32, device=dev),
                torch.as_tensor(np.concatenate([x.reshape(-1) for x in c0s]), dtype=torch.float32, device=dev))
    loss = float(m.fwd_bwd(torch.as_tensor(tok, dtype=torch.int32, device=dev)).item())
    torch.cuda.synchronize()
    lo, gl, glm = OLM.stacked_lm_forward_backward(cells, ps, plm, tok, h0s, c0s)
    assert abs(loss - lo) / abs(lo) <= TOL_FP32
    for l, g in enumerate(gl):
        for k in g:
            e = rel_err(m.view(f"L{l}.{k}", m.grads).cpu().numpy().reshape(np.shape(g[k])), g[k])
            assert e <= TOL_FP32, (l, k, e)
