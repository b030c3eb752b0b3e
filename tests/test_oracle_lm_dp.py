"""Pins for the oracle's LM head / cross-entropy / embedding / SGD / DP.

No GPU, no product code.  Library pins: torch.nn.functional.cross_entropy and autograd in
fp64; central finite differences of the whole LM loss; DP linearity (mean of shard gradients
equals the full-batch gradient).
"""
import numpy as np
import pytest
import torch

import synth
from oracle import cells as C
from oracle import dp, lm

SEED = synth.config_seed(0) + 7


def test_cross_entropy_matches_torch():
    logits = synth.normal(SEED, "lg", (37, 11), 3.0)
    tgt = synth.zipf_tokens(SEED, "tg", (37,), 11)
    loss, d = lm.cross_entropy(logits, tgt)
    lt = torch.tensor(logits, requires_grad=True)
    ref = torch.nn.functional.cross_entropy(lt, torch.tensor(tgt, dtype=torch.long))
    ref.backward()
    assert abs(loss - ref.item()) < 1e-14
    np.testing.assert_allclose(d, lt.grad.numpy(), atol=1e-16)


def _lm_setup(cell, T=3, B=4, I=5, H=6, V=9, S=4, L=2):
    if cell == "milstm":
        shapes = C.milstm_param_shapes(I, H)
        Hout = H
    elif cell == "scrn":
        shapes = C.scrn_param_shapes(I, H, S)
        Hout = H + S
    else:
        shapes = C.rhn_param_shapes(I, H, L)
        Hout = H
    shapes.update(lm.head_param_shapes(Hout, V))
    shapes["E"] = (V, I)
    p = synth.weights(SEED, shapes, H, {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)})
    tok = synth.zipf_tokens(SEED, "tok", (T + 1, B), V, n_symbols=V - 2)
    h0 = synth.uniform(SEED, "h0", (B, H), -0.5, 0.5)
    c0 = synth.uniform(SEED, "c0", (B, S if cell == "scrn" else H), -0.5, 0.5) if cell != "rhn" else None
    return p, tok, h0, c0


@pytest.mark.parametrize("cell", ["milstm", "scrn", "rhn"])
def test_lm_fd(cell):
    """Central FD of the mean-CE loss w.r.t. every parameter, including the embedding E
    (which checks the scatter-add embedding backward and repeated tokens)."""
    kw = {"alpha": 0.9} if cell == "scrn" else {}
    p, tok, h0, c0 = _lm_setup(cell)
    loss, g, _ = lm.lm_forward_backward(cell, p, tok, h0, c0, **kw)
    assert len(np.unique(tok[:-1])) < tok[:-1].size   # repeated tokens exercise the segment sum
    rng = np.random.default_rng(3)
    eps = 1e-6
    for k in p:
        for trial in range(3):
            d = rng.standard_normal(p[k].shape)
            orig = p[k].copy()
            p[k] = orig + eps * d
            lp = lm.lm_forward_backward(cell, p, tok, h0, c0, **kw)[0]
            p[k] = orig - eps * d
            lmn = lm.lm_forward_backward(cell, p, tok, h0, c0, **kw)[0]
            p[k] = orig
            fd = (lp - lmn) / (2 * eps)
            an = float((g[k] * d).sum())
            assert abs(fd - an) <= 1e-7 * max(1.0, abs(an)) + 1e-10, (k, fd, an)


def test_lm_head_matches_torch_autograd():
    """logits/CE/dW_o/db_o/dY of the head against torch autograd in fp64."""
    T, B, H, V = 3, 4, 6, 9
    y = synth.uniform(SEED, "y", (T * B, H), -1, 1)
    W = synth.uniform(SEED, "W", (H, V), -0.4, 0.4)
    b = synth.uniform(SEED, "b", (V,), -0.4, 0.4)
    tgt = synth.zipf_tokens(SEED, "t", (T * B,), V)
    logits = y @ W + b
    loss, dl = lm.cross_entropy(logits, tgt)
    yt, Wt, bt = (torch.tensor(a, requires_grad=True) for a in (y, W, b))
    ref = torch.nn.functional.cross_entropy(yt @ Wt + bt, torch.tensor(tgt, dtype=torch.long))
    ref.backward()
    np.testing.assert_allclose(y.T @ dl, Wt.grad.numpy(), atol=1e-15)
    np.testing.assert_allclose(dl.sum(0), bt.grad.numpy(), atol=1e-15)
    np.testing.assert_allclose(dl @ W.T, yt.grad.numpy(), atol=1e-15)


def test_sgd_step():
    p = {"a": np.array([1.0, -2.0]), "b": np.array([3.0])}
    g = {"a": np.array([0.5, 0.25])}
    q = lm.sgd(p, g, 0.1)
    assert np.array_equal(q["a"], np.array([1.0 - 0.05, -2.0 - 0.025])) and np.array_equal(q["b"], p["b"])


def test_sgd_decreases_loss():
    cell = "milstm"
    p, tok, h0, c0 = _lm_setup(cell)
    l0, p1, _, _ = lm.lm_train_step(cell, p, tok, h0, c0, 0.05)
    l1 = lm.lm_forward_backward(cell, p1, tok, h0, c0)[0]
    assert l1 < l0


@pytest.mark.parametrize("N", [2, 4])
def test_dp_linearity(N):
    """(1/N)Σ_r g_r over contiguous batch-column shards == full-batch mean gradient."""
    cell = "milstm"
    p, tok, h0, c0 = _lm_setup(cell, B=8)
    loss, g, _ = lm.lm_forward_backward(cell, p, tok, h0, c0)
    ldp, gdp = dp.dp_gradients(cell, p, tok, h0, c0, N)
    assert abs(loss - ldp) < 1e-13
    for k in g:
        np.testing.assert_allclose(gdp[k], g[k], atol=1e-13)


def _stack_setup(cells, T=3, B=4, I=5, H=6, V=9, L=2):
    ps, h0s, c0s = [], [], []
    n_in = I
    for l, cell in enumerate(cells):
        if cell in ("lstm", "milstm"):
            shapes = C.milstm_param_shapes(n_in, H) if cell == "milstm" else C.lstm_param_shapes(n_in, H)
        else:
            shapes = C.rhn_param_shapes(n_in, H, L)
        ps.append(synth.weights(SEED + l, shapes, H, {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)}))
        h0s.append(synth.uniform(SEED + l, "h0", (B, H), -0.5, 0.5))
        c0s.append(synth.uniform(SEED + l, "c0", (B, H), -0.5, 0.5) if cell != "rhn" else None)
        n_in = H
    plm = synth.weights(SEED, {"E": (V, I), **lm.head_param_shapes(H, V)}, H)
    tok = synth.zipf_tokens(SEED, "tok", (T + 1, B), V, n_symbols=V - 2)
    return ps, plm, tok, h0s, c0s


def test_stacked_lstm_lm_matches_torch():
    """Two stacked LSTM layers + head + mean CE == torch.nn.LSTM(num_layers=2) + Linear +
    cross_entropy with autograd (fp64): loss and every gradient (W_ih = Wᵀ, W_hh = Uᵀ, b_hh = 0)."""
    T, B, I, H, V = 4, 3, 5, 6, 9
    ps, plm, tok, h0s, c0s = _stack_setup(["lstm", "lstm"], T, B, I, H, V)
    loss, gl, glm = lm.stacked_lm_forward_backward(["lstm", "lstm"], ps, plm, tok, h0s, c0s)
    net = torch.nn.LSTM(I, H, num_layers=2).double()
    with torch.no_grad():
        for l in range(2):
            getattr(net, f"weight_ih_l{l}").copy_(torch.tensor(ps[l]["W"].T))
            getattr(net, f"weight_hh_l{l}").copy_(torch.tensor(ps[l]["U"].T))
            getattr(net, f"bias_ih_l{l}").copy_(torch.tensor(ps[l]["b"]))
            getattr(net, f"bias_hh_l{l}").zero_()
    E = torch.tensor(plm["E"], requires_grad=True)
    Wo = torch.tensor(plm["W_o"], requires_grad=True)
    bo = torch.tensor(plm["b_o"], requires_grad=True)
    x = E[torch.tensor(tok[:T], dtype=torch.long)]
    h0 = torch.tensor(np.stack(h0s))
    c0 = torch.tensor(np.stack(c0s))
    y, _ = net(x, (h0, c0))
    ref = torch.nn.functional.cross_entropy(y.reshape(T * B, H) @ Wo + bo,
                                            torch.tensor(tok[1:].reshape(-1), dtype=torch.long))
    ref.backward()
    assert abs(loss - ref.item()) < 1e-13
    np.testing.assert_allclose(glm["E"], E.grad.numpy(), atol=1e-14)
    np.testing.assert_allclose(glm["W_o"], Wo.grad.numpy(), atol=1e-14)
    for l in range(2):
        np.testing.assert_allclose(gl[l]["W"], getattr(net, f"weight_ih_l{l}").grad.numpy().T, atol=1e-14)
        np.testing.assert_allclose(gl[l]["U"], getattr(net, f"weight_hh_l{l}").grad.numpy().T, atol=1e-14)
        np.testing.assert_allclose(gl[l]["b"], getattr(net, f"bias_ih_l{l}").grad.numpy(), atol=1e-14)


@pytest.mark.parametrize("cells", [["milstm", "milstm"], ["rhn", "rhn", "rhn"]])
def test_stacked_lm_fd(cells):
    """Central FD of the stacked LM loss in random directions, every layer's parameters and E."""
    ps, plm, tok, h0s, c0s = _stack_setup(cells)
    loss, gl, glm = lm.stacked_lm_forward_backward(cells, ps, plm, tok, h0s, c0s)
    rng = np.random.default_rng(5)
    eps = 1e-6
    targets = [(ps[l], k, gl[l][k]) for l in range(len(cells)) for k in ps[l]] + [(plm, "E", glm["E"])]
    for p, k, g in targets:
        d = rng.standard_normal(p[k].shape)
        orig = p[k].copy()
        p[k] = orig + eps * d
        lp = lm.stacked_lm_forward_backward(cells, ps, plm, tok, h0s, c0s)[0]
        p[k] = orig - eps * d
        lmn = lm.stacked_lm_forward_backward(cells, ps, plm, tok, h0s, c0s)[0]
        p[k] = orig
        fd = (lp - lmn) / (2 * eps)
        an = float((g * d).sum())
        assert abs(fd - an) <= 1e-7 * max(1.0, abs(an)) + 1e-10, (k, fd, an)
