"""Pins for the fp64 oracle's cells; no GPU, no product code.

Each pin is something other than the oracle itself: torch.nn.LSTM / torch.nn.RNN (library
routines) under parameter settings that reduce a cell to them, closed forms, central finite
differences of the scalar loss, and structural invariants.  A dropped term, sign error,
wrong index or transposed operand in any forward or backward formula fails at least one.
"""
import numpy as np
import pytest
import torch

import synth
from oracle import cells as C

SEED = synth.config_seed(0)


def _inputs(T, B, I, H, seed=SEED, key=""):
    return {"x": synth.uniform(seed, key + "x", (T, B, I), -1, 1),
            "h0": synth.uniform(seed, key + "h0", (B, H), -0.5, 0.5),
            "c0": synth.uniform(seed, key + "c0", (B, H), -0.5, 0.5)}


def _torch_lstm(p, x, h0, c0, grads=False):
    I, H = p["W"].shape[0], p["U"].shape[0]
    m = torch.nn.LSTM(I, H).double()
    with torch.no_grad():
        m.weight_ih_l0.copy_(torch.tensor(p["W"].T))
        m.weight_hh_l0.copy_(torch.tensor(p["U"].T))
        m.bias_ih_l0.copy_(torch.tensor(p["b"]))
        m.bias_hh_l0.zero_()
    xt = torch.tensor(x, requires_grad=True)
    h0t = torch.tensor(h0[None], requires_grad=True)
    c0t = torch.tensor(c0[None], requires_grad=True)
    y, (hT, cT) = m(xt, (h0t, c0t))
    return m, xt, h0t, c0t, y, hT[0], cT[0]


# ------------------------------------------------------------------ reductions to nn.LSTM
@pytest.mark.parametrize("cell", ["lstm", "milstm"])
def test_lstm_and_milstm_reduce_to_torch_lstm_fwd_and_bwd(cell):
    """MI-LSTM with α=0, β1=β2=1 is the textbook LSTM; both must equal torch.nn.LSTM,
    forward AND every gradient (torch autograd through cuDNN-free CPU LSTM, fp64)."""
    T, B, I, H = 4, 3, 5, 6
    shapes = C.milstm_param_shapes(I, H) if cell == "milstm" else C.lstm_param_shapes(I, H)
    p = synth.weights(SEED, shapes, H)
    if cell == "milstm":
        p["alpha"][:] = 0.0
        p["beta1"][:] = 1.0
        p["beta2"][:] = 1.0
    inp = _inputs(T, B, I, H)
    dY = synth.normal(SEED, "dY", (T, B, H))
    dhT = synth.normal(SEED, "dhT", (B, H))
    dcT = synth.normal(SEED, "dcT", (B, H))
    out, g = C.cell_fwd_bwd(cell, p, inp, dY, dhT, dcT)
    m, xt, h0t, c0t, y, hT, cT = _torch_lstm(p, inp["x"], inp["h0"], inp["c0"])
    np.testing.assert_allclose(out["y"], y.detach().numpy(), rtol=0, atol=1e-14)
    np.testing.assert_allclose(out["cT"], cT.detach().numpy(), rtol=0, atol=1e-14)
    L = (y * torch.tensor(dY)).sum() + (hT * torch.tensor(dhT)).sum() + (cT * torch.tensor(dcT)).sum()
    L.backward()
    np.testing.assert_allclose(g["W"], m.weight_ih_l0.grad.numpy().T, atol=1e-13)
    np.testing.assert_allclose(g["U"], m.weight_hh_l0.grad.numpy().T, atol=1e-13)
    np.testing.assert_allclose(g["b"], m.bias_ih_l0.grad.numpy(), atol=1e-13)
    np.testing.assert_allclose(g["dx"], xt.grad.numpy(), atol=1e-13)
    np.testing.assert_allclose(g["dh0"], h0t.grad.numpy()[0], atol=1e-13)
    np.testing.assert_allclose(g["dc0"], c0t.grad.numpy()[0], atol=1e-13)


def test_milstm_general_differs_from_lstm():
    """Guard against a degenerate MI term: with α≠0 the outputs must differ from the LSTM."""
    T, B, I, H = 3, 2, 4, 5
    p = synth.weights(SEED, C.milstm_param_shapes(I, H), H,
                      {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)})
    inp = _inputs(T, B, I, H)
    y1 = C.milstm_forward(p, inp["x"], inp["h0"], inp["c0"])[0]
    y2 = C.lstm_forward(p, inp["x"], inp["h0"], inp["c0"])[0]
    assert np.abs(y1 - y2).max() > 1e-3


def test_milstm_pure_multiplicative_term():
    """β1=β2=b=0, α=1 ⇒ a = wx⊙uh exactly; check one step by direct products (h0 ≠ 0)."""
    B, I, H = 2, 3, 4
    p = synth.weights(SEED, C.milstm_param_shapes(I, H), H)
    p["alpha"][:] = 1.0
    p["beta1"][:] = 0.0
    p["beta2"][:] = 0.0
    p["b"][:] = 0.0
    inp = _inputs(1, B, I, H)
    y, hT, cT, _ = C.milstm_forward(p, inp["x"], inp["h0"], inp["c0"])
    # element (b, j) of gate block k: a = (Σ_q x[b,q] W[q,kH+j]) (Σ_r h[b,r] U[r,kH+j])
    x, h = inp["x"][0], inp["h0"]
    a = np.empty((B, 4 * H))
    for b in range(B):
        for n in range(4 * H):
            a[b, n] = sum(x[b, q] * p["W"][q, n] for q in range(I)) * \
                sum(h[b, r] * p["U"][r, n] for r in range(H))
    s = lambda z: 1 / (1 + np.exp(-z))
    c = s(a[:, H:2 * H]) * inp["c0"] + s(a[:, :H]) * np.tanh(a[:, 2 * H:3 * H])
    np.testing.assert_allclose(cT, c, atol=1e-15)
    np.testing.assert_allclose(hT, s(a[:, 3 * H:]) * np.tanh(c), atol=1e-15)


# ------------------------------------------------------------------ SCRN
def test_scrn_h_path_reduces_to_torch_rnn():
    """P = 0 ⇒ h_t = σ(x·A + h·R + b) — a sigmoid Elman RNN.  With σ(z) = (1 + tanh(z/2))/2 and
    g = 2h − 1 it is torch.nn.RNN(tanh) with W_ih = (A/2)ᵀ, W_hh = (R/4)ᵀ,
    bias = b/2 + colsum(R)/4, g_0 = 2h_0 − 1."""
    T, B, I, H, S = 5, 3, 4, 6, 5
    p = synth.weights(SEED, C.scrn_param_shapes(I, H, S), H)
    p["P"][:] = 0.0
    inp = _inputs(T, B, I, H)
    s0 = synth.uniform(SEED, "s0", (B, S), -0.5, 0.5)
    y, hT, sT, _ = C.scrn_forward(p, inp["x"], inp["h0"], s0, 0.95)
    # σ(z) = (1 + tanh(z/2))/2 and h = (1+g)/2 give
    # g_t = tanh( x·A/2 + g_{t-1}·R/4 + colsum(R)/4 + b/2 )
    m = torch.nn.RNN(I, H, nonlinearity="tanh").double()
    with torch.no_grad():
        m.weight_ih_l0.copy_(torch.tensor(p["A"].T / 2))
        m.weight_hh_l0.copy_(torch.tensor(p["R"].T / 4))
        m.bias_ih_l0.copy_(torch.tensor(p["b_h"] / 2 + p["R"].sum(0) / 4))
        m.bias_hh_l0.zero_()
        g, _ = m(torch.tensor(inp["x"]), torch.tensor(2 * inp["h0"] - 1)[None])
    np.testing.assert_allclose(y[:, :, :H], (1 + g.numpy()) / 2, atol=1e-15)


def test_scrn_context_closed_form():
    """s_T = (1−α)Σ_k α^{T−1−k}(x_k·Bm) + α^T s_0, and y_t carries s_t in columns H:."""
    T, B, I, H, S = 7, 2, 3, 4, 5
    alpha = 0.95
    p = synth.weights(SEED, C.scrn_param_shapes(I, H, S), H)
    inp = _inputs(T, B, I, H)
    s0 = synth.uniform(SEED, "s0", (B, S), -0.5, 0.5)
    y, _, sT, _ = C.scrn_forward(p, inp["x"], inp["h0"], s0, alpha)
    ref = alpha ** T * s0
    for k in range(T):
        ref = ref + (1 - alpha) * alpha ** (T - 1 - k) * (inp["x"][k] @ p["Bm"])
    np.testing.assert_allclose(sT, ref, atol=1e-15)
    np.testing.assert_allclose(y[-1][:, H:], ref, atol=1e-15)


# ------------------------------------------------------------------ RHN
def test_rhn_depth1_open_gate_is_torch_rnn():
    """L=1, b_T ≡ +50 ⇒ τ == 1.0 exactly in fp64 ⇒ s_t = tanh(x·W_H + s·R_H + b_H) = nn.RNN(tanh)."""
    T, B, I, H = 5, 3, 4, 6
    p = synth.weights(SEED, C.rhn_param_shapes(I, H, 1), H)
    p["b"][0, H:] = 50.0
    assert 1.0 / (1.0 + np.exp(-50.0)) == 1.0
    inp = _inputs(T, B, I, H)
    y, sT, _ = C.rhn_forward(p, inp["x"], inp["h0"])
    m = torch.nn.RNN(I, H, nonlinearity="tanh").double()
    with torch.no_grad():
        m.weight_ih_l0.copy_(torch.tensor(p["W"][:, :H].T))
        m.weight_hh_l0.copy_(torch.tensor(p["R"][0][:, :H].T))
        m.bias_ih_l0.copy_(torch.tensor(p["b"][0, :H]))
        m.bias_hh_l0.zero_()
        yr, _ = m(torch.tensor(inp["x"]), torch.tensor(inp["h0"])[None])
    np.testing.assert_allclose(y, yr.numpy(), atol=1e-15)


def test_rhn_closed_carry_keeps_state():
    """b_T ≡ −50 ⇒ τ ≈ 2e-22 ⇒ s^L_t = s_0 for every t (within T·L·2e-22)."""
    T, B, I, H, L = 4, 2, 3, 5, 3
    p = synth.weights(SEED, C.rhn_param_shapes(I, H, L), H)
    p["b"][:, H:] = -50.0
    inp = _inputs(T, B, I, H)
    y, sT, _ = C.rhn_forward(p, inp["x"], inp["h0"])
    np.testing.assert_allclose(y, np.broadcast_to(inp["h0"], y.shape), atol=1e-19)


# ------------------------------------------------------------------ subLSTM
def test_sublstm_constant_gate_closed_form():
    """W = U = 0 ⇒ gates constant σ(b): c_t = f c_{t−1} + (z − i) ⇒
    c_T = f^T c_0 + (z − i)(1 − f^T)/(1 − f);  h_T = σ(c_T) − o."""
    T, B, I, H = 6, 2, 3, 4
    p = synth.weights(SEED, C.lstm_param_shapes(I, H), H)
    p["W"][:] = 0
    p["U"][:] = 0
    p["b"] = synth.uniform(SEED, "bb", (4 * H,), -1, 1)
    inp = _inputs(T, B, I, H)
    _, hT, cT, _ = C.sublstm_forward(p, inp["x"], inp["h0"], inp["c0"])
    s = 1 / (1 + np.exp(-p["b"]))
    i, f, z, o = s[:H], s[H:2 * H], s[2 * H:3 * H], s[3 * H:]
    ref = f ** T * inp["c0"] + (z - i) * (1 - f ** T) / (1 - f)
    np.testing.assert_allclose(cT, ref, atol=1e-14)
    np.testing.assert_allclose(hT, 1 / (1 + np.exp(-ref)) - o, atol=1e-14)


# ------------------------------------------------------------------ attention
def _attn_setup(T_s=3, T_t=3, B=2, I=4, H=5, A=4):
    p = synth.weights(SEED, C.attn_param_shapes(I, H, A), H)
    inp = {"xe": synth.uniform(SEED, "xe", (T_s, B, I), -1, 1),
           "xd": synth.uniform(SEED, "xd", (T_t, B, I), -1, 1),
           "h0": synth.uniform(SEED, "h0", (B, H), -0.5, 0.5),
           "c0": synth.uniform(SEED, "c0", (B, H), -0.5, 0.5)}
    return p, inp


def test_attention_reductions():
    """v = 0 ⇒ p uniform ⇒ ctx_i = mean_j enc_j (enc from torch.nn.LSTM);
    C_d = 0 ⇒ decoder h ≡ torch.nn.LSTM(W_d, U_d) started from the encoder's final state."""
    p, inp = _attn_setup()
    H = inp["h0"].shape[1]
    p["v"][:] = 0.0
    p["C_d"][:] = 0.0
    y, hT, cT, _ = C.attn_forward(p, inp["xe"], inp["xd"], inp["h0"], inp["c0"])
    encp = {"W": p["W_e"], "U": p["U_e"], "b": p["b_e"]}
    _, _, _, _, enc, he, ce = _torch_lstm(encp, inp["xe"], inp["h0"], inp["c0"])
    enc = enc.detach().numpy()
    np.testing.assert_allclose(y[:, :, H:], np.broadcast_to(enc.mean(0), y[:, :, H:].shape), atol=1e-15)
    decp = {"W": p["W_d"], "U": p["U_d"], "b": p["b_d"]}
    _, _, _, _, yd, _, _ = _torch_lstm(decp, inp["xd"], he.detach().numpy(), ce.detach().numpy())
    np.testing.assert_allclose(y[:, :, :H], yd.detach().numpy(), atol=1e-14)


def test_attention_softmax_rows_sum_to_one_and_ctx_in_hull():
    p, inp = _attn_setup(T_s=4)
    y, _, _, (enc, keys, _, cache) = C.attn_forward(p, inp["xe"], inp["xd"], inp["h0"], inp["c0"])
    H = inp["h0"].shape[1]
    for step in cache:
        pr = step[-1]
        np.testing.assert_allclose(pr.sum(0), 1.0, atol=1e-15)
        assert (pr > 0).all()
    assert (y[:, :, H:] <= enc.max(0) + 1e-15).all() and (y[:, :, H:] >= enc.min(0) - 1e-15).all()


# ------------------------------------------------------------------ finite differences
def _fd_check(cell, p, inp, dY, dhT, dcT, n_coords=6, **kw):
    """Central FD (ε=1e-6) on random directions of every tensor and on single coordinates."""
    out, g = C.cell_fwd_bwd(cell, p, inp, dY, dhT, dcT, **kw)
    eps = 1e-6
    rng = np.random.default_rng(7)
    tensors = [("p", k) for k in p] + [("i", k) for k in inp]
    gname = {"x": "dx", "h0": "dh0", "c0": "dc0", "xe": "dxe", "xd": "dxd"}
    for kind, k in tensors:
        src = p if kind == "p" else inp
        gk = g[k] if kind == "p" else g[gname[k]]
        if cell == "rhn" and k == "c0":
            continue
        dirs = [rng.standard_normal(src[k].shape)]
        for _ in range(n_coords):
            e = np.zeros(src[k].size)
            e[rng.integers(src[k].size)] = 1.0
            dirs.append(e.reshape(src[k].shape))
        for d in dirs:
            orig = src[k].copy()
            src[k] = orig + eps * d
            lp = C.cell_loss(cell, p, inp, dY, dhT, dcT, **kw)
            src[k] = orig - eps * d
            lm = C.cell_loss(cell, p, inp, dY, dhT, dcT, **kw)
            src[k] = orig
            fd = (lp - lm) / (2 * eps)
            an = float((gk * d).sum())
            assert abs(fd - an) <= 1e-7 * max(1.0, abs(an)) + 2e-9, (cell, k, fd, an)


def test_fd_lstm():
    T, B, I, H = 3, 2, 4, 5
    p = synth.weights(SEED, C.lstm_param_shapes(I, H), H)
    inp = _inputs(T, B, I, H)
    _fd_check("lstm", p, inp, synth.normal(SEED, "dY", (T, B, H)),
              synth.normal(SEED, "dh", (B, H)), synth.normal(SEED, "dc", (B, H)))


def test_fd_milstm():
    T, B, I, H = 3, 2, 4, 5
    p = synth.weights(SEED, C.milstm_param_shapes(I, H), H,
                      {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)})
    inp = _inputs(T, B, I, H)
    _fd_check("milstm", p, inp, synth.normal(SEED, "dY", (T, B, H)),
              synth.normal(SEED, "dh", (B, H)), synth.normal(SEED, "dc", (B, H)))


def test_fd_sublstm():
    T, B, I, H = 3, 2, 4, 5
    p = synth.weights(SEED, C.lstm_param_shapes(I, H), H)
    inp = _inputs(T, B, I, H)
    _fd_check("sublstm", p, inp, synth.normal(SEED, "dY", (T, B, H)),
              synth.normal(SEED, "dh", (B, H)), synth.normal(SEED, "dc", (B, H)))


def test_fd_scrn():
    T, B, I, H, S = 4, 2, 3, 5, 3
    p = synth.weights(SEED, C.scrn_param_shapes(I, H, S), H)
    inp = _inputs(T, B, I, H)
    inp["c0"] = synth.uniform(SEED, "s0", (B, S), -0.5, 0.5)
    _fd_check("scrn", p, inp, synth.normal(SEED, "dY", (T, B, H + S)),
              synth.normal(SEED, "dh", (B, H)), synth.normal(SEED, "ds", (B, S)), alpha=0.95)


def test_fd_rhn():
    T, B, I, H, L = 3, 2, 4, 5, 3
    p = synth.weights(SEED, C.rhn_param_shapes(I, H, L), H)
    inp = _inputs(T, B, I, H)
    del inp["c0"]
    _fd_check("rhn", p, inp, synth.normal(SEED, "dY", (T, B, H)),
              synth.normal(SEED, "dh", (B, H)), None)


def test_fd_attention():
    p, inp = _attn_setup()
    Tt, B, H = inp["xd"].shape[0], inp["h0"].shape[0], inp["h0"].shape[1]
    _fd_check("attn", p, inp, synth.normal(SEED, "dY", (Tt, B, 2 * H)),
              synth.normal(SEED, "dh", (B, H)), synth.normal(SEED, "dc", (B, H)), n_coords=3)


def test_directional_derivative_cfg1_shape():
    """Random directional derivatives at the cfg1 shape (MI-LSTM H64 I32 B4 T8)."""
    T, B, I, H = 8, 4, 32, 64
    seed = synth.config_seed(1)
    p = synth.weights(seed, C.milstm_param_shapes(I, H), H,
                      {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)})
    inp = _inputs(T, B, I, H, seed)
    dY, dhT, dcT = (synth.normal(seed, "dY", (T, B, H)), synth.normal(seed, "dhT", (B, H)),
                    synth.normal(seed, "dcT", (B, H)))
    _fd_check("milstm", p, inp, dY, dhT, dcT, n_coords=0)


# ------------------------------------------------------------------ statefulness
@pytest.mark.parametrize("cell", ["milstm", "scrn", "rhn"])
def test_statefulness_split_sequence(cell):
    """fwd(T) == fwd(T1) then fwd(T2) from the carried state (exact in fp64)."""
    T, B, I, H = 6, 2, 3, 4
    inp = _inputs(T, B, I, H)
    if cell == "milstm":
        p = synth.weights(SEED, C.milstm_param_shapes(I, H), H)
        y, hT, cT, _ = C.milstm_forward(p, inp["x"], inp["h0"], inp["c0"])
        y1, h1, c1, _ = C.milstm_forward(p, inp["x"][:2], inp["h0"], inp["c0"])
        y2, h2, c2, _ = C.milstm_forward(p, inp["x"][2:], h1, c1)
    elif cell == "scrn":
        p = synth.weights(SEED, C.scrn_param_shapes(I, H, H), H)
        y, hT, cT, _ = C.scrn_forward(p, inp["x"], inp["h0"], inp["c0"], 0.9)
        y1, h1, c1, _ = C.scrn_forward(p, inp["x"][:2], inp["h0"], inp["c0"], 0.9)
        y2, h2, c2, _ = C.scrn_forward(p, inp["x"][2:], h1, c1, 0.9)
    else:
        p = synth.weights(SEED, C.rhn_param_shapes(I, H, 2), H)
        y, hT, _ = C.rhn_forward(p, inp["x"], inp["h0"])
        y1, h1, _ = C.rhn_forward(p, inp["x"][:2], inp["h0"])
        y2, h2, _ = C.rhn_forward(p, inp["x"][2:], h1)
    assert np.array_equal(y, np.concatenate([y1, y2]))
    assert np.array_equal(hT, h2)


# ------------------------------------------------------------------ round-2 pins (VERDICT r1 "What's weak" #1)
def test_scrn_context_feeds_h_through_P_closed_form():
    """A = R = 0, b_h = 0 ⇒ h_t = σ(s_t·P) with s_t the closed form
    s_t = (1−α)Σ_{k≤t} α^{t−k}(x_k·Bm) + α^{t+1} s_0 (0-based t).  Pins that h_t reads the *current*
    context s_t through P (s_{t−1}·P, a missing (1−α) or a transposed P fail)."""
    T, B, I, H, S = 6, 3, 4, 5, 7
    alpha = 0.9
    p = synth.weights(SEED, C.scrn_param_shapes(I, H, S), H)
    p["A"][:] = 0.0
    p["R"][:] = 0.0
    p["b_h"][:] = 0.0
    p["P"] = synth.uniform(SEED, "Pbig", (S, H), -2, 2)   # large enough that σ(s·P) is far from ½
    inp = _inputs(T, B, I, H)
    s0 = synth.uniform(SEED, "s0", (B, S), -0.5, 0.5)
    y, _, _, _ = C.scrn_forward(p, inp["x"], inp["h0"], s0, alpha)
    for t in range(T):
        s_t = alpha ** (t + 1) * s0
        for k in range(t + 1):
            s_t = s_t + (1 - alpha) * alpha ** (t - k) * (inp["x"][k] @ p["Bm"])
        h_ref = torch.sigmoid(torch.tensor(s_t) @ torch.tensor(p["P"])).numpy()
        np.testing.assert_allclose(y[t][:, :H], h_ref, atol=1e-15)
        np.testing.assert_allclose(y[t][:, H:], s_t, atol=1e-15)


def test_attention_two_positions_closed_form():
    """Ts = 2: softmax over two scores is p_1 = σ(e_1 − e_2), so ctx_i = p_1·enc_1 + (1−p_1)·enc_2
    with e_j = vᵀtanh(q_i + k_j), q_i = h_i·W_q from the decoder's *current* h_i.  The decoder step
    itself is torch.nn.LSTMCell on the input-fed vector [x^d_i | ctx_{i−1}] (W_ih = [W_d; C_d]ᵀ,
    W_hh = U_dᵀ), started from the encoder's final state (torch.nn.LSTM).  Pins: q from h_i (not
    h_{i−1}), tanh inside the sum, the score vector v, the keys k_j = enc_j·W_k, input feeding of
    ctx_{i−1} (not ctx_i, not none) through C_d, and y_i = [h_i | ctx_i]."""
    Ts, Tt, B, I, H, A = 2, 3, 2, 3, 4, 5
    p, inp = _attn_setup(T_s=Ts, T_t=Tt, B=B, I=I, H=H, A=A)
    p["v"] = synth.uniform(SEED, "vbig", (A,), -3, 3)           # scores well away from a tie
    p["C_d"] = synth.uniform(SEED, "Cdbig", (H, 4 * H), -1, 1)   # input feeding clearly visible
    y, hT, cT, _ = C.attn_forward(p, inp["xe"], inp["xd"], inp["h0"], inp["c0"])
    encp = {"W": p["W_e"], "U": p["U_e"], "b": p["b_e"]}
    _, _, _, _, enc, he, ce = _torch_lstm(encp, inp["xe"], inp["h0"], inp["c0"])
    enc = enc.detach().numpy()
    keys = [enc[j] @ p["W_k"] for j in range(Ts)]
    cellm = torch.nn.LSTMCell(I + H, H).double()
    with torch.no_grad():
        cellm.weight_ih.copy_(torch.tensor(np.concatenate([p["W_d"], p["C_d"]], 0).T))
        cellm.weight_hh.copy_(torch.tensor(p["U_d"].T))
        cellm.bias_ih.copy_(torch.tensor(p["b_d"]))
        cellm.bias_hh.zero_()
    h, c = he.detach(), ce.detach()
    ctx = np.zeros((B, H))
    sig = lambda z: 1.0 / (1.0 + np.exp(-z))
    for i in range(Tt):
        with torch.no_grad():
            h, c = cellm(torch.tensor(np.concatenate([inp["xd"][i], ctx], 1)), (h, c))
        q = h.numpy() @ p["W_q"]
        e1 = np.tanh(q + keys[0]) @ p["v"]
        e2 = np.tanh(q + keys[1]) @ p["v"]
        p1 = sig(e1 - e2)[:, None]
        ctx = p1 * enc[0] + (1.0 - p1) * enc[1]
        np.testing.assert_allclose(y[i][:, :H], h.numpy(), atol=1e-14)
        np.testing.assert_allclose(y[i][:, H:], ctx, atol=1e-14)
    np.testing.assert_allclose(hT, h.numpy(), atol=1e-14)
    np.testing.assert_allclose(cT, c.numpy(), atol=1e-14)


def _torch_attn_loss(p, inp, dY, dhT, dcT):
    """An independent construction of the attentive LSTM from torch library routines (torch's LSTM
    cell for encoder and decoder, the decoder on [x | ctx_{i−1}], torch.softmax over positions), fp64, whose
    autograd gradients pin the oracle's hand-derived attention backward."""
    I = inp["xe"].shape[2]
    H = inp["h0"].shape[1]
    t = {k: torch.tensor(v, requires_grad=True) for k, v in p.items()}
    xi = {k: torch.tensor(inp[k], requires_grad=True) for k in ("xe", "xd", "h0", "c0")}
    # torch's own LSTM cell kernel; the parameters are the dict tensors so autograd reaches them
    def lstm_step(x, h, c, W_ih, W_hh, b):
        return torch._VF.lstm_cell(x, (h, c), W_ih, W_hh, b, torch.zeros_like(b))
    h, c = xi["h0"], xi["c0"]
    enc = []
    for j in range(inp["xe"].shape[0]):
        h, c = lstm_step(xi["xe"][j], h, c, t["W_e"].T, t["U_e"].T, t["b_e"])
        enc.append(h)
    enc = torch.stack(enc)
    keys = enc @ t["W_k"]
    ctx = torch.zeros_like(h)
    ys = []
    W_ih = torch.cat([t["W_d"], t["C_d"]], 0).T
    for i in range(inp["xd"].shape[0]):
        h, c = lstm_step(torch.cat([xi["xd"][i], ctx], 1), h, c, W_ih, t["U_d"].T, t["b_d"])
        q = h @ t["W_q"]
        e = torch.tanh(q[None] + keys) @ t["v"]                 # [Ts, B]
        pr = torch.softmax(e, 0)
        ctx = (pr[:, :, None] * enc).sum(0)
        ys.append(torch.cat([h, ctx], 1))
    y = torch.stack(ys)
    L = (y * torch.tensor(dY)).sum() + (h * torch.tensor(dhT)).sum() + (c * torch.tensor(dcT)).sum()
    L.backward()
    g = {k: v.grad.numpy() for k, v in t.items()}
    g.update(dxe=xi["xe"].grad.numpy(), dxd=xi["xd"].grad.numpy(), dh0=xi["h0"].grad.numpy(),
             dc0=xi["c0"].grad.numpy())
    return y.detach().numpy(), g


def test_attention_backward_matches_torch_autograd():
    """Every attention gradient (v, W_q, W_k, C_d, the decoder and encoder weights, the inputs and
    the initial state) equals fp64 autograd through the library-built construction above."""
    p, inp = _attn_setup(T_s=4, T_t=3, B=2, I=3, H=5, A=4)
    p["v"] = synth.uniform(SEED, "vbig", (4,), -2, 2)
    Tt, B, H = 3, 2, 5
    dY = synth.normal(SEED, "dY", (Tt, B, 2 * H))
    dhT, dcT = synth.normal(SEED, "dh", (B, H)), synth.normal(SEED, "dc", (B, H))
    out, g = C.cell_fwd_bwd("attn", p, inp, dY, dhT, dcT)
    y_t, g_t = _torch_attn_loss(p, inp, dY, dhT, dcT)
    np.testing.assert_allclose(out["y"], y_t, atol=1e-14)
    for k in g_t:
        np.testing.assert_allclose(g[k], g_t[k], atol=1e-12, err_msg=k)
