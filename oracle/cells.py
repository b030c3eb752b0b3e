"""fp64 oracle: recurrent cells, forward and hand-derived backward through time.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  Conventions (SURVEY.md §8 top):
time-major [T, B, ·]; row vectors, y = x·W with W stored [in, out]; gate order (i, f, g, o)
as in PyTorch.  Cell-level loss L = Σ dY⊙Y + Σ dhT⊙hT + Σ dcT⊙cT (DESIGN reading R12), so the
backward functions take the upstream gradients (dY, dhT, dcT) and return the gradient of L
with respect to every parameter, the inputs and the initial state.

The paper only names and cites the cells ("MI-LSTM [36], LSTM with Attention
[35], SC-RNN [22], RHN [39]"; P:352 evaluated models; references P:489, P:504, P:517, P:521,
P:527).  Every definition below is the reading recorded in DESIGN.md §Readings, taken from
the cited work.
"""
from __future__ import annotations

import numpy as np


def sigmoid(x):
    return 1.0 / (1.0 + np.exp(-x))


# --------------------------------------------------------------------------------------
# LSTM (textbook; the reduction base).  PAPER.md P:352 "Stacked LSTM"; P:92 cuDNN LSTM.
# --------------------------------------------------------------------------------------
LSTM_PARAMS = ("W", "U", "b")


def lstm_param_shapes(I, H):
    return {"W": (I, 4 * H), "U": (H, 4 * H), "b": (4 * H,)}


def _lstm_gates(a, H):
    i = sigmoid(a[:, 0:H])
    f = sigmoid(a[:, H:2 * H])
    g = np.tanh(a[:, 2 * H:3 * H])
    o = sigmoid(a[:, 3 * H:4 * H])
    return i, f, g, o


def lstm_forward(p, x, h0, c0):
    """a = x_t·W + h_{t-1}·U + b; i,f,o = σ, g = tanh; c_t = f⊙c + i⊙g; h_t = o⊙tanh(c_t)."""
    T, B, _ = x.shape
    H = h0.shape[1]
    h, c = h0.copy(), c0.copy()
    ys, cache = [], []
    for t in range(T):
        a = x[t] @ p["W"] + h @ p["U"] + p["b"]
        i, f, g, o = _lstm_gates(a, H)
        c_new = f * c + i * g
        h_new = o * np.tanh(c_new)
        cache.append((h, c, i, f, g, o, c_new))
        h, c = h_new, c_new
        ys.append(h)
    return np.stack(ys), h, c, cache


def _lstm_cell_bwd(dh, dc, c_prev, i, f, g, o, c_new):
    """Backward of one LSTM cell update given dL/dh_t (dh) and dL/dc_t (dc, from t+1)."""
    tau = np.tanh(c_new)
    do = dh * tau
    dc = dc + dh * o * (1.0 - tau * tau)
    di = dc * g
    dg = dc * i
    df = dc * c_prev
    dc_prev = dc * f
    da = np.concatenate(
        [di * i * (1 - i), df * f * (1 - f), dg * (1 - g * g), do * o * (1 - o)], axis=1)
    return da, dc_prev


def lstm_backward(p, x, cache, dY, dhT, dcT):
    T = x.shape[0]
    grads = {k: np.zeros_like(v) for k, v in p.items() if k in LSTM_PARAMS}
    dx = np.zeros_like(x)
    dh_rec, dc = dhT.copy(), dcT.copy()
    for t in reversed(range(T)):
        h_prev, c_prev, i, f, g, o, c_new = cache[t]
        dh = dY[t] + dh_rec
        da, dc = _lstm_cell_bwd(dh, dc, c_prev, i, f, g, o, c_new)
        grads["W"] += x[t].T @ da
        grads["U"] += h_prev.T @ da
        grads["b"] += da.sum(0)
        dx[t] = da @ p["W"].T
        dh_rec = da @ p["U"].T
    return grads, dx, dh_rec, dc


# --------------------------------------------------------------------------------------
# MI-LSTM, multiplicative integration [36] (evaluated P:303-314).
# --------------------------------------------------------------------------------------
MILSTM_PARAMS = ("W", "U", "b", "alpha", "beta1", "beta2")


def milstm_param_shapes(I, H):
    s = lstm_param_shapes(I, H)
    s.update({"alpha": (4 * H,), "beta1": (4 * H,), "beta2": (4 * H,)})
    return s


def milstm_forward(p, x, h0, c0):
    """[36]'s general MI form: a = α⊙wx⊙uh + β1⊙uh + β2⊙wx + b, wx = x_t·W, uh = h_{t-1}·U.

    Reading R3: β1 scales U·h and β2 scales W·x; R4: one bias per gate.  Rest as LSTM.
    """
    T, B, _ = x.shape
    H = h0.shape[1]
    h, c = h0.copy(), c0.copy()
    ys, cache = [], []
    for t in range(T):
        wx = x[t] @ p["W"]
        uh = h @ p["U"]
        a = p["alpha"] * wx * uh + p["beta1"] * uh + p["beta2"] * wx + p["b"]
        i, f, g, o = _lstm_gates(a, H)
        c_new = f * c + i * g
        h_new = o * np.tanh(c_new)
        cache.append((h, c, wx, uh, i, f, g, o, c_new))
        h, c = h_new, c_new
        ys.append(h)
    return np.stack(ys), h, c, cache


def milstm_backward(p, x, cache, dY, dhT, dcT):
    """da as LSTM; d_uh = da⊙(α⊙wx + β1); d_wx = da⊙(α⊙uh + β2); dh_rec = d_uh·Uᵀ."""
    T = x.shape[0]
    grads = {k: np.zeros_like(p[k]) for k in MILSTM_PARAMS}
    dx = np.zeros_like(x)
    dh_rec, dc = dhT.copy(), dcT.copy()
    for t in reversed(range(T)):
        h_prev, c_prev, wx, uh, i, f, g, o, c_new = cache[t]
        dh = dY[t] + dh_rec
        da, dc = _lstm_cell_bwd(dh, dc, c_prev, i, f, g, o, c_new)
        d_uh = da * (p["alpha"] * wx + p["beta1"])
        d_wx = da * (p["alpha"] * uh + p["beta2"])
        grads["alpha"] += (da * wx * uh).sum(0)
        grads["beta1"] += (da * uh).sum(0)
        grads["beta2"] += (da * wx).sum(0)
        grads["b"] += da.sum(0)
        grads["U"] += h_prev.T @ d_uh
        grads["W"] += x[t].T @ d_wx
        dx[t] = d_wx @ p["W"].T
        dh_rec = d_uh @ p["U"].T
    return grads, dx, dh_rec, dc


# --------------------------------------------------------------------------------------
# subLSTM [8] (Table 4).  SURVEY §8(f) NEXT #1.
# --------------------------------------------------------------------------------------
def sublstm_forward(p, x, h0, c0):
    """All gates σ: [i, f, z, o] = σ(a); c_t = f⊙c_{t-1} + z − i; h_t = σ(c_t) − o."""
    T, B, _ = x.shape
    H = h0.shape[1]
    h, c = h0.copy(), c0.copy()
    ys, cache = [], []
    for t in range(T):
        a = x[t] @ p["W"] + h @ p["U"] + p["b"]
        s = sigmoid(a)
        i, f, z, o = s[:, :H], s[:, H:2 * H], s[:, 2 * H:3 * H], s[:, 3 * H:]
        c_new = f * c + z - i
        h_new = sigmoid(c_new) - o
        cache.append((h, c, i, f, z, o, c_new))
        h, c = h_new, c_new
        ys.append(h)
    return np.stack(ys), h, c, cache


def sublstm_backward(p, x, cache, dY, dhT, dcT):
    T = x.shape[0]
    grads = {k: np.zeros_like(p[k]) for k in LSTM_PARAMS}
    dx = np.zeros_like(x)
    dh_rec, dc = dhT.copy(), dcT.copy()
    for t in reversed(range(T)):
        h_prev, c_prev, i, f, z, o, c_new = cache[t]
        dh = dY[t] + dh_rec
        sc = sigmoid(c_new)
        dc = dc + dh * sc * (1 - sc)
        do = -dh
        di = -dc
        dz = dc
        df = dc * c_prev
        dc_prev = dc * f
        da = np.concatenate([di * i * (1 - i), df * f * (1 - f), dz * z * (1 - z), do * o * (1 - o)], 1)
        dc = dc_prev
        grads["W"] += x[t].T @ da
        grads["U"] += h_prev.T @ da
        grads["b"] += da.sum(0)
        dx[t] = da @ p["W"].T
        dh_rec = da @ p["U"].T
    return grads, dx, dh_rec, dc


# --------------------------------------------------------------------------------------
# SC-RNN / SCRN [22] (Fig. 1, Table 2).
# --------------------------------------------------------------------------------------
SCRN_PARAMS = ("A", "Bm", "P", "R", "b_h")


def scrn_param_shapes(I, H, S):
    return {"A": (I, H), "Bm": (I, S), "P": (S, H), "R": (H, H), "b_h": (H,)}


def scrn_forward(p, x, h0, s0, alpha):
    """s_t = (1−α)(x_t·Bm) + α s_{t−1};  h_t = σ(x_t·A + s_t·P + h_{t−1}·R + b_h);  y_t = [h_t|s_t].

    Readings R5 (fixed scalar α, default 0.95), R6 (S = H default), R7 (b_h present),
    R8 (dense input x = embedding output).  The context state travels in the `c` slot.
    """
    T = x.shape[0]
    h, s = h0.copy(), s0.copy()
    ys, cache = [], []
    for t in range(T):
        s_new = (1.0 - alpha) * (x[t] @ p["Bm"]) + alpha * s
        h_new = sigmoid(x[t] @ p["A"] + s_new @ p["P"] + h @ p["R"] + p["b_h"])
        cache.append((h, s, s_new, h_new))
        h, s = h_new, s_new
        ys.append(np.concatenate([h, s], 1))
    return np.stack(ys), h, s, cache


def scrn_backward(p, x, cache, dY, dhT, dsT, alpha):
    """Part 1: the h-chain (dz) in reverse; part 2: reverse linear scan for ds."""
    T = x.shape[0]
    H = p["R"].shape[0]
    grads = {k: np.zeros_like(p[k]) for k in SCRN_PARAMS}
    dx = np.zeros_like(x)
    dh_rec = dhT.copy()
    dz_all = [None] * T
    for t in reversed(range(T)):
        h_prev, s_prev, s_new, h_new = cache[t]
        dz = (dY[t][:, :H] + dh_rec) * h_new * (1.0 - h_new)
        dz_all[t] = dz
        grads["R"] += h_prev.T @ dz
        grads["A"] += x[t].T @ dz
        grads["P"] += s_new.T @ dz
        grads["b_h"] += dz.sum(0)
        dh_rec = dz @ p["R"].T
    ds = None
    for t in reversed(range(T)):
        dz = dz_all[t]
        if t == T - 1:
            ds = dY[t][:, H:] + dz @ p["P"].T + dsT
        else:
            ds = dY[t][:, H:] + dz @ p["P"].T + alpha * ds
        grads["Bm"] += x[t].T @ ((1.0 - alpha) * ds)
        dx[t] = dz @ p["A"].T + (1.0 - alpha) * (ds @ p["Bm"].T)
    ds0 = alpha * ds
    return grads, dx, dh_rec, ds0


# --------------------------------------------------------------------------------------
# RHN, recurrent highway network [39] with coupled carry.
# --------------------------------------------------------------------------------------
RHN_PARAMS = ("W", "R", "b")


def rhn_param_shapes(I, H, L):
    """W = [W_H | W_T] (I×2H, input enters at ℓ=1 only); R[ℓ] = [R_H,ℓ | R_T,ℓ]; b[ℓ] = [b_H | b_T]."""
    return {"W": (I, 2 * H), "R": (L, H, 2 * H), "b": (L, 2 * H)}


def rhn_forward(p, x, s0):
    """s^0_t = s^L_{t−1}; for ℓ=1..L: a = [ℓ=1]x_t·W + s^{ℓ−1}·R_ℓ + b_ℓ; h = tanh a_H,
    τ = σ(a_T); s^ℓ = h⊙τ + s^{ℓ−1}⊙(1−τ).  Output y_t = s^L_t (reading R9)."""
    T = x.shape[0]
    L, H = p["R"].shape[0], p["R"].shape[1]
    s = s0.copy()
    ys, cache = [], []
    for t in range(T):
        steps = []
        for l in range(L):
            a = s @ p["R"][l] + p["b"][l]
            if l == 0:
                a = a + x[t] @ p["W"]
            hh = np.tanh(a[:, :H])
            tau = sigmoid(a[:, H:])
            s_new = hh * tau + s * (1.0 - tau)
            steps.append((s, hh, tau))
            s = s_new
        cache.append(steps)
        ys.append(s)
    return np.stack(ys), s, cache


def rhn_backward(p, x, cache, dY, dsT):
    T = x.shape[0]
    L, H = p["R"].shape[0], p["R"].shape[1]
    grads = {k: np.zeros_like(p[k]) for k in RHN_PARAMS}
    dx = np.zeros_like(x)
    ds_carry = dsT.copy()
    for t in reversed(range(T)):
        ds = dY[t] + ds_carry
        for l in reversed(range(L)):
            s_prev, hh, tau = cache[t][l]
            dh = ds * tau
            dtau = ds * (hh - s_prev)
            daH = dh * (1.0 - hh * hh)
            daT = dtau * tau * (1.0 - tau)
            da = np.concatenate([daH, daT], 1)
            grads["R"][l] += s_prev.T @ da
            grads["b"][l] += da.sum(0)
            if l == 0:
                grads["W"] += x[t].T @ da
                dx[t] = da @ p["W"].T
            ds = ds * (1.0 - tau) + da @ p["R"][l].T
        ds_carry = ds
    return grads, dx, ds_carry


# --------------------------------------------------------------------------------------
# LSTM with attention, reduced GNMT [35].
# --------------------------------------------------------------------------------------
ATTN_PARAMS = ("W_e", "U_e", "b_e", "W_k", "W_d", "U_d", "C_d", "b_d", "W_q", "v")


def attn_param_shapes(I, H, A):
    return {"W_e": (I, 4 * H), "U_e": (H, 4 * H), "b_e": (4 * H,), "W_k": (H, A),
            "W_d": (I, 4 * H), "U_d": (H, 4 * H), "C_d": (H, 4 * H), "b_d": (4 * H,),
            "W_q": (H, A), "v": (A,)}


def attn_forward(p, xe, xd, h0, c0):
    """Encoder LSTM over Ts from (h0, c0) → enc_j, keys k_j = enc_j·W_k.  Decoder from the
    encoder's final state, ctx_0 = 0; for i = 1..Tt:
      a_i = x^d_i·W_d + h_{i−1}·U_d + ctx_{i−1}·C_d + b_d → LSTM → h_i;
      q_i = h_i·W_q; e_ij = vᵀ tanh(q_i + k_j); p_i = softmax_j e_i; ctx_i = Σ_j p_ij enc_j;
      y_i = [h_i | ctx_i]   (reading R10: additive attention, input feeding, A = H, no head).
    """
    H = h0.shape[1]
    encp = {"W": p["W_e"], "U": p["U_e"], "b": p["b_e"]}
    enc, he, ce, enc_cache = lstm_forward(encp, xe, h0, c0)   # enc [Ts, B, H]
    keys = enc @ p["W_k"]                                      # [Ts, B, A]
    Tt, B, _ = xd.shape
    h, c = he.copy(), ce.copy()
    ctx = np.zeros((B, H))
    ys, cache = [], []
    for i in range(Tt):
        a = xd[i] @ p["W_d"] + h @ p["U_d"] + ctx @ p["C_d"] + p["b_d"]
        gi, gf, gg, go = _lstm_gates(a, H)
        c_new = gf * c + gi * gg
        h_new = go * np.tanh(c_new)
        q = h_new @ p["W_q"]                                   # [B, A]
        u = np.tanh(q[None, :, :] + keys)                      # [Ts, B, A]
        e = u @ p["v"]                                         # [Ts, B]
        e = e - e.max(0, keepdims=True)
        w = np.exp(e)
        pr = w / w.sum(0, keepdims=True)                       # [Ts, B]
        ctx_new = (pr[:, :, None] * enc).sum(0)                # [B, H]
        cache.append((h, c, ctx, gi, gf, gg, go, c_new, h_new, u, pr))
        h, c, ctx = h_new, c_new, ctx_new
        ys.append(np.concatenate([h_new, ctx_new], 1))
    return np.stack(ys), h, c, (enc, keys, enc_cache, cache)


def attn_backward(p, xe, xd, fcache, dY, dhT, dcT):
    H = dhT.shape[1]
    enc, keys, enc_cache, cache = fcache
    Tt = xd.shape[0]
    grads = {k: np.zeros_like(p[k]) for k in ATTN_PARAMS}
    dxd = np.zeros_like(xd)
    denc = np.zeros_like(enc)
    dkeys = np.zeros_like(keys)
    dh_rec, dc = dhT.copy(), dcT.copy()
    dctx_rec = np.zeros_like(dY[0][:, H:])
    for i in reversed(range(Tt)):
        h_prev, c_prev, ctx_prev, gi, gf, gg, go, c_new, h_new, u, pr = cache[i]
        # attention backward: ctx_i = Σ_j p_ij enc_j, p = softmax(e), e = v·tanh(q + k)
        dctx = dY[i][:, H:] + dctx_rec
        dp = (dctx[None, :, :] * enc).sum(2)                   # [Ts, B]
        de = pr * (dp - (pr * dp).sum(0, keepdims=True))       # [Ts, B]
        denc += pr[:, :, None] * dctx[None, :, :]
        grads["v"] += np.einsum("jb,jba->a", de, u)
        du = de[:, :, None] * p["v"][None, None, :] * (1.0 - u * u)   # [Ts, B, A]
        dq = du.sum(0)                                         # [B, A]
        dkeys += du
        grads["W_q"] += h_new.T @ dq
        dh = dY[i][:, :H] + dh_rec + dq @ p["W_q"].T
        da, dc = _lstm_cell_bwd(dh, dc, c_prev, gi, gf, gg, go, c_new)
        grads["W_d"] += xd[i].T @ da
        grads["U_d"] += h_prev.T @ da
        grads["C_d"] += ctx_prev.T @ da
        grads["b_d"] += da.sum(0)
        dxd[i] = da @ p["W_d"].T
        dh_rec = da @ p["U_d"].T
        dctx_rec = da @ p["C_d"].T
    # keys k_j = enc_j·W_k
    Ts = enc.shape[0]
    for j in range(Ts):
        grads["W_k"] += enc[j].T @ dkeys[j]
        denc[j] += dkeys[j] @ p["W_k"].T
    encp = {"W": p["W_e"], "U": p["U_e"], "b": p["b_e"]}
    eg, dxe, dh0, dc0 = lstm_backward(encp, xe, enc_cache, denc, dh_rec, dc)
    grads["W_e"], grads["U_e"], grads["b_e"] = eg["W"], eg["U"], eg["b"]
    return grads, dxe, dxd, dh0, dc0


# --------------------------------------------------------------------------------------
# Uniform cell-level driver used by the tests: run forward, then backward of
# L = Σ dY⊙Y + Σ dhT⊙hT + Σ dcT⊙cT.
# --------------------------------------------------------------------------------------
def cell_fwd_bwd(cell, p, inputs, dY, dhT, dcT, **kw):
    """Returns (outputs, grads) as dicts.  outputs: y, hT, cT(or sT); grads: params + dx/dh0/dc0."""
    if cell in ("lstm", "milstm", "sublstm"):
        fwd = {"lstm": lstm_forward, "milstm": milstm_forward, "sublstm": sublstm_forward}[cell]
        bwd = {"lstm": lstm_backward, "milstm": milstm_backward, "sublstm": sublstm_backward}[cell]
        y, hT, cT, cache = fwd(p, inputs["x"], inputs["h0"], inputs["c0"])
        g, dx, dh0, dc0 = bwd(p, inputs["x"], cache, dY, dhT, dcT)
        return {"y": y, "hT": hT, "cT": cT}, dict(g, dx=dx, dh0=dh0, dc0=dc0)
    if cell == "scrn":
        a = kw["alpha"]
        y, hT, sT, cache = scrn_forward(p, inputs["x"], inputs["h0"], inputs["c0"], a)
        g, dx, dh0, ds0 = scrn_backward(p, inputs["x"], cache, dY, dhT, dcT, a)
        return {"y": y, "hT": hT, "cT": sT}, dict(g, dx=dx, dh0=dh0, dc0=ds0)
    if cell == "rhn":
        y, sT, cache = rhn_forward(p, inputs["x"], inputs["h0"])
        g, dx, ds0 = rhn_backward(p, inputs["x"], cache, dY, dhT)
        return {"y": y, "hT": sT}, dict(g, dx=dx, dh0=ds0)
    if cell == "attn":
        y, hT, cT, cache = attn_forward(p, inputs["xe"], inputs["xd"], inputs["h0"], inputs["c0"])
        g, dxe, dxd, dh0, dc0 = attn_backward(p, inputs["xe"], inputs["xd"], cache, dY, dhT, dcT)
        return {"y": y, "hT": hT, "cT": cT}, dict(g, dxe=dxe, dxd=dxd, dh0=dh0, dc0=dc0)
    raise ValueError(cell)


def cell_loss(cell, p, inputs, dY, dhT, dcT, **kw):
    """The scalar L whose gradient cell_fwd_bwd returns (used by finite-difference pins)."""
    if cell in ("lstm", "milstm", "sublstm"):
        fwd = {"lstm": lstm_forward, "milstm": milstm_forward, "sublstm": sublstm_forward}[cell]
        y, hT, cT, _ = fwd(p, inputs["x"], inputs["h0"], inputs["c0"])
    elif cell == "scrn":
        y, hT, cT, _ = scrn_forward(p, inputs["x"], inputs["h0"], inputs["c0"], kw["alpha"])
    elif cell == "rhn":
        y, hT, _ = rhn_forward(p, inputs["x"], inputs["h0"])
        return float((dY * y).sum() + (dhT * hT).sum())
    elif cell == "attn":
        y, hT, cT, _ = attn_forward(p, inputs["xe"], inputs["xd"], inputs["h0"], inputs["c0"])
    else:
        raise ValueError(cell)
    return float((dY * y).sum() + (dhT * hT).sum() + (dcT * cT).sum())
