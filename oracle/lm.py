"""fp64 oracle: language-model training step around a recurrent cell.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

One LM training step (forward pass over a mini-batch, loss against the ground
truth, back-propagation, "stochastic gradient descent [27]"):
  x[t,b]  = E[tok[t,b]]                              (embedding; targets are tok[t+1,b])
  y       = cell(x, h0, c0)                           (oracle.cells)
  logits  = y·W_o + b_o
  loss    = mean_{t,b} (logsumexp(logits) − logits[target])      (reading R12)
  dlogits = (softmax − onehot) / (T·B)
  dE[v]   = Σ_{(t,b): tok[t,b] = v} dx[t,b]
  θ      ← θ − lr·g                                   (reading R15: plain SGD)
"""
from __future__ import annotations

import numpy as np

from . import cells as C


def head_param_shapes(Hout, V):
    return {"W_o": (Hout, V), "b_o": (V,)}


def cross_entropy(logits, targets):
    """Mean CE over rows and its gradient w.r.t. logits.  logits [N, V], targets [N]."""
    m = logits.max(1, keepdims=True)
    z = logits - m
    lse = np.log(np.exp(z).sum(1, keepdims=True))
    logp = z - lse
    n = logits.shape[0]
    loss = -logp[np.arange(n), targets].mean()
    dlogits = np.exp(logp)
    dlogits[np.arange(n), targets] -= 1.0
    dlogits /= n
    return float(loss), dlogits


def lm_forward_backward(cell, p, tokens, h0, c0, **kw):
    """Loss, gradients (including dE, dW_o, db_o) and the carried final state.

    tokens: int [T+1, B].  p holds the cell's parameters plus 'E', 'W_o', 'b_o'.
    """
    T = tokens.shape[0] - 1
    B = tokens.shape[1]
    x = p["E"][tokens[:T]]                                     # a0
    inputs = {"x": x, "h0": h0, "c0": c0}
    if cell in ("lstm", "milstm", "sublstm"):
        fwd = {"lstm": C.lstm_forward, "milstm": C.milstm_forward, "sublstm": C.sublstm_forward}[cell]
        y, hT, cT, cache = fwd(p, x, h0, c0)
    elif cell == "scrn":
        y, hT, cT, cache = C.scrn_forward(p, x, h0, c0, kw["alpha"])
    elif cell == "rhn":
        y, hT, cache = C.rhn_forward(p, x, h0)
        cT = None
    else:
        raise ValueError(cell)
    Hout = y.shape[2]
    Y = y.reshape(T * B, Hout)
    logits = Y @ p["W_o"] + p["b_o"]                           # a4
    loss, dlogits = cross_entropy(logits, tokens[1:].reshape(-1))
    grads = {"W_o": Y.T @ dlogits, "b_o": dlogits.sum(0)}
    dY = (dlogits @ p["W_o"].T).reshape(T, B, Hout)
    zeros_h = np.zeros_like(h0)
    if cell in ("lstm", "milstm", "sublstm"):
        bwd = {"lstm": C.lstm_backward, "milstm": C.milstm_backward, "sublstm": C.sublstm_backward}[cell]
        g, dx, _, _ = bwd(p, x, cache, dY, zeros_h, np.zeros_like(c0))
    elif cell == "scrn":
        g, dx, _, _ = C.scrn_backward(p, x, cache, dY, zeros_h, np.zeros_like(c0), kw["alpha"])
    else:
        g, dx, _ = C.rhn_backward(p, x, cache, dY, zeros_h)
    grads.update(g)
    dE = np.zeros_like(p["E"])
    np.add.at(dE, tokens[:T].reshape(-1), dx.reshape(T * B, -1))   # a6: embedding backward
    grads["E"] = dE
    del inputs
    return loss, grads, (hT, cT)


def _cell_forward(cell, p, x, h0, c0, **kw):
    if cell in ("lstm", "milstm", "sublstm"):
        fwd = {"lstm": C.lstm_forward, "milstm": C.milstm_forward, "sublstm": C.sublstm_forward}[cell]
        return fwd(p, x, h0, c0)
    if cell == "scrn":
        return C.scrn_forward(p, x, h0, c0, kw["alpha"])
    if cell == "rhn":
        y, hT, cache = C.rhn_forward(p, x, h0)
        return y, hT, None, cache
    raise ValueError(cell)


def _cell_backward(cell, p, x, cache, dY, h0, c0, **kw):
    zeros_h = np.zeros_like(h0)
    if cell in ("lstm", "milstm", "sublstm"):
        bwd = {"lstm": C.lstm_backward, "milstm": C.milstm_backward, "sublstm": C.sublstm_backward}[cell]
        g, dx, _, _ = bwd(p, x, cache, dY, zeros_h, np.zeros_like(c0))
    elif cell == "scrn":
        g, dx, _, _ = C.scrn_backward(p, x, cache, dY, zeros_h, np.zeros_like(c0), kw["alpha"])
    else:
        g, dx, _ = C.rhn_backward(p, x, cache, dY, zeros_h)
    return g, dx


def stacked_lm_forward_backward(cells, ps, plm, tokens, h0s, c0s, **kw):
    """Stacked LM (PTB stacked LSTM): x_0 = E[tok], layer l maps
    x_l to y_l = x_{l+1}, the head reads the top layer; BPTT runs top down, layer l's input
    gradient being layer l-1's upstream gradient.  ps: per-layer parameter dicts; plm: E, W_o, b_o.
    Returns (loss, [per-layer grads], head/embedding grads)."""
    T = tokens.shape[0] - 1
    B = tokens.shape[1]
    x = plm["E"][tokens[:T]]
    xs, caches = [], []
    for cell, p, h0, c0 in zip(cells, ps, h0s, c0s):
        xs.append(x)
        y, _, _, cache = _cell_forward(cell, p, x, h0, c0, **kw)
        caches.append(cache)
        x = y
    Hout = x.shape[2]
    Y = x.reshape(T * B, Hout)
    logits = Y @ plm["W_o"] + plm["b_o"]
    loss, dlogits = cross_entropy(logits, tokens[1:].reshape(-1))
    glm = {"W_o": Y.T @ dlogits, "b_o": dlogits.sum(0)}
    dy = (dlogits @ plm["W_o"].T).reshape(T, B, Hout)
    gl = [None] * len(cells)
    for l in range(len(cells) - 1, -1, -1):
        gl[l], dy = _cell_backward(cells[l], ps[l], xs[l], caches[l], dy, h0s[l], c0s[l], **kw)
    dE = np.zeros_like(plm["E"])
    np.add.at(dE, tokens[:T].reshape(-1), dy.reshape(T * B, -1))
    glm["E"] = dE
    return loss, gl, glm


def sgd(p, grads, lr):
    """θ ← θ − lr·g for every parameter that has a gradient (a8)."""
    return {k: (v - lr * grads[k]) if k in grads else v for k, v in p.items()}


def lm_train_step(cell, p, tokens, h0, c0, lr, **kw):
    loss, grads, state = lm_forward_backward(cell, p, tokens, h0, c0, **kw)
    return loss, sgd(p, grads, lr), grads, state
