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


def sgd(p, grads, lr):
    """θ ← θ − lr·g for every parameter that has a gradient (a8)."""
    return {k: (v - lr * grads[k]) if k in grads else v for k, v in p.items()}


def lm_train_step(cell, p, tokens, h0, c0, lr, **kw):
    loss, grads, state = lm_forward_backward(cell, p, tokens, h0, c0, **kw)
    return loss, sgd(p, grads, lr), grads, state
