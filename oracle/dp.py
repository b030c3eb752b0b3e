"""fp64 oracle: data-parallel semantics (BASELINE.json north_star (5)).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The paper is single-GPU and names multi-GPU only as a future dimension (P:134,
P:451).  The north star fixes the reading: the global batch of B_g sequences is split into
N contiguous batch-column shards; every rank computes its shard-mean gradient g_r; the
synchronised gradient is g = (1/N)·Σ_r g_r, which equals the full-batch mean gradient
because every shard has the same number of predicted tokens.
"""
from __future__ import annotations

import numpy as np

from . import lm


def shard_columns(B_g, N, r):
    """Columns [r·B_g/N, (r+1)·B_g/N) of the time-major token matrix."""
    assert B_g % N == 0
    b = B_g // N
    return slice(r * b, (r + 1) * b)


def dp_gradients(cell, p, tokens, h0, c0, N, **kw):
    """Mean of the N shard gradients (and the mean of shard losses)."""
    B_g = tokens.shape[1]
    acc, loss = None, 0.0
    for r in range(N):
        sl = shard_columns(B_g, N, r)
        l, g, _ = lm.lm_forward_backward(cell, p, tokens[:, sl], h0[sl], None if c0 is None else c0[sl], **kw)
        loss += l / N
        if acc is None:
            acc = {k: v / N for k, v in g.items()}
        else:
            for k in acc:
                acc[k] = acc[k] + g[k] / N
    return loss, acc
