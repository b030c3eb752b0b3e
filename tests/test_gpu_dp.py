"""Data parallelism (north star item 5) on one B200: the NCCL bucket path with a
single-rank communicator is an exact identity, and "virtual DP" — shard gradients computed
separately and averaged — matches the full-batch gradient (oracle/dp.py semantics)."""
import numpy as np
import pytest
import torch

import synth
from oracle import lm as OLM

from helpers import TOL_FP32, cell_shapes, rel_err

pytestmark = pytest.mark.gpu


def _lm(cell, T, B, I, H, V, dtype, p, tok, comm=False):
    import paper_conf_asplos_sivathanucsz19_b200 as A
    c = A.Cell(cell, H, I, B, T, dtype=dtype)
    if comm:
        c.comm_init(A.comm_unique_id(), 0, 1)
    m = A.LM(c, V)
    m.load(p)
    tokens = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
    m.fwd_bwd(tokens)
    torch.cuda.synchronize()
    return m


def _case(T, B, I, H, V, seed):
    shapes = cell_shapes("milstm", I, H)
    shapes.update({"E": (V, I), "W_o": (H, V), "b_o": (V,)})
    p = synth.weights(seed, shapes, H, {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)})
    tok = synth.zipf_tokens(seed, "tok", (T + 1, B), V, V - 3)
    return p, tok


@pytest.mark.parametrize("dtype", ["fp32", "bf16"])
def test_single_rank_nccl_bucket_path_is_identity(dtype):
    T, B, I, H, V = 5, 16, 64, 64, 40
    p, tok = _case(T, B, I, H, V, 31)
    a = _lm("milstm", T, B, I, H, V, dtype, p, tok, comm=False)
    b = _lm("milstm", T, B, I, H, V, dtype, p, tok, comm=True)
    assert torch.equal(a.grads, b.grads)
    assert torch.equal(a.loss, b.loss)


def test_virtual_dp_mean_of_shards_equals_full_batch():
    T, B, I, H, V, N = 4, 16, 64, 64, 40, 4
    p, tok = _case(T, B, I, H, V, 32)
    full = _lm("milstm", T, B, I, H, V, "fp32", p, tok)
    acc = None
    for r in range(N):
        sl = slice(r * B // N, (r + 1) * B // N)
        m = _lm("milstm", T, B // N, I, H, V, "fp32", p, np.ascontiguousarray(tok[:, sl]))
        g = m.grads.double().cpu() / N
        acc = g if acc is None else acc + g
    for name in ("W", "U", "b", "alpha", "E", "W_o", "b_o"):
        v_full = full.view(name, full.grads).double().cpu().numpy()
        off, r_, c_ = full.param_info[name]
        v_dp = acc[off:off + r_ * c_].numpy().reshape(v_full.shape)
        assert rel_err(v_dp, v_full) <= TOL_FP32, name
    # and the full-batch gradient matches the oracle
    lo, go, _ = OLM.lm_forward_backward("milstm", p, tok, np.zeros((B, H)), np.zeros((B, H)))
    assert rel_err(full.view("U", full.grads).cpu().numpy(), go["U"]) <= TOL_FP32
