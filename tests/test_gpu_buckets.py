"""Bucketed profiling of variable-length mini-batches (§5.5; Table 8).

A step of length len runs at the smallest bucket T_b >= len on right-padded tokens with the loss
restricted to the first len positions, so its loss and gradients must equal the fp64 oracle's on
the unpadded length-len mini-batch (zero initial state).  Each bucket explores its own update tree,
and exploration stays value-preserving across bucket switches."""
import numpy as np
import pytest
import torch

import synth
from oracle import lm as OLM

from helpers import TOL_BF16, TOL_FP32, rel_err
from test_gpu_lm import _cell_kw, _lm_case

pytestmark = pytest.mark.gpu

TMAX, B, I, H, V = 10, 8, 64, 64, 50
BUCKETS = [4, 7, 10]


def _lm(cell, dtype, p, Tmax=TMAX, b=B):
    import paper_conf_asplos_sivathanucsz19_b200 as A
    c = A.Cell(cell, H, I, b, Tmax, dtype=dtype, **_cell_kw(cell)[0])
    m = A.LM(c, V)
    m.load(p)
    return c, m


@pytest.mark.parametrize("dtype,tol", [("fp32", TOL_FP32), ("bf16", TOL_BF16)])
@pytest.mark.parametrize("cell", ["milstm", "scrn", "rhn"])
def test_bucketed_step_matches_unpadded_oracle(cell, dtype, tol):
    seed = synth.config_seed(5) + 31
    p, tok, _, _ = _lm_case(cell, TMAX, B, I, H, V, seed, dtype == "bf16", 40)
    c, m = _lm(cell, dtype, p)
    m.set_buckets(BUCKETS)
    h0 = np.zeros((B, H))
    c0 = None if cell == "rhn" else np.zeros((B, 24 if cell == "scrn" else H))
    for L in (3, 5, 7, 10):   # padded to 4, 7, 7, 10
        t = torch.as_tensor(tok[:L + 1], dtype=torch.int32, device=c.device).contiguous()
        loss = float(m.fwd_bwd_len(t, L).item())
        torch.cuda.synchronize()
        lo, go, _ = OLM.lm_forward_backward(cell, p, tok[:L + 1], h0, c0, **_cell_kw(cell)[1])
        assert abs(loss - lo) / abs(lo) <= tol, (L, loss, lo)
        g = {k: m.view(k, m.grads).cpu().numpy().reshape(np.shape(p[k])) for k in go}
        errs = {k: rel_err(g[k], go[k]) for k in go}
        assert all(v <= tol for v in errs.values()), (L, errs)


def test_len_out_of_range_rejected():
    import paper_conf_asplos_sivathanucsz19_b200 as A
    p, tok, _, _ = _lm_case("milstm", TMAX, B, I, H, V, synth.config_seed(5), True, 40)
    c, m = _lm("milstm", "bf16", p)
    t = torch.as_tensor(tok, dtype=torch.int32, device=c.device)
    for bad in (0, TMAX + 1):
        with pytest.raises(A.AstraError):
            m.fwd_bwd_len(t, bad)
    with pytest.raises(A.AstraError):
        m.set_buckets([5, 3])
    with pytest.raises(A.AstraError):
        m.set_buckets([4, TMAX + 1])


def test_bucket_tuner_independent_and_value_preserving():
    """Lengths alternating over two buckets with the tuner exploring vs frozen at the default:
    bitwise-identical parameters; each bucket has its own exploration state and index keys."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    seed = synth.config_seed(5) + 33
    Tmax, b = 12, 128
    lengths = [5, 12, 3, 12, 6, 9] * 8
    out = []
    for mode in (A.TUNE_OFF, A.TUNE_ON):
        p, tok, _, _ = _lm_case("milstm", Tmax, b, I, H, V, seed, True, 40)
        c, m = _lm("milstm", "bf16", p, Tmax, b)
        m.set_buckets([6, 12])
        c.tune_mode(mode)
        for L in lengths:
            t = torch.as_tensor(tok[:L + 1], dtype=torch.int32, device=c.device).contiguous()
            m.train_step_len(t, L, 0.1)
            c.tune_next()
        torch.cuda.synchronize()
        out.append((m.params.clone(), float(m.loss.item()), c.tune_report()))
    assert torch.equal(out[0][0], out[1][0]) and out[0][1] == out[1][1]
    rep = out[1][2]
    assert rep["bucket"] == 12 and "6" in rep["other_buckets"]
    assert rep["configs_explored"] >= 2 and rep["other_buckets"]["6"]["configs_explored"] >= 2
    assert all("|b=12|" in k for k in rep["index"])


def test_full_step_after_buckets_restores_seq():
    """A plain train step after bucketed ones runs the full length again (same bits as a fresh LM)."""
    seed = synth.config_seed(5) + 35
    p, tok, _, _ = _lm_case("milstm", TMAX, B, I, H, V, seed, True, 40)
    c1, m1 = _lm("milstm", "bf16", p)
    m1.set_buckets(BUCKETS)
    t = torch.as_tensor(tok, dtype=torch.int32, device=c1.device)
    m1.fwd_bwd_len(t[:4].contiguous(), 3)
    m1.set_state(None, None)
    l1 = float(m1.fwd_bwd(t).item())
    g1 = m1.grads.clone()
    c2, m2 = _lm("milstm", "bf16", p)
    l2 = float(m2.fwd_bwd(t).item())
    torch.cuda.synchronize()
    assert l1 == l2 and torch.equal(g1, m2.grads)
