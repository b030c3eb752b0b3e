"""Multi-step training trajectories against the fp64 oracle (
round-1 VERDICT "What's weak" #3): SGD θ ← θ − lr·g ("stochastic gradient descent") applied by
the library's own kernels over several LM steps, with the recurrent state carried between steps
(reading R13), compared step by step with oracle.lm.lm_train_step iterated on the host.

bf16 path: the library keeps fp32 master weights and regenerates the bf16 operand mirrors from them
on every forward (K9); the oracle keeps fp64 masters and feeds the bf16-rounded GEMM weights to
each step (reading R18), so both sides see the same operands up to the master precision.
Compared: every step's loss, and the accumulated update θ_k − θ_0 of every parameter tensor after
the last step (the update, not θ itself, so an error in lr·g is not hidden under θ_0), element-wise
with a floor of ½ fp32 ulp of θ per step (the fp32 master storage, R16: an update far below θ's
resolution — MI-LSTM's α — is otherwise dominated by storage rounding on both sides)."""
import numpy as np
import pytest
import torch

import synth
from oracle import lm as OLM

from helpers import TOL_BF16, TOL_FP32, bf16_round, cell_shapes, fp32_ulp, rel_err

pytestmark = pytest.mark.gpu

BF16_OPERANDS = ("W", "U", "A", "Bm", "P", "R", "E", "W_o")
S_CTX, L_DEPTH, ALPHA = 24, 2, 0.95


def _case(cell, T, B, I, H, V, seed):
    shapes = cell_shapes(cell, I, H, S_CTX, L_DEPTH)
    Hout = H + S_CTX if cell == "scrn" else H
    shapes.update({"E": (V, I), "W_o": (Hout, V), "b_o": (V,)})
    p = synth.weights(seed, shapes, H, {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)})
    # fp32-representable masters on both sides
    p = {k: np.asarray(v, dtype=np.float32).astype(np.float64) for k, v in p.items()}
    toks = [synth.zipf_tokens(seed, f"tok{k}", (T + 1, B), V, V - 7) for k in range(3)]
    h0 = synth.uniform(seed, "h0", (B, H), -0.5, 0.5)
    c0 = None if cell == "rhn" else synth.uniform(seed, "c0", (B, S_CTX if cell == "scrn" else H), -0.5, 0.5)
    return p, toks, h0, c0


@pytest.mark.parametrize("dtype,tol", [("fp32", TOL_FP32), ("bf16", TOL_BF16)])
@pytest.mark.parametrize("cell", ["milstm", "scrn", "rhn"])
def test_lm_sgd_trajectory_vs_oracle(cell, dtype, tol):
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H, V, lr = 5, 16, 64, 64, 48, 0.5
    p0, toks, h0, c0 = _case(cell, T, B, I, H, V, synth.config_seed(5) + 31)
    kw = {"context": S_CTX, "scrn_alpha": ALPHA} if cell == "scrn" else {"depth": L_DEPTH} if cell == "rhn" else {}
    okw = {"alpha": np.float32(ALPHA).item()} if cell == "scrn" else {}
    c = A.Cell(cell, H, I, B, T, dtype=dtype, **kw)
    m = A.LM(c, V)
    m.load(p0)
    dev = c.device
    f32 = lambda a: None if a is None else torch.as_tensor(np.asarray(a, dtype=np.float32), device=dev)
    m.set_state(f32(h0), f32(c0))
    # oracle: fp64 masters; each step computes on the bf16-rounded operands on the bf16 path
    po, ho, co = dict(p0), h0, c0
    for k, tok in enumerate(toks):
        loss = float(m.train_step(torch.as_tensor(tok, dtype=torch.int32, device=dev), lr).item())
        pc = {kk: (bf16_round(v) if dtype == "bf16" and kk in BF16_OPERANDS else v) for kk, v in po.items()}
        lo, grads, (ho, co) = OLM.lm_forward_backward(cell, pc, tok, ho, co, **okw)
        po = OLM.sgd(po, grads, lr)
        assert abs(loss - lo) / abs(lo) <= tol, (k, loss, lo)
    torch.cuda.synchronize()
    errs = {}
    for k in p0:
        theta = m.view(k).cpu().numpy().astype(np.float64).reshape(np.shape(p0[k]))
        # the library stores fp32 masters (R16): each SGD step rounds θ to fp32 (≤ ½ ulp), a floor
        # every element of the accumulated update may carry regardless of the gradient's accuracy
        floor = len(toks) * 0.5 * np.maximum(fp32_ulp(theta), fp32_ulp(p0[k]))
        errs[k] = rel_err(theta - p0[k], po[k] - p0[k], floor)
    bad = {k: v for k, v in errs.items() if not v <= tol}
    assert not bad, (bad, errs)
