"""K11p, the deterministic peer-memory DP backend (SURVEY §8(e) backend 2), through the C ABI.

Two ranks run as two processes sharing cuda:0 (the same CUDA IPC mappings and flag barriers as on
two NVLink peers; the gradient windows are exchanged over a gloo process group).  Each rank trains
on its contiguous batch shard (§8(c.3) item 8).  The expected result is built in this process
from two single-rank instances WITHOUT any communication: g = (g_0 + g_1)·(1/2) in fp32 (rank
order) and θ ← θ − lr·g.  The backend must reproduce it bit for bit on both ranks, over several
steps (state carried per shard), and the full-batch mean it computes must match the fp64 oracle.
"""
import os

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import synth
from oracle import lm as OLM

from helpers import TOL_BF16, TOL_FP32, bf16_round, cell_shapes, fp32_ulp, make_cell_case, rel_err

pytestmark = pytest.mark.gpu

T, B, I, H, V, LR, STEPS = 5, 16, 64, 64, 40, 0.5, 3


def _lm_case(dtype, seed=41):
    shapes = cell_shapes("milstm", I, H)
    shapes.update({"E": (V, I), "W_o": (H, V), "b_o": (V,)})
    p = synth.weights(seed, shapes, H, {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)})
    if dtype == "bf16":
        for k in ("W", "U", "E", "W_o"):
            p[k] = bf16_round(p[k])
    tok = synth.zipf_tokens(seed, "tok", (T + 1, B), V, V - 3)
    return p, tok


def _shard(a, r, world, axis=1):
    n = a.shape[axis] // world
    return np.ascontiguousarray(np.take(a, range(r * n, (r + 1) * n), axis=axis))


def _worker(rank, world, port, kind, dtype, q, variant=None, steps=STEPS):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        os.environ.setdefault("ASTRA_PEER_TIMEOUT_S", "30")
        import torch.distributed as dist
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        import paper_conf_asplos_sivathanucsz19_b200 as A
        if kind == "lm":
            p, tok = _lm_case(dtype)
            c = A.Cell("milstm", H, I, B // world, T, dtype=dtype)
            m = A.LM(c, V)
            m.load(p)
            if variant:
                c.tune_mode(A.TUNE_FROZEN, variant)
            A.peer_exchange(m)
            tokens = torch.as_tensor(_shard(tok, rank, world), dtype=torch.int32, device="cuda")
            losses = []
            for _ in range(steps):
                m.train_step(tokens, LR)
                losses.append(m.loss.item())
            torch.cuda.synchronize()
            q.put((rank, m.params.cpu().numpy(), m.grads.cpu().numpy(), losses))
        else:
            p, inp, dY, dhT, dcT = make_cell_case("lstm", T, B, I, H, 43, bf16=dtype == "bf16")
            c = A.Cell("lstm", H, I, B // world, T, dtype=dtype)
            c.load(p)
            A.peer_exchange(c)
            tdt = torch.bfloat16 if dtype == "bf16" else torch.float32
            dev = torch.device("cuda", 0)
            x = torch.as_tensor(_shard(inp["x"], rank, world), dtype=tdt, device=dev)
            dy = torch.as_tensor(_shard(dY, rank, world), dtype=tdt, device=dev)
            h0 = torch.as_tensor(_shard(inp["h0"], rank, world, 0), dtype=torch.float32, device=dev)
            c0 = torch.as_tensor(_shard(inp["c0"], rank, world, 0), dtype=torch.float32, device=dev)
            y = torch.empty(T, B // world, H, dtype=tdt, device=dev)
            for _ in range(STEPS):
                c.forward(x, h0, c0, y)
                c.backward(dy)
                c.sgd(LR)
            torch.cuda.synchronize()
            q.put((rank, c.params.cpu().numpy(), c.grads.cpu().numpy(), []))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:   # surface the error in the parent
        q.put((rank, None, None, repr(e)))
        raise


def _run_world(kind, dtype, world=2, variant=None, steps=STEPS):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29650 + os.getpid() % 300
    procs = [ctx.Process(target=_worker, args=(r, world, port, kind, dtype, q, variant, steps)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = {}
    for _ in range(world):
        r, pp, gg, extra = q.get(timeout=300)
        assert pp is not None, f"rank {r}: {extra}"
        res[r] = (pp, gg, extra)
    for pr in procs:
        pr.join(120)
        assert pr.exitcode == 0
    return res


def _reference_lm(dtype, world=2):
    """Single-rank instances, no communication: the rank-ordered fp32 mean and SGD by hand."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    p, tok = _lm_case(dtype)
    ms = []
    for r in range(world):
        c = A.Cell("milstm", H, I, B // world, T, dtype=dtype)
        m = A.LM(c, V)
        m.load(p)
        m._tok = torch.as_tensor(_shard(tok, r, world), dtype=torch.int32, device="cuda")
        ms.append(m)
    for _ in range(STEPS):
        for m in ms:
            m.fwd_bwd(m._tok)
        g = ms[0].grads.clone()
        for m in ms[1:]:
            g = g + m.grads
        g = g * (1.0 / world)
        newp = ms[0].params - LR * g
        for m in ms:
            m.params.copy_(newp)
    torch.cuda.synchronize()
    return newp.cpu().numpy(), g.cpu().numpy(), [m.grads.cpu().numpy() for m in ms], p, tok


@pytest.mark.parametrize("dtype,variant", [("fp32", None), ("bf16", None), ("fp32", "dpb=2"), ("bf16", "dpb=3")])
def test_peer_lm_bitwise_equals_rank_ordered_mean(dtype, variant, monkeypatch):
    """dpb = 2 / 3 (AV dp_bucket) cut the buckets into 32 / 8 KB pieces here (ASTRA_DPB_DIV = 1024):
    the bits do not move (the per-element rank-ordered sum does not see bucket boundaries)."""
    monkeypatch.setenv("ASTRA_DPB_DIV", "1024")
    res = _run_world("lm", dtype, variant=variant)
    p_ref, g_ref, g_shards, p0, tok = _reference_lm(dtype)
    for r, (pp, gg, losses) in res.items():
        assert np.array_equal(pp, p_ref), f"rank {r}: parameters differ from the rank-ordered mean SGD"
        # each element holds the global mean on its owner and this rank's shard mean elsewhere
        assert np.all((gg == g_ref) | (gg == g_shards[r])), f"rank {r}: gradient neither mean nor own"
    owned = np.zeros(g_ref.shape, bool)
    for r, (pp, gg, _) in res.items():
        owned |= gg == g_ref
    assert owned.all(), "some gradient element is the global mean on no rank"
    # first step = the full-batch step of the fp64 oracle: mean of the equal-size shard losses
    lo, _, _ = OLM.lm_forward_backward("milstm", p0, tok, np.zeros((B, H)), np.zeros((B, H)))
    l1 = 0.5 * (res[0][2][0] + res[1][2][0])
    assert abs(l1 - lo) / abs(lo) < (TOL_BF16 if dtype == "bf16" else TOL_FP32)


def test_peer_cell_api_bitwise_equals_rank_ordered_mean():
    import paper_conf_asplos_sivathanucsz19_b200 as A
    dtype, world = "bf16", 2
    res = _run_world("cell", dtype)
    p, inp, dY, dhT, dcT = make_cell_case("lstm", T, B, I, H, 43, bf16=True)
    cs = []
    dev = torch.device("cuda", 0)
    for r in range(world):
        c = A.Cell("lstm", H, I, B // world, T, dtype=dtype)
        c.load(p)
        c._x = torch.as_tensor(_shard(inp["x"], r, world), dtype=torch.bfloat16, device=dev)
        c._dy = torch.as_tensor(_shard(dY, r, world), dtype=torch.bfloat16, device=dev)
        c._h0 = torch.as_tensor(_shard(inp["h0"], r, world, 0), dtype=torch.float32, device=dev)
        c._c0 = torch.as_tensor(_shard(inp["c0"], r, world, 0), dtype=torch.float32, device=dev)
        c._y = torch.empty(T, B // world, H, dtype=torch.bfloat16, device=dev)
        cs.append(c)
    for _ in range(STEPS):
        for c in cs:
            c.forward(c._x, c._h0, c._c0, c._y)
            c.backward(c._dy)
        g = (cs[0].grads + cs[1].grads) * 0.5
        newp = cs[0].params - LR * g
        for c in cs:
            c.params.copy_(newp)
    ref = newp.cpu().numpy()
    for r, (pp, gg, _) in res.items():
        assert np.array_equal(pp, ref), f"rank {r}"


@pytest.mark.parametrize("dtype,tol", [("fp32", TOL_FP32), ("bf16", TOL_BF16)])
def test_peer_lm_step_vs_oracle_dp(dtype, tol):
    """One K11p step against the fp64 oracle's DP semantics (oracle.dp.dp_gradients: the mean of
    the two shard-mean gradients, §8(c.3) item 8) and its SGD (oracle.lm.sgd): the parameter update
    θ_1 − θ_0 of every tensor, identical on both ranks, equals −lr·g_oracle."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    from oracle import dp as ODP
    res = _run_world("lm", dtype, steps=1)
    p0, tok = _lm_case(dtype)
    _, g_o = ODP.dp_gradients("milstm", p0, tok, np.zeros((B, H)), np.zeros((B, H)), 2)
    c = A.Cell("milstm", H, I, B // 2, T, dtype=dtype)
    m = A.LM(c, V)
    assert np.array_equal(res[0][0], res[1][0])
    theta1 = res[0][0]
    errs = {}
    for k, (off, r, cc) in m.param_info.items():
        th0 = np.asarray(p0[k], np.float32).astype(np.float64).ravel()
        th1 = theta1[off:off + r * cc].astype(np.float64)
        floor = 0.5 * np.maximum(fp32_ulp(th1), fp32_ulp(th0))   # fp32 master storage (R16)
        errs[k] = rel_err((th1 - th0).reshape(r, cc) if r > 1 else th1 - th0,
                          (-LR * np.asarray(g_o[k])).reshape(r, cc) if r > 1 else -LR * np.asarray(g_o[k]),
                          floor.reshape(r, cc) if r > 1 else floor)
    bad = {k: v for k, v in errs.items() if not v <= tol}
    assert not bad, (bad, errs)
