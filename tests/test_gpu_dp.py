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


def _case_bf16(T, B, I, H, V, seed):
    from helpers import bf16_round
    p, tok = _case(T, B, I, H, V, seed)
    for k in ("W", "U", "E", "W_o"):
        p[k] = bf16_round(p[k])
    return p, tok


def _nccl_worker(rank, world, port, q, stacked):
    """One rank per GPU: the library's bucketed NCCL all-reduce (one communicator for the LM,
    astra_lm_comm_init) on the rank's contiguous batch shard; returns its gradients and loss."""
    import os
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    try:
        import torch.distributed as dist
        import paper_conf_asplos_sivathanucsz19_b200 as A
        torch.cuda.set_device(rank)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        T, B, I, H, V = 5, 16, 64, 64, 40
        p, tok = _case_bf16(T, B, I, H, V, 33)
        sl = slice(rank * B // world, (rank + 1) * B // world)
        cells = [A.Cell("milstm", H, I, B // world, T, dtype="bf16", device=rank)]
        m = A.LM(cells[0], V)
        m.load(p)
        uid = [A.comm_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        m.comm_init(uid[0], rank, world)
        tokens = torch.as_tensor(np.ascontiguousarray(tok[:, sl]), dtype=torch.int32, device=f"cuda:{rank}")
        m.fwd_bwd(tokens)
        torch.cuda.synchronize()
        q.put((rank, m.grads.cpu().numpy(), float(m.loss.item()), {k: v for k, v in m.param_info.items()}))
        dist.barrier()
        dist.destroy_process_group()
    except Exception as e:   # surface the failure in the parent
        q.put((rank, None, repr(e), None))


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="NCCL needs one GPU per rank (a 1-GPU box cannot run it)")
def test_nccl_world2_bucketed_allreduce_vs_oracle_dp():
    """The NCCL bucketed gradient all-reduce with world = 2 (two GPUs): both ranks hold the same
    gradients, equal to the fp64 oracle's DP semantics (mean of the two shard-mean gradients,
    oracle.dp.dp_gradients) within the bf16 tolerance."""
    import os
    import torch.multiprocessing as mp
    from oracle import dp as ODP
    from helpers import TOL_BF16
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29950 + os.getpid() % 40
    procs = [ctx.Process(target=_nccl_worker, args=(r, 2, port, q, False)) for r in range(2)]
    for pr in procs:
        pr.start()
    res = {}
    for _ in range(2):
        r, g, loss, info = q.get(timeout=300)
        assert g is not None, loss
        res[r] = (g, loss, info)
    for pr in procs:
        pr.join(60)
    assert np.array_equal(res[0][0], res[1][0])
    T, B, I, H, V = 5, 16, 64, 64, 40
    p, tok = _case_bf16(T, B, I, H, V, 33)
    _, g_o = ODP.dp_gradients("milstm", p, tok, np.zeros((B, H)), np.zeros((B, H)), 2)
    info = res[0][2]
    for k, (off, r_, c_) in info.items():
        got = res[0][0][off:off + r_ * c_].reshape(np.shape(g_o[k]))
        assert rel_err(got, g_o[k]) <= TOL_BF16, k
