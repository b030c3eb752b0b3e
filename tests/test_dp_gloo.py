"""World-size-2 gloo check (CPU) of the DP host logic used by bench.py: the contiguous batch-column
sharding of the global token matrix and the mean-of-shard-gradients reduction reproduce the
full-batch gradient of the oracle (oracle/dp.py)."""
import os

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import bench
    from oracle import cells as C
    from oracle import lm as OLM
    T, B_g, I, H, V = 3, 8, 6, 5, 11
    shapes = C.milstm_param_shapes(I, H)
    shapes.update({"E": (V, I), "W_o": (H, V), "b_o": (V,)})
    p = synth.weights(99, shapes, H, {"alpha": (0.5, 1.5), "beta1": (0.5, 1.5), "beta2": (0.5, 1.5)})
    tok = bench.make_inputs(B_g, T, V, V - 2, rank, world)          # the bench's own shard function
    B = B_g // world
    _, g, _ = OLM.lm_forward_backward("milstm", p, tok, np.zeros((B, H)), np.zeros((B, H)))
    flat = torch.tensor(np.concatenate([g[k].ravel() for k in sorted(g)]))
    dist.all_reduce(flat)
    flat /= world
    if rank == 0:
        full = bench.make_inputs(B_g, T, V, V - 2, 0, 1)
        _, gf, _ = OLM.lm_forward_backward("milstm", p, full, np.zeros((B_g, H)), np.zeros((B_g, H)))
        ref = np.concatenate([gf[k].ravel() for k in sorted(gf)])
        q.put(float(np.abs(flat.numpy() - ref).max() / np.abs(ref).max()))
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_world2_dp_mean_equals_full_batch():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + os.getpid() % 1000
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    for pr in procs:
        pr.join(120)
        assert pr.exitcode == 0
    assert q.get(timeout=5) < 1e-12


class _FakeWindow:
    """Stands in for a Cell / LM: the handle exchange of the peer-memory backend is host logic."""

    def __init__(self, rank):
        self.rank = rank
        self.got = None

    def comm_peer_handle(self):
        return bytes([self.rank + 1]) * 256

    def comm_peer_init(self, handles, rank, world):
        self.got = (handles, rank, world)


def _peer_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_asplos_sivathanucsz19_b200 as A
    w = _FakeWindow(rank)
    A.peer_exchange(w)
    handles, r, n = w.got
    q.put((rank, r, n, handles == b"".join(bytes([k + 1]) * 256 for k in range(world))))
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_world2_peer_handle_exchange_is_rank_ordered():
    """K11p host plumbing (SURVEY §8(e) backend 2): every rank receives all window handles in rank
    order and maps them with its own rank and the world size."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + (os.getpid() + 7) % 1000
    procs = [ctx.Process(target=_peer_worker, args=(r, 2, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    for pr in procs:
        pr.join(120)
        assert pr.exitcode == 0
    got = sorted(q.get(timeout=5) for _ in range(2))
    assert got == [(0, 0, 2, True), (1, 1, 2, True)]
