"""Stacked LSTM word LM vs cuDNN (Table 5): the paper's PTB "large"
stacked LSTM (2 layers, input = hidden = 1500, vocab 10k, 35 steps) at mini-batch 8..256.

  astra : astra_lm_create_stacked over two LSTM cells, every layer explored by its tuner on live
          steps, then frozen and replayed as a CUDA graph (bf16 GEMM operands, fp32 state).
  cudnn : torch.nn.LSTM(num_layers=2) in bf16 (cuDNN) + embedding + linear head + cross-entropy,
          backward, SGD — the library baseline the paper normalises Table 5 to (context only: not
          part of the product, and not the oracle).

Prints one JSON line per batch size: train samples/s of both and the ratio astra / cuDNN.

  python bench_stacked.py [--batches 8,16,32,64,128,256] [--steps 20]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

H = I = 1500
V = 10000
T = 35
LAYERS = 2
SEED = 20190413 + 7000


def time_steps(torch, fn, steps, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / 1e3 / steps


def astra_arm(torch, A, synth, B, tok, steps):
    layers = [A.Cell("lstm", H, I, B, T, dtype="bf16") for _ in range(LAYERS)]
    m = A.LM(layers, V)
    shapes = {k: (r, c) if r > 1 else (c,) for k, (off, r, c) in m.param_info.items()}
    m.load(synth.weights(SEED, shapes, H))
    for c in layers:
        c.tune_mode(A.TUNE_ON)
    n = 0
    while n < 600:
        m.train_step(tok, 0.01)
        st = [c.tune_next() for c in layers]
        n += 1
        if all(s == A.TUNE_CONVERGED for s in st):
            break
    for c in layers:
        c.tune_mode(A.TUNE_FROZEN, c.tune_report()["variant"])
    sec = time_steps(torch, lambda: m.train_step(tok, 0.01), steps)
    return sec, n, [c.tune_report()["variant"] for c in layers]


def cudnn_arm(torch, B, tok, steps):
    dt = torch.bfloat16
    emb = torch.nn.Embedding(V, I).cuda().to(dt)
    rnn = torch.nn.LSTM(I, H, num_layers=LAYERS).cuda().to(dt)
    head = torch.nn.Linear(H, V).cuda().to(dt)
    params = list(emb.parameters()) + list(rnn.parameters()) + list(head.parameters())
    opt = torch.optim.SGD(params, lr=0.01)
    x, y = tok[:T].long(), tok[1:].long().reshape(-1)

    def step():
        opt.zero_grad(set_to_none=True)
        out, _ = rnn(emb(x))
        loss = torch.nn.functional.cross_entropy(head(out).reshape(T * B, V).float(), y)
        loss.backward()
        opt.step()
    return time_steps(torch, step, steps), torch.backends.cudnn.version()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batches", default="8,16,32,64,128,256")
    ap.add_argument("--steps", type=int, default=20)
    a = ap.parse_args()
    import torch
    import paper_conf_asplos_sivathanucsz19_b200 as A
    import synth
    for B in [int(x) for x in a.batches.split(",")]:
        tok = torch.as_tensor(synth.zipf_tokens(SEED, "tokens", (T + 1, B), V), dtype=torch.int32, device="cuda")
        s_a, n_explore, variants = astra_arm(torch, A, synth, B, tok, a.steps)
        s_c, cudnn_v = cudnn_arm(torch, B, tok, a.steps)
        print(json.dumps({"metric": "stacked LSTM LM train samples/s", "layers": LAYERS, "hidden": H, "input": I,
                          "vocab": V, "seq_len": T, "batch": B, "dtype": "bf16", "data": "synthetic",
                          "astra": B / s_a, "cudnn": B / s_c, "astra_over_cudnn": s_c / s_a,
                          "astra_ms": 1e3 * s_a, "cudnn_ms": 1e3 * s_c, "explore_steps": n_explore,
                          "cudnn_version": cudnn_v, "variants": variants}), flush=True)


if __name__ == "__main__":
    main()
