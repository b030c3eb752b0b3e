"""Bucketed-profiling benchmark: variable-length mini-batches (§5.5, §6.5 P:420,
Table 8).  Not the headline bench (bench.py is); this measures the SURVEY §8(f) "next"
row: a word LM whose mini-batches have PTB-like sentence lengths, run three ways through the C ABI:

  bucketed    : 5 buckets 13/18/24/30/83 (the paper's PTB calibration), each explored by the tuner
                on live steps, then replayed (one CUDA graph per bucket);
  exact_length: every length its own shape, default variant, eager launches — the analogue of the
                paper's "dynamic graph" baseline (no padding, no exploration);
  pad_to_max  : every mini-batch padded to 83 (one bucket), explored and replayed.

Shapes: the cfg2 word-LM sizes (H = I = 1024, V = 10k; SCRN context S = 1024) at the paper's
Table 8 batch sizes 16 and 32.  Lengths ~ synth.ptb_like_lengths; tokens Zipf over V.  Prints one
JSON line per (cell, batch): sentences/s and real tokens/s for each mode.

  python bench_buckets.py [--cells scrn,sublstm] [--batches 16,32] [--steps 300]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

BUCKETS = [13, 18, 24, 30, 83]
H = I = S = 1024
V = 10000
TMAX = 83
SEED = 20190413 + 1000 * 2 + 500


def params(cell):
    import synth
    if cell == "scrn":
        shapes = {"A": (I, H), "Bm": (I, S), "P": (S, H), "R": (H, H), "b_h": (H,)}
        hout = H + S
    else:
        shapes = {"W": (I, 4 * H), "U": (H, 4 * H), "b": (4 * H,)}
        hout = H
    shapes.update({"E": (V, I), "W_o": (hout, V), "b_o": (V,)})
    return synth.weights(SEED, shapes, H)


def run_mode(A, torch, cell, B, mode, lengths_explore, lengths_time, tok):
    kw = {"context": S, "scrn_alpha": 0.95} if cell == "scrn" else {}
    c = A.Cell(cell, H, I, B, TMAX, dtype="bf16", **kw)
    m = A.LM(c, V)
    m.load(params(cell))
    explore = 0
    if mode == "bucketed":
        m.set_buckets(BUCKETS)
    elif mode == "exact_length":
        m.set_buckets(list(range(1, TMAX + 1)))
        m.set_graph(False)
    if mode == "exact_length":
        c.tune_mode(A.TUNE_OFF)
    else:
        c.tune_mode(A.TUNE_ON)
        for L in lengths_explore:   # work-conserving exploration on live steps, until every bucket converged
            m.train_step_len(tok[:L + 1], int(L), 0.01)
            c.tune_next()
            explore += 1
            rep = c.tune_report()
            buckets = [rep] + list(rep.get("other_buckets", {}).values())
            seen = 1 + len(rep.get("other_buckets", {}))
            want = len(BUCKETS) if mode == "bucketed" else 1
            if seen >= want and all(b.get("converged") for b in buckets):
                break
    for L in lengths_time[:10]:   # warm-up (graph captures, tensor maps of every shape)
        m.train_step_len(tok[:L + 1], int(L), 0.01)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for L in lengths_time:
        m.train_step_len(tok[:L + 1], int(L), 0.01)
    e1.record()
    torch.cuda.synchronize()
    sec = e0.elapsed_time(e1) / 1e3
    rep = c.tune_report()
    n_cfg = {str(rep.get("bucket")): rep.get("configs_explored", 0)}
    for k, v in rep.get("other_buckets", {}).items():
        n_cfg[k] = v.get("configs_explored", 0)
    return {"sentences_per_s": len(lengths_time) * B / sec, "tokens_per_s": float(sum(lengths_time)) * B / sec,
            "ms_per_step": 1e3 * sec / len(lengths_time), "explore_steps": explore, "configs_per_bucket": n_cfg}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cells", default="scrn,sublstm")
    ap.add_argument("--batches", default="16,32")
    ap.add_argument("--steps", type=int, default=300)
    ap.add_argument("--max-explore", type=int, default=2500)
    a = ap.parse_args()
    import torch
    import paper_conf_asplos_sivathanucsz19_b200 as A
    import synth
    lex = synth.ptb_like_lengths(SEED, "lengths/explore", a.max_explore)
    ltm = synth.ptb_like_lengths(SEED, "lengths/timed", a.steps)
    for cell in a.cells.split(","):
        for B in [int(x) for x in a.batches.split(",")]:
            tok = torch.as_tensor(synth.zipf_tokens(SEED, "tokens", (TMAX + 1, B), V), dtype=torch.int32,
                                  device="cuda")
            res = {m: run_mode(A, torch, cell, B, m, lex, ltm, tok) for m in ("bucketed", "exact_length", "pad_to_max")}
            line = {"metric": "bucketed word-LM train sentences/s", "cell": cell, "batch": B, "hidden": H,
                    "vocab": V, "buckets": BUCKETS, "timed_steps": a.steps,
                    "mean_len": float(sum(ltm)) / len(ltm), "dtype": "bf16", "data": "synthetic", **res,
                    "speedup_vs_exact_length": res["bucketed"]["sentences_per_s"] / res["exact_length"]["sentences_per_s"],
                    "speedup_vs_pad_to_max": res["bucketed"]["sentences_per_s"] / res["pad_to_max"]["sentences_per_s"]}
            print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
