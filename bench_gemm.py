"""K1 microbenchmarks: the tcgen05 GEMM at the shapes of one cfg5 training step
and at the paper's Table 1 / fusion-example shapes, for every tile
width / cluster shape.  Device time from CUDA events over many back-to-back launches.

  python bench_gemm.py [--quick]
Launches are replayed from a CUDA graph (no host overhead in the device time).
Prints one JSON line per (shape, layout, config) with TFLOP/s and the fraction of the measured
bf16 peak (MEASURED_PEAKS.json, burst figure: kernels timed alone).
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
import paper_conf_asplos_sivathanucsz19_b200 as A  # noqa: E402

SHAPES = [  # name, M, N, K, a_mn, b_mn
    ("cfg5 a1 X·W", 51200, 8192, 2048, 0, 0),
    ("cfg5 rec h·U (per step)", 512, 8192, 2048, 0, 0),
    ("cfg5 bptt d·Uᵀ (per step, MN-major U)", 512, 2048, 8192, 0, 1),
    ("cfg5 bptt d·Uᵀ (per step, K-major U copy)", 512, 2048, 8192, 0, 0),
    ("cfg5 dU = Hᵀ·D", 2048, 8192, 51200, 1, 1),
    ("cfg5 dX = D·Wᵀ", 51200, 2048, 8192, 0, 1),
    ("Table 1 fwd 64x1024x4096", 64, 4096, 1024, 0, 0),
    ("Table 1 bwd 64x4096x1024", 64, 1024, 4096, 0, 0),
    ("P:122 fused 512x1024x1024", 512, 1024, 1024, 0, 0),
]
CONFIGS = [(256, 1, 1), (128, 1, 1), (64, 1, 1), (256, 1, 1, 2), (128, 1, 1, 2), (256, 2, 1), (256, 1, 2),
           (256, 2, 2), (128, 2, 2), (64, 2, 2), (128, 4, 1), (64, 4, 2), (128, 4, 2)]


def peak():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["bf16_tflops"]
    except Exception:
        return 1590.0


def run(name, M, N, K, a_mn, b_mn, cfgs, reps):
    dev = torch.device("cuda")
    As = torch.randn((K, M) if a_mn else (M, K), device=dev).to(torch.bfloat16)
    Bs = torch.randn((K, N) if b_mn else (N, K), device=dev).to(torch.bfloat16)
    out = torch.empty(1, M, N, device=dev)
    pk = peak()
    for cfg in cfgs:
        bn, cm, cn = cfg[:3]
        cg = cfg[3] if len(cfg) > 3 else 1
        try:
            for _ in range(3):
                A.gemm_bf16_ex(As, Bs, M, N, K, a_mn, b_mn, bn, cm, cn, cg, out=out)
            torch.cuda.synchronize()
            # replay the launches from a CUDA graph: device time without host launch overhead
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                for _ in range(reps):
                    A.gemm_bf16_ex(As, Bs, M, N, K, a_mn, b_mn, bn, cm, cn, cg, out=out)
            g.replay()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record()
            g.replay()
            e1.record()
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / reps
            tf = 2.0 * M * N * K / (ms * 1e-3) / 1e12
            print(json.dumps({"shape": name, "M": M, "N": N, "K": K, "a_mn": a_mn, "b_mn": b_mn,
                              "cfg": ".".join(map(str, cfg)), "us": round(ms * 1e3, 2), "tflops": round(tf, 1),
                              "frac_of_peak": round(tf / pk, 3)}), flush=True)
        except A.AstraError as e:
            print(json.dumps({"shape": name, "cfg": ".".join(map(str, cfg)), "error": str(e)[:80]}), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--all", action="store_true")
    ap.add_argument("--shapes", default="", help="comma-separated substrings of shape names to run")
    args = ap.parse_args()
    for s in SHAPES:
        if args.shapes and not any(k in s[0] for k in args.shapes.split(",")):
            continue
        big = s[1] * s[2] * s[3] > 1e11
        run(*s, CONFIGS[:5] if args.quick else CONFIGS if args.all else CONFIGS, 5 if big else 50)


if __name__ == "__main__":
    main()
