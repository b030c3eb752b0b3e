"""Day-1 microbenchmarks of SURVEY §8(d.4b) and the chain-latency floors of §8(d.3), on one B200.

  python bench_micro.py [--json out.json]

Measures, through the library's own kernels (astra_micro_*):
  - streaming-read bandwidth by buffer size (L2-resident vs HBM): the per-step weight-stream time;
  - grid-wide flag-barrier latency of a persistent one-CTA-per-SM kernel;
  - the per-kernel latency of a chain of dependent launches (PDL on / off, eager / CUDA graph);
then derives, per BASELINE config, the floor of one dependent recurrent step — max(launch floor,
weight bytes / bandwidth at that size) per launched kernel of the step — against which the chains'
measured µs per step are reported in DESIGN.md §6b.  Prints one JSON object.
"""
from __future__ import annotations

import argparse
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--json", default=None)
    args = ap.parse_args()
    import torch
    import paper_conf_asplos_sivathanucsz19_b200 as A
    L = A.lib()
    st = torch.cuda.current_stream()
    sp = ctypes.c_void_p(st.cuda_stream)
    ev = lambda: torch.cuda.Event(enable_timing=True)

    def timed(fn, reps=3):
        best = None
        for _ in range(reps):
            torch.cuda.synchronize()
            a, b = ev(), ev()
            a.record()
            fn()
            b.record()
            torch.cuda.synchronize()
            t = a.elapsed_time(b)
            best = t if best is None else min(best, t)
        return best   # ms

    out = {"device": torch.cuda.get_device_name(0),
           "l2_bytes": torch.cuda.get_device_properties(0).L2_cache_size,
           "sms": torch.cuda.get_device_properties(0).multi_processor_count}
    sink = torch.zeros(1, device="cuda")
    # streaming read by size
    bw = {}
    for mb in (2, 4, 8, 16, 32, 48, 64, 96, 128, 256, 1024):
        nbytes = mb << 20
        buf = torch.rand(nbytes // 4, device="cuda")
        passes = max(3, (4 << 30) // nbytes)
        A._check(L.astra_micro_stream_read(A._ptr(buf), nbytes, 1, A._ptr(sink), sp))   # warm
        ms = timed(lambda: A._check(L.astra_micro_stream_read(A._ptr(buf), nbytes, passes, A._ptr(sink), sp)))
        bw[mb] = nbytes * passes / (ms / 1e3) / 1e9
        del buf
    out["stream_read_gbs"] = {str(k): round(v, 1) for k, v in bw.items()}
    # grid barrier
    ctr = torch.zeros(16, dtype=torch.int32, device="cuda")
    iters = 20000
    ms = timed(lambda: A._check(L.astra_micro_grid_barrier(A._ptr(ctr), iters, sp)))
    out["grid_barrier_us"] = round(ms * 1e3 / iters, 3)
    # launch chains
    chain = {}
    n = 2000
    for pdl in (1, 0):
        for blocks in (148, 592):
            ms = timed(lambda: A._check(L.astra_micro_launch_chain(n, pdl, blocks, sp)))
            chain[f"eager_pdl{pdl}_b{blocks}"] = round(ms * 1e3 / n, 3)
            g = torch.cuda.CUDAGraph()
            s2 = torch.cuda.Stream()
            with torch.cuda.stream(s2):
                with torch.cuda.graph(g, stream=s2):
                    A._check(L.astra_micro_launch_chain(n, pdl, blocks, ctypes.c_void_p(s2.cuda_stream)))
            g.replay()
            ms = timed(lambda: g.replay())
            chain[f"graph_pdl{pdl}_b{blocks}"] = round(ms * 1e3 / n, 3)
    out["launch_chain_us_per_kernel"] = chain
    # K11p: the rank-ordered reduce kernel with N simulated ranks on this device (local HBM, not
    # NVLink): one round reads every rank's cfg5-sized gradient buffer once and writes it once
    n = 34_640_000   # cfg5 flat gradient (139 MB)
    k11p = {}
    seq = 1
    for world in (2, 4, 8):
        bufs = [torch.rand(n, device="cuda") for _ in range(world)]
        sigs = [torch.zeros(1024, dtype=torch.int32, device="cuda") for _ in range(world)]
        streams = [torch.cuda.Stream() for _ in range(world)]
        bp = (ctypes.c_void_p * world)(*[b.data_ptr() for b in bufs])
        sgp = (ctypes.c_void_p * world)(*[g.data_ptr() for g in sigs])
        stp = (ctypes.c_void_p * world)(*[x.cuda_stream for x in streams])
        reps = 5

        def run(r=reps):
            nonlocal seq
            e0 = torch.cuda.Event()
            e0.record(st)
            for x in streams:
                x.wait_event(e0)
            A._check(L.astra_micro_peer_reduce(ctypes.cast(bp, ctypes.c_void_p), ctypes.cast(sgp, ctypes.c_void_p),
                                               world, n, r, seq, ctypes.cast(stp, ctypes.c_void_p)))
            seq += r
            for x in streams:
                e = torch.cuda.Event()
                e.record(x)
                st.wait_event(e)

        run(1)
        ms = timed(run) / reps
        gbs = 4.0 * n * (world + 1) / (ms / 1e3) / 1e9
        k11p[str(world)] = {"ms_per_round": round(ms, 4), "gbs": round(gbs, 1), "frac_of_hbm": round(gbs / bw[1024], 3)}
        del bufs
    out["k11p_reduce_local"] = k11p
    # per-config floors of one dependent chain step (bf16 weight bytes streamed per launched GEMM)
    launch = chain["graph_pdl1_b148"]

    def bw_at(nbytes):
        mb = nbytes / (1 << 20)
        for k in sorted(bw):
            if mb <= k:
                return bw[k]
        return bw[max(bw)]

    cfgs = {
        # name: (kernels per dependent step, weight bytes streamed per step, dependent steps per direction)
        "cfg2_scrn": (2, 1024 * 1024 * 2, 35),             # h·R GEMM + sigmoid kernel
        "cfg3_rhn": (2, 830 * 1660 * 2, 350),              # per micro-step: s·R_l GEMM + highway kernel
        "cfg4_attn_decoder": (4, 1024 * 5120 * 2 + 1024 * 4096 * 2, 50),
        "cfg5_milstm": (2, 2048 * 8192 * 2, 100),          # h·U GEMM + gate kernel
    }
    floors = {}
    for name, (k, wb, steps) in cfgs.items():
        stream_us = wb / (bw_at(wb) * 1e9) * 1e6
        floors[name] = {"kernels_per_step": k, "weight_mb": round(wb / 2**20, 2),
                        "weight_stream_us": round(stream_us, 2), "launch_floor_us": round(k * launch, 2),
                        "step_floor_us": round(max(k * launch, stream_us + (k - 1) * launch), 2),
                        "dependent_steps": steps}
    out["chain_step_floor"] = floors
    line = json.dumps(out)
    print(line)
    if args.json:
        with open(args.json, "w") as f:
            f.write(line + "\n")


if __name__ == "__main__":
    main()
