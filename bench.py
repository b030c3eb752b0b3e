"""Benchmark: custom-RNN training samples/s on B200 (BASELINE.json metric), workload = cfg5
(BASELINE.json configs[4]): MI-LSTM char LM, hidden 2048, GLOBAL batch 512, seq 100, data-parallel
over N GPUs.  Default: strong scaling as BASELINE configs[4] and SURVEY §8(d.1) state — the global
batch stays 512 and each of the N ranks trains its contiguous shard of 512/N sequences; `--weak`
gives every rank its own 512 sequences instead (global batch 512·N).  One step = embedding →
MI-LSTM forward → head + CE → BPTT → weight gradients → gradient all-reduce (N > 1) → SGD, all in
the library's kernels through the C ABI.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl astra|reference]

Prints ONE JSON line on rank 0.  `--impl reference` times the fp64 CPU oracle (the paper
publishes no code, so the oracle is the reference arm) on a bounded sample of the same workload:
every step is one full fwd + bwd + SGD step over 64 of the sequences (so its BLAS calls are GEMMs,
not GEMVs), W warm-up steps and K timed steps, and the line states the steps, batch and per-step
time it actually ran.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOAD = {"workload": "cfg5: MI-LSTM char LM (BASELINE.json configs[4])", "cell": "milstm", "hidden": 2048,
            "input": 2048, "global_batch": 512, "seq_len": 100, "vocab": 256, "symbols": 205}
CFG_SEED = 20190413 + 1000 * 5
METRIC = "custom-RNN train samples/s"


def flops_per_sample(T, H, I, V):
    """Algorithmic FLOPs per sequence: 3x the cell's forward GEMM flops + head."""
    return 24.0 * T * H * (I + H) + 6.0 * T * H * V


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            mp = json.load(f)
        return mp["bf16_tflops"], mp["bf16_tflops_sustained"], mp["hbm_gbs"], "measured"
    except Exception:
        return 1590.0, 1400.0, 6650.0, "fallback (B200_PROFILING.md)"


def a1_traffic():
    """DRAM bytes (read + write) per launch of the a1 GEMM from the committed ncu --set full capture
    (profiles/r2_roofline_traffic.json: the round-2 ncu --set full capture of the tuned variant's a1)."""
    try:
        with open(os.path.join(ROOT, "profiles", "r2_roofline_traffic.json")) as f:
            return json.load(f)["a1_dram_bytes_per_launch"]
    except Exception:
        return None


class Clocks:
    """nvidia-smi clock/throttle sampling during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, index):
        self.index = index
        self.p = None
        self.path = os.path.join(ROOT, "gpurun_out", f"clocks_{os.getpid()}.csv")

    def __enter__(self):
        try:
            os.makedirs(os.path.dirname(self.path), exist_ok=True)
            self.f = open(self.path, "w")
            self.p = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=clocks.sm,clocks.max.sm,power.draw,"
                 "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                 "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap",
                 "--format=csv,noheader,nounits", "-lms", "50"], stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None
        return self

    def __exit__(self, *a):
        if self.p is not None:
            self.p.terminate()
            try:
                self.p.wait(timeout=5)
            except Exception:
                self.p.kill()
            self.f.close()

    def summary(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        rows = []
        for line in open(self.path):
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 7:
                try:
                    rows.append(parts)
                except Exception:
                    pass
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        sm = [float(r[0]) for r in rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[3 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


def make_inputs(B_g, T, V, n_sym, rank, world):
    import synth
    tok = synth.zipf_tokens(CFG_SEED, "tokens", (T + 1, B_g), V, n_sym)
    b = B_g // world
    return tok[:, rank * b:(rank + 1) * b].copy()


def make_params(I, H, V):
    import synth
    shapes = {"W": (I, 4 * H), "U": (H, 4 * H), "b": (4 * H,), "alpha": (4 * H,), "beta1": (4 * H,),
              "beta2": (4 * H,), "E": (V, I), "W_o": (H, V), "b_o": (V,)}
    p = synth.weights(CFG_SEED, shapes, H, {"alpha": (1.0, 1.0), "beta1": (0.5, 0.5), "beta2": (0.5, 0.5)})
    return p


# ------------------------------------------------------------------------------------------ oracle
ORACLE_SAMPLE_B = 64   # sequences per oracle step: GEMM-shaped BLAS calls (B=4 was GEMV-bound)


def host_info():
    """The host the oracle runs on: logical cores, CPU model, BLAS threads."""
    from threadpoolctl import threadpool_info
    model = None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    threads = max([i.get("num_threads", 1) for i in threadpool_info()] + [1])
    return {"cores": threads, "cpu_count": os.cpu_count(), "cpu_model": model}


def run_oracle(T, H, I, V, n_sym, B_sample, steps=1, warm=0):
    """Time the fp64 numpy oracle (as it stands) on a bounded sample of the workload: `warm`
    untimed then `steps` timed fwd + bwd + SGD steps over B_sample sequences (state not carried,
    parameters updated).  Returns (samples/s, seconds per step)."""
    import numpy as np
    from oracle import lm as OLM
    import synth
    p = make_params(I, H, V)
    tok = synth.zipf_tokens(CFG_SEED, "tokens", (T + 1, B_sample), V, n_sym)
    h0 = np.zeros((B_sample, H))
    c0 = np.zeros((B_sample, H))
    for _ in range(warm):
        _, p, _, _ = OLM.lm_train_step("milstm", p, tok, h0, c0, 0.1)
    t0 = time.perf_counter()
    for _ in range(steps):
        loss, p, _, _ = OLM.lm_train_step("milstm", p, tok, h0, c0, 0.1)
    dt = (time.perf_counter() - t0) / steps
    return B_sample / dt, dt


# ------------------------------------------------------------------------------------------ main
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="astra", choices=["astra", "reference"])
    ap.add_argument("--no-tune", action="store_true")
    ap.add_argument("--tune-warmup", type=int, default=0,
                    help="untimed steps before the exploration starts (settles the power-capped SM clock)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--profile", action="store_true", help="1 warm-up + --steps steps, nothing else (for ncu)")
    ap.add_argument("--batch", type=int, default=None, help="override the global batch (strong) / per-rank batch (weak)")
    ap.add_argument("--weak", action="store_true", help="every rank trains its own --batch sequences (global batch x N)")
    ap.add_argument("--seq", type=int, default=None, help="override seq (debug)")
    ap.add_argument("--dp", default="nccl", choices=["nccl", "peer"],
                    help="N > 1 gradient sum: NCCL all-reduce (K11) or the deterministic peer-memory "
                         "reduce-scatter + fused SGD / all-gather over NVLink (K11p)")
    args = ap.parse_args()

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    T = args.seq or WORKLOAD["seq_len"]
    H, I, V, n_sym = WORKLOAD["hidden"], WORKLOAD["input"], WORKLOAD["vocab"], WORKLOAD["symbols"]
    B_unit = args.batch or WORKLOAD["global_batch"]
    B_g = B_unit * max(world, 1) if args.weak else B_unit     # global batch of this run
    scaling = "weak" if args.weak else "strong"
    cfg = {"workload": WORKLOAD["workload"], "cell": "MI-LSTM", "hidden": H, "input": I, "global_batch": B_g,
           "seq_len": T, "vocab": V, "parallelism": f"dp{args.gpus}", "dp_backend": args.dp, "per_gpu_batch": B_g // max(world, 1),
           "l2": "working set per step (GB of activations, 139 MB of fp32 grads) >> 126 MB L2: inputs larger than L2"}

    if args.impl == "reference":
        if rank != 0:
            return
        Bs = min(ORACLE_SAMPLE_B, B_g)
        wall0 = time.perf_counter()
        val, dt = run_oracle(T, H, I, V, n_sym, Bs, steps=args.steps, warm=args.warmup)
        hi = host_info()
        sample = (f"each step: {Bs} of the {B_g} sequences (T={T}, H=I=2048, V=256), one full fwd+bwd+SGD step "
                  f"of the fp64 numpy oracle; {args.warmup} warm-up + {args.steps} timed steps, "
                  f"{time.perf_counter() - wall0:.1f} s wall")
        line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "samples/s", "n_gpus": args.gpus,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3,
                "samples_per_step": Bs, "higher_is_better": True, "scaling": scaling, "vs_baseline": None,
                "dtype": "f64", "data": "synthetic (seeded Zipf tokens, random-init weights)", "config": cfg,
                "cpu_baseline": {"value": val, "unit": "samples/s", "kind": "oracle", "sample": sample, **hi},
                "e2e": {"value": val, "unit": "samples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line), flush=True)
        return

    import numpy as np
    import torch
    import torch.distributed as dist
    import paper_conf_asplos_sivathanucsz19_b200 as A

    torch.cuda.set_device(local)
    distributed = "RANK" in os.environ          # launched by torch.distributed.run (any N, incl. 1)
    if distributed:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    B = B_g // world
    dev = torch.device("cuda", local)

    cell = A.Cell("milstm", H, I, B, T, dtype="bf16", device=local)
    lm = A.LM(cell, V)
    lm.load(make_params(I, H, V))
    if distributed:   # the process group only broadcasts the NCCL id; the library owns the comm (K11)
        uid = [A.comm_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        lm.comm_init(uid[0], rank, world)   # one communicator for the LM; also the tuner's cross-rank decisions (R29)
        if args.dp == "peer" and world > 1:
            A.peer_exchange(lm)
    tok_host = torch.as_tensor(make_inputs(B_g, T, V, n_sym, rank, world), dtype=torch.int32).pin_memory()
    tokens = tok_host.to(dev)
    lr = 0.05
    st = torch.cuda.current_stream()

    def barrier():
        torch.cuda.synchronize()
        if distributed:
            dist.barrier()
            torch.cuda.synchronize()

    if args.profile:
        if os.environ.get("ASTRA_VARIANT"):
            cell.tune_mode(A.TUNE_FROZEN, os.environ["ASTRA_VARIANT"])
        cell.set_profiling(2)   # the phase regions too (diagnostics)
        lm.train_step(tokens, lr)
        torch.cuda.synchronize()
        for _ in range(args.steps):
            lm.train_step(tokens, lr)
        torch.cuda.synchronize()
        print(json.dumps({"profile_steps": args.steps, "regions_ms": region_times(cell)}))
        return
    # ---- online exploration (work-conserving: every explored step is a real training step)
    tune_steps, tune_t0 = 0, time.perf_counter()
    tune_info = {"mode": "off"}
    if args.no_tune and os.environ.get("ASTRA_VARIANT"):   # A/B runs: a forced variant, no exploration
        cell.tune_mode(A.TUNE_FROZEN, os.environ["ASTRA_VARIANT"])
        tune_info = {"mode": "frozen (ASTRA_VARIANT)", "variant": os.environ["ASTRA_VARIANT"]}
    if not args.no_tune:
        for _ in range(args.tune_warmup):   # real training steps at the default variant
            lm.train_step(tokens, lr)
        cell.tune_mode(A.TUNE_ON)
        while True:
            lm.train_step(tokens, lr)
            tune_steps += 1
            s = cell.tune_next()
            if s == A.TUNE_CONVERGED or tune_steps > 1000:
                break
        torch.cuda.synchronize()
        rep = cell.tune_report()
        if os.environ.get("ASTRA_DUMP_REPORT"):   # diagnostics: the tuner's profile index
            with open(os.environ["ASTRA_DUMP_REPORT"], "w") as f:
                json.dump(rep, f)
        cell.tune_mode(A.TUNE_FROZEN, rep["variant"])
        tune_info = {"mode": "explored then frozen", "converged": s == A.TUNE_CONVERGED, "steps": tune_steps,
                     "configs_explored": rep.get("configs_explored"), "harvest_waits": rep.get("harvest_waits"),
                     "wall_s": round(time.perf_counter() - tune_t0, 3), "variant": rep["variant"]}
    # ---- warm-up, then the timed region (device time, CUDA events on the launching stream; max
    # over ranks).  nvidia-smi samples clocks from the last warm-up steps through the timed region.
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with Clocks(local) as clk:
        for _ in range(max(3, args.warmup)):
            lm.train_step(tokens, lr)
        barrier()
        l0 = A.launch_count()
        barrier()
        e0.record(st)
        for _ in range(args.steps):
            lm.train_step(tokens, lr)
        e1.record(st)
        torch.cuda.synchronize()
    launches = (A.launch_count() - l0) // args.steps
    ms = e0.elapsed_time(e1) / args.steps
    t = torch.tensor([ms], device=dev)
    if distributed:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms = float(t.item())
    value = B_g / (ms / 1e3)

    # ---- profiling overhead ("<0.5%"): the same frozen steps with the region events on and
    # off, in interleaved windows (clocks drift under the power cap: one pair of windows is noise)
    def window(on, n):
        cell.set_profiling(on)
        lm.train_step(tokens, lr)          # (re)captures the step graph of this mode outside the window
        barrier()
        g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        g0.record(st)
        for _ in range(n):
            lm.train_step(tokens, lr)
        g1.record(st)
        torch.cuda.synchronize()
        return g0.elapsed_time(g1) / n
    n_win = 6
    per = max(3, min(args.steps, 10))
    pairs = []
    for w in range(n_win):
        order = (True, False) if w % 2 == 0 else (False, True)
        r = {o: window(o, per) for o in order}
        pairs.append(100.0 * (r[True] - r[False]) / r[False])
    cell.set_profiling(True)
    pairs.sort()

    # ---- dominant kernel live: the hoisted a1 GEMM region (one K1 launch, on the main stream)
    region = cell_region_ms(cell, lm, tokens, lr, steps=3)

    # ---- end-to-end through the C ABI with host buffers (H2D tokens + D2H loss every step)
    host_loss = torch.empty(1, dtype=torch.float32).pin_memory()
    barrier()
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    f0.record(st)
    for _ in range(args.steps):
        tokens.copy_(tok_host, non_blocking=True)
        lm.train_step(tokens, lr)
        host_loss.copy_(lm.loss, non_blocking=True)
    f1.record(st)
    torch.cuda.synchronize()
    ms_e2e = f0.elapsed_time(f1) / args.steps
    t = torch.tensor([ms_e2e], device=dev)
    if distributed:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_e2e = float(t.item())

    if rank == 0:
        burst, sustained, hbm, src = peaks()
        fl = flops_per_sample(T, H, I, V)
        a1_flops = 2.0 * (T * B) * I * (4 * H)
        a1_tf = a1_flops / (region["a1_ms"] / 1e3) / 1e12 if region.get("a1_ms") else None
        step_tf = value * fl / 1e12
        line = {
            "metric": METRIC, "value": value, "unit": "samples/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": max(3, args.warmup), "ms_per_step": ms, "higher_is_better": True, "scaling": scaling,
            "vs_baseline": None, "dtype": "bf16", "data": "synthetic (seeded Zipf tokens over 205 symbols, "
            "random-init weights)", "config": cfg,
            "tokens_per_s": value * T,
            "roofline": {"bound": "tensor", "kernel": "K1 tcgen05 GEMM, hoisted input projection a1 "
                         f"[{T*B}x{I}]x[{I}x{4*H}]", "achieved": a1_tf, "peak": burst, "unit": "TFLOP/s",
                         "frac": (a1_tf / burst) if a1_tf else None, "traffic": a1_traffic(),
                         "peak_source": f"{src} bf16_tflops (burst): a1 is the first GEMM of a step launched after "
                                        "a device synchronize, so it runs at burst clocks (it exceeds the "
                                        f"sustained figure {sustained})",
                         "step_tflops": step_tf, "step_frac_of_sustained": step_tf / (sustained * args.gpus)},
            "regions_ms": region,
            "e2e": {"value": B_g / (ms_e2e / 1e3), "unit": "samples/s", "h2d_bytes_per_step": int(tok_host.numel() * 4),
                    "d2h_bytes_per_step": 4},
            "gpu_launches": int(launches),
            "profiling_overhead": {"pct": statistics.median(pairs), "min_pct": pairs[0], "max_pct": pairs[-1],
                                   "windows": n_win, "steps_per_window": per,
                                   "method": "median over interleaved region-events on/off window pairs"},
            "clocks": clk.summary(),
            "tuner": tune_info,
        }
        if not args.no_cpu_baseline:
            try:
                Bs = min(ORACLE_SAMPLE_B, B_g)
                val, dt = run_oracle(T, H, I, V, n_sym, Bs, steps=1)
                line["cpu_baseline"] = {"value": val, "unit": "samples/s", "kind": "oracle",
                                        "sample": f"{Bs} sequences of the cfg5 workload (T={T}, H=I=2048, V=256), "
                                                  f"one fwd+bwd+SGD step, fp64 numpy, {dt:.1f} s", **host_info()}
            except Exception as e:  # pragma: no cover
                line["cpu_baseline"] = {"value": None, "error": str(e)}
        print(json.dumps(line), flush=True)
    if distributed:
        dist.barrier()
        dist.destroy_process_group()


def cell_region_ms(cell, lm, tokens, lr, steps=3):
    """Per-region device times from the library's own cudaEvent pairs, min over steps."""
    import torch
    out = {}
    cell.set_profiling(2)   # phase regions for these diagnostic steps (the timed ones record the step only)
    keys = {"a1_ms": "t_a1", "fwd_chain_ms": "t_fwd", "bptt_chain_ms": "t_bptt", "head_ms": "t_head",
            "wgrad_ms": "t_se4", "step_ms": "t_step"}
    for _ in range(steps):
        lm.train_step(tokens, lr)
        torch.cuda.synchronize()
        r = region_times(cell)
        for k, v in r.items():
            out[k] = min(out.get(k, 1e30), v)
    cell.set_profiling(1)   # back to the always-on level
    return out


def region_times(cell):
    import ctypes
    import paper_conf_asplos_sivathanucsz19_b200 as A
    buf = (ctypes.c_double * 16)()
    n = ctypes.c_int()
    A._check(A.lib().astra_region_times(cell.h, buf, 16, ctypes.byref(n)))
    names = ["a1_ms", "fwd_chain_ms", "head_ms", "bptt_chain_ms", "du_ms", "dw_ms", "dx_ms", "wgrad_ms", "step_ms"]
    return {names[i]: buf[i] for i in range(min(n.value, len(names)))}


if __name__ == "__main__":
    main()
