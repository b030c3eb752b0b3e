"""Cell-level parity of the CUDA path (through the C ABI) against the fp64 oracle on identical seeded
inputs: every output and every gradient, fp32 path ≤ 1e-4 and bf16 path ≤ 2e-2 relative L2
(BASELINE.json north_star; reading R18), plus bitwise equality across tuner variants."""
import numpy as np
import pytest
import torch

import synth
from oracle import cells as C

from helpers import TOL_BF16, TOL_FP32, make_cell_case, rel_err, run_gpu_cell

pytestmark = pytest.mark.gpu


ALPHA = 0.95


def _check(cell, T, B, I, H, dtype, seed, tol, variant=None, S=None, L=None):  # noqa: C901
    p, inp, dY, dhT, dcT = make_cell_case(cell, T, B, I, H, seed, bf16=(dtype == "bf16"), S=S, L=L)
    kw, okw = {}, {}
    if cell == "scrn":
        kw = {"context": S or H, "scrn_alpha": ALPHA}
        okw = {"alpha": np.float32(ALPHA).item()}
    if cell == "rhn":
        kw = {"depth": L}
    out_o, g_o = C.cell_fwd_bwd(cell, p, inp, dY, dhT, dcT, **okw)
    out_g, g_g, _ = run_gpu_cell(cell, p, inp, dY, dhT, dcT, dtype, variant, **kw)
    errs = {}
    for k in out_o:
        errs[k] = rel_err(out_g[k], out_o[k])
    for k in g_o:
        errs["d" + k if not k.startswith("d") else k] = rel_err(g_g[k], g_o[k])
    bad = {k: v for k, v in errs.items() if not v <= tol}
    assert not bad, (cell, dtype, (T, B, I, H), bad, errs)
    return errs


@pytest.mark.parametrize("cell", ["milstm", "lstm", "sublstm"])
def test_fp32_cfg1(cell):
    """BASELINE.json configs[0]: MI-LSTM H64 I32 B4 T8 fp32 (≤ 1e-4)."""
    _check(cell, 8, 4, 32, 64, "fp32", synth.config_seed(1), TOL_FP32)


@pytest.mark.parametrize("cell", ["milstm", "lstm", "sublstm"])
def test_fp32_ragged(cell):
    """Hidden/input sizes that are not multiples of the 64-unit gate block; tiny batch."""
    _check(cell, 5, 3, 20, 70, "fp32", synth.config_seed(1) + 11, TOL_FP32)


@pytest.mark.parametrize("cell", ["milstm", "lstm", "sublstm"])
def test_bf16_small(cell):
    _check(cell, 8, 4, 32, 64, "bf16", synth.config_seed(1) + 1, TOL_BF16)


@pytest.mark.parametrize("cell", ["milstm", "lstm"])
def test_bf16_multi_tile_ragged(cell):
    """Several M/N tiles and ragged tails: B=200 (2 row tiles), H=200 (Hp=256), I=72."""
    _check(cell, 6, 200, 72, 200, "bf16", synth.config_seed(5) + 2, TOL_BF16)


def test_bf16_cfg5_reduced():
    """cfg5 reduced rung: full H=I=2048 and per-GPU batch 64, T=8."""
    _check("milstm", 8, 64, 2048, 2048, "bf16", synth.config_seed(5), TOL_BF16)


@pytest.mark.parametrize("cell", ["milstm", "lstm", "sublstm"])
@pytest.mark.parametrize("fwd", [0, 1, 2])
def test_fused_forward_modes(cell, fwd):
    """K2 unfused / fused-per-step / fused-persistent against the oracle, several row blocks."""
    _check(cell, 6, 260, 64, 192, "bf16", synth.config_seed(5) + 40, TOL_BF16, variant=f"fwd={fwd}")


@pytest.mark.parametrize("cell", ["milstm", "lstm", "sublstm"])
@pytest.mark.parametrize("T,B,H", [(5, 64, 2048), (4, 100, 256), (3, 16, 200), (6, 1, 64)])
def test_small_batch_persistent_forward_bitwise(cell, T, B, H):
    """K2 small-batch persistent form (fwd=3: one cooperative launch, U slices resident in shared
    memory, fused gate epilogue, grid counter per step) gives the same bits as GEMM + pointwise
    (fwd=0) for every output and gradient — H = 2048 streams part of U (18 of 32 k-blocks resident),
    B = 100 uses 128-row A boxes, H = 200 has padding units, B = 1 a nearly empty tile — and also
    with the recompute context (no UH saved by the forward) and against the oracle."""
    I = 64
    p, inp, dY, dhT, dcT = make_cell_case(cell, T, B, I, H, 93, bf16=True)
    ref = None
    for v in ("fwd=0", "fwd=3", "fwd=3,rc=1"):
        out, g, _ = run_gpu_cell(cell, p, inp, dY, dhT, dcT, "bf16", v)
        cur = {**out, **g}
        if ref is None:
            ref = cur
            continue
        for k in ref:
            assert np.array_equal(ref[k], cur[k]), (v, k)
    _check(cell, T, B, I, H, "bf16", 93, TOL_BF16, variant="fwd=3")


@pytest.mark.parametrize("cell", ["milstm", "lstm", "sublstm"])
@pytest.mark.parametrize("T,B,H", [(5, 64, 2048), (4, 37, 2000), (3, 100, 2048), (1, 64, 2048)])
def test_small_batch_persistent_bptt_bitwise(cell, T, B, H):
    """K4 small-batch persistent BPTT (bwd=2: one cooperative launch of 4-CTA clusters, the R25
    chunk partials summed in chunk order over distributed shared memory, the cell backward fused,
    a counter per K chunk) gives the same bits as BPTT GEMM + pointwise (bwd=0) for every gradient,
    dx, dh0, dc0 — with the small-batch persistent forward too, B = 37 / H = 2000 (ragged rows and
    padding units), B = 100 (128-row A boxes), T = 1 (no GEMM step) — and against the oracle."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    I = 64
    p, inp, dY, dhT, dcT = make_cell_case(cell, T, B, I, H, 97, bf16=True)
    ref = None
    launches = {}
    for v in ("bwd=0", "bwd=2", "bwd=3,fwd=3"):
        n0 = A.launch_count()
        out, g, c = run_gpu_cell(cell, p, inp, dY, dhT, dcT, "bf16", v)
        launches[v] = A.launch_count() - n0
        cur = {**out, **g}
        if ref is None:
            ref = cur
            continue
        for k in ref:
            assert np.array_equal(ref[k], cur[k]), (v, k)
    if T > 1:   # the persistent chain really ran: one launch instead of a GEMM + pointwise per step
        assert launches["bwd=2"] <= launches["bwd=0"] - 2 * (T - 1) + 2, launches
    _check(cell, T, B, I, H, "bf16", 97, TOL_BF16, variant="bwd=2")


@pytest.mark.parametrize("gc", [1, 2, 3, 4])
def test_gate_chunking_bitwise(gc):
    """gate_chunking (§8(a.9), P:196 / P:220): the hoisted gate projection as 2 or 4 GEMMs over
    gate-column blocks, on one stream or alternating over two, gives the same bits as the
    one fused GEMM — outputs and every gradient — and the AV is in the live update tree."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H = 4, 96, 64, 320
    p, inp, dY, dhT, dcT = make_cell_case("milstm", T, B, I, H, 95, bf16=True)
    ref = None
    for v in ("gc=0", f"gc={gc}"):
        out, g, c = run_gpu_cell("milstm", p, inp, dY, dhT, dcT, "bf16", v)
        cur = {**out, **g}
        if ref is None:
            ref = cur
            continue
        for k in ref:
            assert np.array_equal(ref[k], cur[k]), (v, k)
    c.tune_mode(A.TUNE_ON)
    c.tune_next()
    assert "gate_chunking" in c.tune_report()["tree_avs"]


@pytest.mark.parametrize("cell", ["milstm", "lstm", "sublstm"])
@pytest.mark.parametrize("dtype", ["bf16", "fp32"])
@pytest.mark.parametrize("T,B,H", [(4, 100, 200), (3, 512, 2048), (5, 33, 130)])
def test_bwd_pointwise_forms_bitwise(cell, dtype, T, B, H):
    """The backward pointwise kernel's two forms (AV bwd_pw: the wide row x 4-unit kernel and the
    row-lane kernel) give the same bits — D_uh / D_wx, dc, and the fixed-order bias / α / β column
    sums (R5) — with ragged row chunks, padding units (H = 130, 200) and the R25 4-way split."""
    p, inp, dY, dhT, dcT = make_cell_case(cell, T, B, 64, H, 99, bf16=dtype == "bf16")
    ref = None
    for v in ("bpw=0", "bpw=1"):
        out, g, _ = run_gpu_cell(cell, p, inp, dY, dhT, dcT, dtype, v)
        cur = {**out, **g}
        if ref is None:
            ref = cur
            continue
        for k in ref:
            assert np.array_equal(ref[k], cur[k]), (v, k)
    if T * B * H <= 5 * 33 * 130:
        _check(cell, T, B, 64, H, dtype, 99, TOL_BF16 if dtype == "bf16" else TOL_FP32)


@pytest.mark.parametrize("cell", ["milstm", "lstm"])
@pytest.mark.parametrize("T,B,H", [(4, 256, 192), (5, 320, 130)])
@pytest.mark.parametrize("v", ["rsp=1", "rsp=1,bpw=1,wg_side=1"])
def test_row_streams_bitwise(cell, T, B, H, v):
    """row_streams (stream assignment): the batch's two row halves as independent chains on two
    streams (forward and BPTT) give the same bits as the one chain — outputs, every gradient, the
    fixed-order column sums — and the AV is in the live tree."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    p, inp, dY, dhT, dcT = make_cell_case(cell, T, B, 64, H, 103, bf16=True)
    ref = None
    for var in ("rsp=0", v):
        out, g, c = run_gpu_cell(cell, p, inp, dY, dhT, dcT, "bf16", var)
        cur = {**out, **g}
        if ref is None:
            ref = cur
            continue
        for k in ref:
            assert np.array_equal(ref[k], cur[k]), (var, k)
    c.tune_mode(A.TUNE_ON)
    c.tune_next()
    assert "row_streams" in c.tune_report()["tree_avs"]


@pytest.mark.parametrize("v", ["wgs=1", "wgs=2", "wgs=2,wg_side=1,rc=1", "wgs=1,hov=0,fwd=3"])
def test_wgrad_schedule_bitwise(v):
    """wgrad_schedule (§8(a.9)): the input dgrad in 4 / 10 time chunks on a side stream
    while BPTT is still running (with the dU side stream and the recompute context too) gives the
    same bits as dX after BPTT, and the AV is in the live update tree."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    T, B, I, H = 10, 64, 128, 192
    p, inp, dY, dhT, dcT = make_cell_case("milstm", T, B, I, H, 97, bf16=True)
    ref = None
    for var in ("wgs=0", v):
        out, g, c = run_gpu_cell("milstm", p, inp, dY, dhT, dcT, "bf16", var.replace(",hov=0", ""))
        cur = {**out, **g}
        if ref is None:
            ref = cur
            continue
        for k in ref:
            assert np.array_equal(ref[k], cur[k]), (var, k)
    c.tune_mode(A.TUNE_ON)
    c.tune_next()
    assert "wgrad_schedule" in c.tune_report()["tree_avs"]


@pytest.mark.parametrize("cell", ["lstm", "milstm", "sublstm"])
def test_fused_pair_forward_ragged(cell):
    """The CTA-pair fused forward (fwd=1): ragged batch (a half-empty CTA pair), hidden size not a
    multiple of the 32-unit epilogue slice (TMA-clipped tails), and the external y output."""
    _check(cell, 4, 300, 64, 100, "bf16", synth.config_seed(5) + 41, TOL_BF16, variant="fwd=1")


@pytest.mark.parametrize("cell", ["milstm", "lstm", "sublstm"])
@pytest.mark.parametrize("T,B,H", [(6, 260, 192), (4, 300, 128), (3, 64, 2048)])
def test_fused_bwd_bitwise(cell, T, B, H):
    """K4 fused (GEMM + cell backward in one kernel per step, bwd=1) gives the same bits as the
    BPTT GEMM + unfused pointwise kernel (bwd=0): ragged row tiles, split-K 1 / 4, and the oracle."""
    I = 64
    p, inp, dY, dhT, dcT = make_cell_case(cell, T, B, I, H, 91, bf16=True)
    ref = None
    for v in ("bwd=0", "bwd=1"):
        out, g, _ = run_gpu_cell(cell, p, inp, dY, dhT, dcT, "bf16", v)
        cur = {**out, **g}
        if ref is None:
            ref = cur
            continue
        for k in ref:
            assert np.array_equal(ref[k], cur[k]), (v, k)
    _check(cell, T, B, I, H, "bf16", 91, TOL_BF16, variant="bwd=1")


@pytest.mark.parametrize("cell", ["lstm", "milstm", "sublstm"])
@pytest.mark.parametrize("dtype,tol", [("fp32", TOL_FP32), ("bf16", TOL_BF16)])
def test_recompute_bitwise_and_parity(cell, dtype, tol, monkeypatch):
    """Recompute-vs-store fork: UH recomputed in BPTT from the saved h operands
    in 2-step chunks (the ring wraps at T = 6) — the same bits as the stored UH, and oracle parity."""
    monkeypatch.setenv("ASTRA_RC_STEPS", "2")
    T, B, I, H = 6, 72, 64, 96
    p, inp, dY, dhT, dcT = make_cell_case(cell, T, B, I, H, 78, bf16=dtype == "bf16")
    ref = None
    for v in ("rc=0", "rc=1", "rc=1,wg_side=1"):
        out, g, _ = run_gpu_cell(cell, p, inp, dY, dhT, dcT, dtype, v)
        cur = {**out, **g}
        if ref is None:
            ref = cur
            continue
        for k in ref:
            assert np.array_equal(ref[k], cur[k]), (v, k)
    _check(cell, T, B, I, H, dtype, 78, tol, variant="rc=1")


@pytest.mark.parametrize("cell", ["lstm", "milstm", "sublstm"])
@pytest.mark.parametrize("T,B,I,H", [(5, 72, 64, 96), (4, 160, 128, 192), (3, 64, 256, 1024)])
def test_gate_blocked_alloc_bitwise(cell, T, B, I, H):
    """The `alloc` fork's gate layout (reading R38): gate-blocked mirrors / gate tensors
    (gb=1) with the gate-contracting GEMMs (per-step BPTT dh_rec = D_uh·Uᵀ, input dgrad D_wx·Wᵀ)
    reading their k-blocks in the interleaved layout's order give the same bits as the gate-
    interleaved layout for every output and gradient — with per-gate a1 GEMMs (gc=2: the paper's G
    separate gate GEMMs; gc=4 on two streams), both backward pointwise forms, the chunked dX,
    CTA-pair BPTT GEMMs, the recompute context, and at H = 1024 the 2-way split-K BPTT GEMM —
    and match the oracle.  Hp > H (padding units) in the first case."""
    p, inp, dY, dhT, dcT = make_cell_case(cell, T, B, I, H, 91, bf16=True)
    out0, g0, _ = run_gpu_cell(cell, p, inp, dY, dhT, dcT, "bf16", "fwd=0")
    ref = {**out0, **g0}
    vs = ["gb=1", "gb=1,gc=2,bpw=1", "gb=1,gc=4,wg_side=1,wgs=1",
          "a1=256.1.1.2,rec=256.1.1.2,bptt=128.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,wg_side=0,fwd=0,gb=1",
          "gb=1,rc=1", "gb=1,fwd=2,bwd=1"]
    for v in vs:
        out, g, _ = run_gpu_cell(cell, p, inp, dY, dhT, dcT, "bf16", v)
        cur = {**out, **g}
        for k in ref:
            assert np.array_equal(ref[k], cur[k]), (v, k)
    _check(cell, T, B, I, H, "bf16", 91, TOL_BF16, variant="gb=1,gc=2")


def test_variants_bitwise():
    """Every tile-width / stream variant gives bitwise-identical outputs and gradients."""
    T, B, I, H = 6, 160, 128, 192
    p, inp, dY, dhT, dcT = make_cell_case("milstm", T, B, I, H, 77, bf16=True)
    variants = ["a1=256,rec=256,bptt=128,du=256,dw=256,dx=256,wg_side=0,fwd=0",
                "a1=128.2.2,rec=128.2.1,bptt=64.2.1,du=128.1.2,dw=128,dx=128.4.1,wg_side=1,fwd=0",
                "a1=64.4.1,rec=64,bptt=256.1.1,du=64.2.2,dw=64.2.1,dx=64.2.2,wg_side=0,fwd=1",
                "a1=256.2.2,rec=256.2.1,bptt=128.2.1,du=256.2.2,dw=256.1.2,dx=256.4.1,wg_side=1,fwd=2"]
    ref = None
    for v in variants:
        out, g, _ = run_gpu_cell("milstm", p, inp, dY, dhT, dcT, "bf16", v)
        cur = {**out, **g}
        if ref is None:
            ref = cur
            continue
        for k in ref:
            assert np.array_equal(ref[k], cur[k]), (v, k)


# ------------------------------------------------------------------ SCRN [22] and RHN [39]
@pytest.mark.parametrize("dtype,tol", [("fp32", TOL_FP32), ("bf16", TOL_BF16)])
def test_scrn_small(dtype, tol):
    _check("scrn", 6, 4, 32, 64, dtype, synth.config_seed(2) + 1, tol, S=40)


@pytest.mark.parametrize("dtype,tol", [("fp32", TOL_FP32), ("bf16", TOL_BF16)])
def test_scrn_ragged_multi_tile(dtype, tol):
    _check("scrn", 5, 130, 72, 100, dtype, synth.config_seed(2) + 2, tol, S=70)


@pytest.mark.parametrize("T,B,I,H,S", [(6, 64, 1024, 1024, 1024), (5, 33, 72, 200, 70), (3, 100, 64, 128, 40)])
def test_scrn_persistent_forward_bitwise(T, B, I, H, S):
    """SC-RNN's fused persistent h-chains — forward (fwd=1: one cooperative launch, R slices resident,
    the R33 split kept as TMEM accumulators, σ(Q + Σ partials + b_h) in the epilogue) and BPTT (bwd=1:
    dz·Rᵀ split likewise, dz = (dy + Σ partials)·h(1−h) and the db_h row-lane partials fused) — give
    the same bits as GEMM + pointwise per step for every output and gradient — cfg2's shapes
    (H = S = 1024, 4-way split), a ragged batch with padding units, a 128-row A box — and match the
    oracle."""
    p, inp, dY, dhT, dcT = make_cell_case("scrn", T, B, I, H, 101, bf16=True, S=S)
    kw = {"context": S, "scrn_alpha": ALPHA}
    ref = None
    for v in ("fwd=0", "fwd=1", "bwd=1", "fwd=1,bwd=1"):
        out, g, _ = run_gpu_cell("scrn", p, inp, dY, dhT, dcT, "bf16", v, **kw)
        cur = {**out, **g}
        if ref is None:
            ref = cur
            continue
        for k in ref:
            assert np.array_equal(ref[k], cur[k]), (v, k)
    if T * B * H <= 5 * 33 * 200:
        _check("scrn", T, B, I, H, "bf16", 101, TOL_BF16, variant="fwd=1,bwd=1", S=S)


def test_scrn_cfg2_reduced():
    """cfg2 reduced rung: H = S = I = 1024, B = 64, T = 8 (bf16)."""
    _check("scrn", 8, 64, 1024, 1024, "bf16", synth.config_seed(2), TOL_BF16, S=1024)


@pytest.mark.parametrize("dtype,tol", [("fp32", TOL_FP32), ("bf16", TOL_BF16)])
def test_rhn_small(dtype, tol):
    _check("rhn", 4, 4, 32, 64, dtype, synth.config_seed(3) + 1, tol, L=3)


@pytest.mark.parametrize("dtype,tol", [("fp32", TOL_FP32), ("bf16", TOL_BF16)])
def test_rhn_ragged(dtype, tol):
    """H = 830 is the cfg3 hidden size (not a multiple of 64: padded internally)."""
    _check("rhn", 3, 20, 72, 830, dtype, synth.config_seed(3) + 2, tol, L=2)


@pytest.mark.parametrize("T,B,I,H,L", [(3, 4, 32, 64, 3), (3, 20, 72, 830, 2), (2, 200, 64, 128, 2),
                                       (4, 64, 830, 830, 10)])
def test_rhn_fused_forward_bitwise(T, B, I, H, L):
    """The persistent fused RHN forward chain (fwd=1: one cooperative launch for all T·L micro-steps,
    split-K chunks as TMEM accumulators, highway epilogue from TMEM) gives the same bits as the
    GEMM + pointwise launch per micro-step (fwd=0) — outputs and every gradient (the backward reads
    the pre-activations and states it saved) — and matches the oracle."""
    p, inp, dY, dhT, dcT = make_cell_case("rhn", T, B, I, H, synth.config_seed(3) + 7, bf16=True, L=L)
    ref = None
    for v in ("fwd=0", "fwd=1"):
        out, g, _ = run_gpu_cell("rhn", p, inp, dY, dhT, dcT, "bf16", v, depth=L)
        cur = {**out, **g}
        if ref is None:
            ref = cur
            continue
        for k in ref:
            assert np.array_equal(ref[k], cur[k]), (v, k)
    _check("rhn", T, B, I, H, "bf16", synth.config_seed(3) + 7, TOL_BF16, variant="fwd=1", L=L)


@pytest.mark.parametrize("T,B,I,H,L", [(3, 64, 64, 830, 10), (2, 16, 32, 64, 2), (4, 37, 48, 200, 3), (1, 64, 64, 256, 2)])
def test_rhn_persistent_bptt_bitwise(T, B, I, H, L):
    """The persistent RHN BPTT chain (bwd=1: one cooperative launch of 4-CTA clusters = the R33
    chunks, partials exchanged over distributed shared memory, the micro-step backward fused, db in
    the row-lane order) gives the same bits as the per-micro-step pointwise + split-K GEMM launches
    (bwd=0) — every gradient, dx, ds0 — with and without the fused forward, and matches the oracle;
    the launch count drops, i.e. the persistent kernel really ran."""
    import paper_conf_asplos_sivathanucsz19_b200 as A
    p, inp, dY, dhT, dcT = make_cell_case("rhn", T, B, I, H, synth.config_seed(3) + 9, bf16=True, L=L)
    ref, launches = None, {}
    for v in ("bwd=0", "bwd=1", "bwd=1,fwd=1"):
        n0 = A.launch_count()
        out, g, _ = run_gpu_cell("rhn", p, inp, dY, dhT, dcT, "bf16", v, depth=L)
        launches[v] = A.launch_count() - n0
        cur = {**out, **g}
        if ref is None:
            ref = cur
            continue
        for k in ref:
            assert np.array_equal(ref[k], cur[k]), (v, k)
    Hp = -(-H // 64) * 64
    nk, s = -(-2 * Hp // 64), min(4, 64 // max(1, -(-B // 128) * -(-Hp // 64)))
    while s > 1 and nk // s < 4:
        s -= 1
    if T * L > 1 and s == 4 and B <= 64:   # the persistent chain's shapes (R33 split of 4)
        assert launches["bwd=1"] < launches["bwd=0"] - T * L, launches
    _check("rhn", T, B, I, H, "bf16", synth.config_seed(3) + 9, TOL_BF16, variant="bwd=1", L=L)


def test_rhn_cfg3_reduced():
    """cfg3 reduced rung: L = 10, H = I = 830, B = 64, T = 8 (bf16)."""
    _check("rhn", 8, 64, 830, 830, "bf16", synth.config_seed(3), TOL_BF16, L=10)


# ------------------------------------------------------------------ LSTM + attention [35]
def _attn_case(Ts, Tt, B, I, H, A, seed, bf16):
    from helpers import bf16_round
    shapes = C.attn_param_shapes(I, H, A)
    p = synth.weights(seed, shapes, H)
    inp = {"xe": synth.uniform(seed, "xe", (Ts, B, I), -1, 1), "xd": synth.uniform(seed, "xd", (Tt, B, I), -1, 1),
           "h0": synth.uniform(seed, "h0", (B, H), -0.5, 0.5), "c0": synth.uniform(seed, "c0", (B, H), -0.5, 0.5)}
    dY = synth.normal(seed, "dY", (Tt, B, 2 * H))
    if bf16:
        for k in ("W_e", "U_e", "W_k", "W_d", "U_d", "C_d", "W_q"):
            p[k] = bf16_round(p[k])
        inp["xe"], inp["xd"], dY = bf16_round(inp["xe"]), bf16_round(inp["xd"]), bf16_round(dY)
    return p, inp, dY, synth.normal(seed, "dhT", (B, H)), synth.normal(seed, "dcT", (B, H))


def _attn_check(Ts, Tt, B, I, H, A, dtype, seed, tol, variant=None):
    import paper_conf_asplos_sivathanucsz19_b200 as AS
    p, inp, dY, dhT, dcT = _attn_case(Ts, Tt, B, I, H, A, seed, dtype == "bf16")
    out_o, g_o = C.cell_fwd_bwd("attn", p, inp, dY, dhT, dcT)
    c = AS.Cell("attn", H, I, B, Tt, dtype=dtype, src_seq=Ts, attn_dim=A)
    if variant is not None:
        c.tune_mode(AS.TUNE_FROZEN, variant)
    c.load(p)
    dev = c.device
    tdt = torch.bfloat16 if dtype == "bf16" else torch.float32
    f32 = lambda a: torch.as_tensor(np.asarray(a, dtype=np.float32), device=dev)
    x = torch.cat([f32(inp["xe"]).reshape(-1), f32(inp["xd"]).reshape(-1)]).to(tdt).contiguous()
    y = torch.empty(Tt, B, 2 * H, dtype=tdt, device=dev)
    hT, cT = torch.empty(B, H, device=dev), torch.empty(B, H, device=dev)
    c.forward(x, f32(inp["h0"]), f32(inp["c0"]), y, hT, cT)
    dx = torch.empty((Ts + Tt) * B * I, dtype=tdt, device=dev)
    dh0, dc0 = torch.empty(B, H, device=dev), torch.empty(B, H, device=dev)
    c.backward(f32(dY).to(tdt).contiguous(), f32(dhT), f32(dcT), dx, dh0, dc0)
    torch.cuda.synchronize()
    dxn = dx.float().cpu().numpy()
    got = {"y": y.float().cpu().numpy(), "hT": hT.cpu().numpy(), "cT": cT.cpu().numpy(),
           "dxe": dxn[:Ts * B * I].reshape(Ts, B, I), "dxd": dxn[Ts * B * I:].reshape(Tt, B, I),
           "dh0": dh0.cpu().numpy(), "dc0": dc0.cpu().numpy()}
    for k in p:
        got[k] = c.view(k, c.grads).cpu().numpy().reshape(np.shape(p[k]))
    ref = dict(out_o)
    ref.update(g_o)
    errs = {k: rel_err(got[k], ref[k]) for k in ref}
    bad = {k: v for k, v in errs.items() if not v <= tol}
    assert not bad, (dtype, bad, errs)
    return got


@pytest.mark.parametrize("Ts,Tt,B,H", [(6, 4, 128, 256), (5, 3, 37, 128), (3, 5, 160, 192)])
def test_attn_encoder_persistent_bitwise(Ts, Tt, B, H):
    """The attention cell's fuse_fwd AV: bit 0 runs its encoder chain as the small-batch persistent
    forward (encoder fwd_mode 3), bit 1 runs each decoder step's K-concatenated recurrent GEMM with
    the gate epilogue fused (lstm_rec_fwd_kernel, K = 2Hp).  Every output and gradient of modes 1-3
    bitwise equal to the launched chains (fwd=0), all against the oracle.  B = 160: two row tiles,
    a ragged one, and no persistent encoder (bit 0 is then a no-op)."""
    import paper_conf_asplos_sivathanucsz19_b200 as AS
    n0 = AS.launch_count()
    ga = _attn_check(Ts, Tt, B, 64, H, H, "bf16", synth.config_seed(4) + 7, TOL_BF16, variant="fwd=0")
    launches = {0: AS.launch_count() - n0}
    for mode in (1, 2, 3):
        n0 = AS.launch_count()
        gb = _attn_check(Ts, Tt, B, 64, H, H, "bf16", synth.config_seed(4) + 7, TOL_BF16, variant=f"fwd={mode}")
        launches[mode] = AS.launch_count() - n0
        for k in ga:
            assert np.array_equal(ga[k], gb[k]), (mode, k)
    # the fused decoder really ran: one launch per decoder step instead of GEMM + pointwise
    # (B ≤ 128: the small-batch kernel run one step per launch; B = 160: lstm_rec_fwd_kernel)
    assert launches[2] <= launches[0] - Tt, launches


@pytest.mark.parametrize("dtype,tol", [("fp32", TOL_FP32), ("bf16", TOL_BF16)])
def test_attn_small(dtype, tol):
    _attn_check(5, 4, 4, 32, 64, 48, dtype, synth.config_seed(4) + 1, tol)


@pytest.mark.parametrize("dtype,tol", [("fp32", TOL_FP32), ("bf16", TOL_BF16)])
def test_attn_ragged(dtype, tol):
    _attn_check(7, 3, 20, 40, 100, 72, dtype, synth.config_seed(4) + 2, tol)


@pytest.mark.parametrize("H,A", [(512, 256), (1024, 512)])
def test_attn_split_bptt_vs_oracle(H, A):
    """Reading R42: the decoder's per-step BPTT GEMMs split into 2 (4Hp = 2048) and 4 (4Hp = 4096)
    K chunks — partials summed in chunk order by the attention backward and the pointwise kernel,
    dq·W_qᵀ accumulated chunk by chunk — match the oracle, with a ragged batch."""
    _attn_check(5, 4, 72, 64, H, A, "bf16", synth.config_seed(4) + 9, TOL_BF16)


def test_attn_cfg4_reduced():
    """cfg4 reduced rung: H = A = I = 1024, B = 128, Ts = Tt = 8 (bf16)."""
    _attn_check(8, 8, 128, 1024, 1024, 1024, "bf16", synth.config_seed(4), TOL_BF16)
