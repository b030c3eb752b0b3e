"""K1 (tcgen05/TMA/TMEM GEMM) on B200 against an fp64 product of the same bf16 operands, for every
operand layout the step uses, ragged tails, and the bitwise tile-shape invariance (R1, R7)."""
import numpy as np
import pytest
import torch

import paper_conf_asplos_sivathanucsz19_b200 as A

pytestmark = pytest.mark.gpu


def _operands(M, N, K, a_mn, b_mn, seed=0):
    g = torch.Generator().manual_seed(seed)
    a = torch.randn(M, K, generator=g).to(torch.bfloat16)
    b = torch.randn(K, N, generator=g).to(torch.bfloat16)
    ref = a.double() @ b.double()
    A_store = (a.t() if a_mn else a).contiguous().cuda()      # MN-major A is stored [K][M]
    B_store = (b if b_mn else b.t()).contiguous().cuda()      # K-major B is stored [N][K]
    return A_store, B_store, ref


@pytest.mark.parametrize("a_mn,b_mn", [(0, 0), (0, 1), (1, 0), (1, 1)])
@pytest.mark.parametrize("M,N,K", [(128, 256, 64), (256, 512, 1024), (300, 200, 136), (64, 64, 32)])
def test_gemm_layouts(a_mn, b_mn, M, N, K):
    if (a_mn and M % 8) or (b_mn and N % 8) or (not a_mn and K % 8) or (not b_mn and K % 8):
        pytest.skip("TMA needs 16-byte row strides")
    A_s, B_s, ref = _operands(M, N, K, a_mn, b_mn)
    for bn in (64, 128, 256):
        out = A.gemm_bf16(A_s, B_s, M, N, K, a_mn=a_mn, b_mn=b_mn, bn=bn)
        torch.cuda.synchronize()
        err = (out.double().cpu() - ref).abs().max().item()
        scale = ref.abs().max().item()
        assert err <= 1e-5 * scale * max(1, K / 64) + 1e-6, (bn, err, scale)


CLUSTERS = [(1, 1), (2, 1), (4, 1), (1, 2), (2, 2), (1, 4), (4, 2), (2, 4)]


def test_tile_shapes_bitwise():
    """R1/R7: the accumulation order of every output element depends on neither the tile width nor
    the cluster/multicast shape."""
    M, N, K = 512, 768, 2048
    for a_mn, b_mn in [(0, 0), (1, 1), (0, 1), (1, 0)]:
        A_s, B_s, _ = _operands(M, N, K, a_mn, b_mn, seed=3)
        outs = [A.gemm_bf16(A_s, B_s, M, N, K, a_mn=a_mn, b_mn=b_mn, bn=bn, cm=cm, cn=cn)
                for bn in (64, 128, 256) for cm, cn in CLUSTERS]
        torch.cuda.synchronize()
        for o in outs[1:]:
            assert torch.equal(outs[0], o)


@pytest.mark.parametrize("cm,cn", CLUSTERS)
@pytest.mark.parametrize("a_mn,b_mn", [(0, 0), (1, 1), (0, 1), (1, 0)])
def test_cluster_multicast_ragged(cm, cn, a_mn, b_mn):
    """Cluster multicast with tile counts that are not multiples of the cluster shape."""
    M, N, K = 392, 200, 264
    if a_mn and M % 8:
        pytest.skip()
    A_s, B_s, ref = _operands(M, N, K, a_mn, b_mn, seed=11)
    for bn in (64, 128, 256):
        out = A.gemm_bf16(A_s, B_s, M, N, K, a_mn=a_mn, b_mn=b_mn, bn=bn, cm=cm, cn=cn)
        torch.cuda.synchronize()
        err = (out.double().cpu() - ref).abs().max().item()
        assert err <= 2e-6 * K ** 0.5 * ref.abs().max().item(), (bn, cm, cn, err)


def test_paper_table1_shapes():
    """The paper's Table 1 GEMMs: 64x1024x4096 (LSTM fwd fused) and 64x4096x1024 (bwd)."""
    for M, K, N in [(64, 1024, 4096), (64, 4096, 1024)]:
        A_s, B_s, ref = _operands(M, N, K, 0, 0, seed=5)
        out = A.gemm_bf16(A_s, B_s, M, N, K)
        torch.cuda.synchronize()
        # fp32 accumulation of exact bf16 products: error ~ sqrt(K)·2^-24·|terms|
        assert (out.double().cpu() - ref).abs().max().item() <= 2e-6 * K ** 0.5 * ref.abs().max().item()


@pytest.mark.parametrize("ksplit", [2, 3, 4])
@pytest.mark.parametrize("a_mn,b_mn", [(0, 1), (0, 0)])
def test_split_k_partials(ksplit, a_mn, b_mn):
    """Fixed split-K (the BPTT GEMM's numerics, R25): partial s equals the fp64 product over its own
    K chunk (chunk = ceil(ceil(K/64)/ksplit)·64 elements, ragged last chunk), every tile width gives
    the same bits, and the partials summed in chunk order match the full product."""
    M, N, K = 200, 320, 64 * 9 + 40
    A_s, B_s, _ = _operands(M, N, K, a_mn, b_mn, seed=ksplit)
    g = torch.Generator().manual_seed(ksplit)
    a = torch.randn(M, K, generator=g).to(torch.bfloat16).double()
    b = torch.randn(K, N, generator=g).to(torch.bfloat16).double()
    kper = -(-(-(-K // 64)) // ksplit) * 64
    outs = []
    for bn in (64, 128, 256):
        out = A.gemm_bf16_ex(A_s, B_s, M, N, K, a_mn=a_mn, b_mn=b_mn, bn=bn, ksplit=ksplit)
        torch.cuda.synchronize()
        outs.append(out.cpu())
    for o in outs[1:]:
        assert torch.equal(o, outs[0])
    o = outs[0].double()
    for s in range(ksplit):
        k0, k1 = s * kper, min(K, (s + 1) * kper)
        ref = a[:, k0:k1] @ b[k0:k1] if k1 > k0 else torch.zeros(M, N, dtype=torch.float64)
        err = (o[s] - ref).abs().max().item()
        assert err <= 1e-5 * max(1.0, ref.abs().max().item()) * max(1, (k1 - k0) / 64) + 1e-6, (s, err)
    full = a @ b
    tot = o[0].clone()
    for s in range(1, ksplit):
        tot = tot + o[s]
    assert (tot - full).abs().max().item() <= 1e-5 * full.abs().max().item() * K / 64


@pytest.mark.parametrize("a_mn,b_mn", [(0, 0), (0, 1), (1, 0), (1, 1)])
@pytest.mark.parametrize("M,N,K", [(512, 1024, 512), (300, 200, 136), (128, 256, 64), (700, 640, 1000)])
def test_cta_pair_bitwise(a_mn, b_mn, M, N, K):
    """cta_group::2 (CTA pair, 256 x bn tiles) gives the same bits as the single-CTA kernel, with
    ragged M (half-empty pairs), ragged N and K, every operand layout, and with split-K."""
    if (a_mn and M % 8) or (b_mn and N % 8) or K % 8:
        pytest.skip("TMA needs 16-byte row strides")
    A_s, B_s, ref = _operands(M, N, K, a_mn, b_mn, seed=7)
    base = A.gemm_bf16(A_s, B_s, M, N, K, a_mn=a_mn, b_mn=b_mn, bn=128)
    torch.cuda.synchronize()
    err = (base.double().cpu() - ref).abs().max().item()
    assert err <= 1e-5 * ref.abs().max().item() * max(1, K / 64) + 1e-6
    for bn in (128, 224, 256):   # 224: 112 B rows per CTA (K-major B; MN-major B runs it as 256)
        out = A.gemm_bf16_ex(A_s, B_s, M, N, K, a_mn=a_mn, b_mn=b_mn, bn=bn, cta_group=2)
        torch.cuda.synchronize()
        assert torch.equal(out[0].cpu(), base.cpu()), bn
    s1 = A.gemm_bf16_ex(A_s, B_s, M, N, K, a_mn=a_mn, b_mn=b_mn, bn=256, ksplit=3)
    s2 = A.gemm_bf16_ex(A_s, B_s, M, N, K, a_mn=a_mn, b_mn=b_mn, bn=128, cta_group=2, ksplit=3)
    torch.cuda.synchronize()
    assert torch.equal(s1.cpu(), s2.cpu())


def test_day1_microbenchmarks_run():
    """The astra_micro_* kernels (bench_micro.py) run and do what they claim: the
    grid barrier counter ends at iters × #SMs, the streaming read and the launch chain complete."""
    import ctypes
    import torch
    import paper_conf_asplos_sivathanucsz19_b200 as A
    L = A.lib()
    sp = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    buf = torch.rand(4 << 20, device="cuda")
    sink = torch.zeros(1, device="cuda")
    A._check(L.astra_micro_stream_read(A._ptr(buf), buf.numel() * 4, 3, A._ptr(sink), sp))
    ctr = torch.zeros(4, dtype=torch.int32, device="cuda")
    A._check(L.astra_micro_grid_barrier(A._ptr(ctr), 100, sp))
    A._check(L.astra_micro_launch_chain(50, 1, 148, sp))
    A._check(L.astra_micro_launch_chain(50, 0, 148, sp))
    torch.cuda.synchronize()
    assert int(ctr[0].item()) == 100 * torch.cuda.get_device_properties(0).multi_processor_count
    assert float(sink.item()) == 0.0
    assert L.astra_micro_grid_barrier(None, 10, sp) == 1
