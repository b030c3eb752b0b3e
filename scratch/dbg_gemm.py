import sys, torch
sys.path.insert(0, '.')
import paper_conf_asplos_sivathanucsz19_b200 as A
def run(M, N, K, a_mn, b_mn, lda=None, ldb=None, bn=256):
    g = torch.Generator().manual_seed(0)
    a = torch.randn(M, K, generator=g).to(torch.bfloat16)
    b = torch.randn(K, N, generator=g).to(torch.bfloat16)
    ref = a.double() @ b.double()
    As = (a.t() if a_mn else a).contiguous()
    Bs = (b if b_mn else b.t()).contiguous()
    if lda and lda > As.shape[1]:
        As = torch.nn.functional.pad(As, (0, lda - As.shape[1]))
    if ldb and ldb > Bs.shape[1]:
        Bs = torch.nn.functional.pad(Bs, (0, ldb - Bs.shape[1]))
    out = A.gemm_bf16(As.cuda(), Bs.cuda(), M, N, K, a_mn=a_mn, b_mn=b_mn, bn=bn)
    torch.cuda.synchronize()
    err = (out.double().cpu() - ref).abs().max().item()
    zero_rows = (out.abs().sum(1) == 0).sum().item()
    print(f"M={M} N={N} K={K} a_mn={a_mn} b_mn={b_mn} lda={lda} ldb={ldb} bn={bn} err={err:.3e} zero_rows={zero_rows}")
for K in (16, 32, 48, 64, 80):
    for N in (128, 256):
        run(32, N, K, 1, 1, lda=64, bn=256)
run(64, 128, 16, 1, 1, bn=256)
run(64, 128, 16, 1, 1, bn=128)
run(32, 128, 16, 1, 1, lda=64, bn=128)
run(32, 128, 16, 0, 1, bn=256)
run(128, 128, 16, 1, 1, bn=256)
