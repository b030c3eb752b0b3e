import sys, torch
sys.path.insert(0, "/root/repo")
import paper_conf_asplos_sivathanucsz19_b200 as A
M, N, K, bn, cg = (int(x) for x in sys.argv[1:6])
cm = int(sys.argv[6]) if len(sys.argv) > 6 else 1
cn = int(sys.argv[7]) if len(sys.argv) > 7 else 1
ks = int(sys.argv[8]) if len(sys.argv) > 8 else 1
a = torch.randn(M, K, device="cuda").to(torch.bfloat16)
b = torch.randn(N, K, device="cuda").to(torch.bfloat16)
out = torch.zeros(ks, M, N, device="cuda")
for _ in range(3):
    A.gemm_bf16_ex(a, b, M, N, K, bn=bn, cm=cm, cn=cn, cta_group=cg, ksplit=ks, out=out)
torch.cuda.synchronize()
