import sys, torch
sys.path.insert(0, "/root/repo")
import paper_conf_asplos_sivathanucsz19_b200 as A
M, N, K, bn, cg = (int(x) for x in sys.argv[1:6])
a = torch.randn(M, K, device="cuda").to(torch.bfloat16)
b = torch.randn(N, K, device="cuda").to(torch.bfloat16)
out = torch.zeros(1, M, N, device="cuda")
for _ in range(3):
    A.gemm_bf16_ex(a, b, M, N, K, bn=bn, cta_group=cg, out=out)
torch.cuda.synchronize()
