import sys, torch
sys.path.insert(0, "/root/repo")
import paper_conf_asplos_sivathanucsz19_b200 as A
shapes = [(512, 8192, 2048), (512, 2048, 8192), (512, 1024, 1024), (128, 256, 64), (512, 8192, 256)]
for M, N, K in shapes:
    a = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    b = torch.randn(N, K, device="cuda").to(torch.bfloat16)
    for cg, bn in ((1, 256), (2, 256), (1, 128)):
        for _ in range(3):
            A.gemm_bf16_ex(a, b, M, N, K, bn=bn, cta_group=cg)
torch.cuda.synchronize()
