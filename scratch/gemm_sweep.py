"""Event-timed sweep of the K1 GEMM over tile / cluster / pair choices for given shapes."""
import sys, json, torch
sys.path.insert(0, "/root/repo")
import paper_conf_asplos_sivathanucsz19_b200 as A

def run(M, N, K, a_mn, b_mn, cfgs, tag):
    a = (torch.randn(K, M) if a_mn else torch.randn(M, K)).cuda().to(torch.bfloat16)
    b = (torch.randn(K, N) if b_mn else torch.randn(N, K)).cuda().to(torch.bfloat16)
    out = torch.zeros(16, M, N, device="cuda")
    for bn, cm, cn, cg, ks in cfgs:
        try:
            f = lambda: A.gemm_bf16_ex(a, b, M, N, K, a_mn=a_mn, b_mn=b_mn, bn=bn, cm=cm, cn=cn, cta_group=cg, ksplit=ks, out=out)
            for _ in range(3): f()
            torch.cuda.synchronize()
            # 20 launches captured in a CUDA graph: device time without the host's per-call map setup
            g = torch.cuda.CUDAGraph()
            s = torch.cuda.Stream()
            with torch.cuda.stream(s):
                with torch.cuda.graph(g, stream=s):
                    for _ in range(20): f()
            g.replay(); torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            g.replay()
            e1.record(); torch.cuda.synchronize()
            us = e0.elapsed_time(e1) / 20 * 1e3
            print(json.dumps({"tag": tag, "M": M, "N": N, "K": K, "a_mn": a_mn, "b_mn": b_mn, "bn": bn, "cm": cm, "cn": cn,
                              "cg": cg, "ks": ks, "us": round(us, 2), "tflops": round(2 * M * N * K / us / 1e6, 1)}), flush=True)
        except Exception as ex:
            print(json.dumps({"tag": tag, "bn": bn, "cm": cm, "cn": cn, "cg": cg, "ks": ks, "err": str(ex)[:100]}), flush=True)

cf = [(64, 1, 1, 1, 1), (128, 1, 1, 1, 1), (256, 1, 1, 1, 1), (128, 1, 1, 2, 1), (256, 1, 1, 2, 1), (64, 2, 1, 1, 1),
      (64, 1, 2, 1, 1), (128, 2, 1, 1, 1), (128, 1, 2, 1, 1), (64, 1, 1, 1, 2), (128, 1, 1, 1, 2), (128, 1, 1, 1, 4)]
run(1024, 1024, 2240, 1, 1, cf, "cfg2 wgrad (both MN-major)")
run(1024, 1024, 2240, 0, 0, cf, "same shape K-major")
run(1120, 2048, 10000, 0, 1, cf, "cfg2 head dgrad")
run(1024, 4096, 4096, 1, 1, cf, "cfg5 wgrad H=1024 4 gates K=T*B/... ")
