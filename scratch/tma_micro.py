"""TMA read throughput per SM (astra_micro_tma_read) vs box rows, CTAs, ring depth, sharing."""
import sys, json, ctypes, torch
sys.path.insert(0, "/root/repo")
import paper_conf_asplos_sivathanucsz19_b200 as A
L = A.lib()
rows, kb = 8192, 32          # 8192 x 2048 bf16 = 32 MB (L2-resident)
buf = torch.randn(rows, kb * 64, device="cuda").to(torch.bfloat16)
st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
def run(box, ctas, stages, same, nbox=2048):
    A._check(L.astra_micro_tma_read(A._ptr(buf), rows, kb, box, ctas, stages, nbox, same, st))
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(3):
        A._check(L.astra_micro_tma_read(A._ptr(buf), rows, kb, box, ctas, stages, nbox, same, st))
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 3
    per_sm = nbox * box * 128 / (ms * 1e-3) / 1e9
    return {"box_rows": box, "ctas": ctas, "stages": stages, "same": same, "us": round(ms * 1e3, 1),
            "GBps_per_cta": round(per_sm, 1), "GBps_total": round(per_sm * ctas, 1), "ns_per_box": round(ms * 1e6 / nbox, 1)}
for box in (16, 64, 128, 256):
    for ctas in (1, 128, 148):
        for stages in (2, 8):
            if box * 128 * stages > 200000: continue
            for same in (0, 1):
                print(json.dumps(run(box, ctas, stages, same)), flush=True)
