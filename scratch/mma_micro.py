"""tcgen05.mma chain: per-MMA time vs M, N (astra_micro_mma_chain) and the M = 64 TMEM layout."""
import sys, json, ctypes, torch
import numpy as np
sys.path.insert(0, "/root/repo")
import paper_conf_asplos_sivathanucsz19_b200 as A
L = A.lib()
st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
cyc = torch.zeros(148, dtype=torch.int64, device="cuda")
for M in (64, 128):
    N = 64
    dump = torch.zeros(128, N, device="cuda")
    A._check(L.astra_micro_mma_chain(M, N, 1, 1, 0, A._ptr(cyc), A._ptr(dump), st))
    torch.cuda.synchronize()
    a = np.array([[((3 * m + k) % 7 - 3) * 0.25 for k in range(16)] for m in range(128)])
    b = np.array([[((5 * n + 2 * k) % 5 - 2) * 0.5 for k in range(16)] for n in range(N)])
    D = a[:M] @ b.T
    d = dump.cpu().numpy()
    # where does row m of D land?
    where = {}
    for m in range(M):
        hits = [l for l in range(128) if np.array_equal(d[l], D[m])]
        where[m] = hits
    print(json.dumps({"M": M, "layout_row_to_lanes": {m: where[m] for m in range(0, M, 4)},
                      "unmatched_lanes_nonzero": [l for l in range(128) if np.abs(d[l]).sum() > 0 and not any(l in where[m] for m in where)][:40]}), flush=True)
for ctas in (1, 148):
    for M in (64, 128):
        for N in (32, 64, 128, 256):
            for iters in (64, 512):
                A._check(L.astra_micro_mma_chain(M, N, iters, ctas, 0, A._ptr(cyc), None, st))
                torch.cuda.synchronize()
                A._check(L.astra_micro_mma_chain(M, N, iters, ctas, 0, A._ptr(cyc), None, st))
                torch.cuda.synchronize()
                c = cyc[:ctas].cpu().numpy()
                print(json.dumps({"ctas": ctas, "M": M, "N": N, "iters": iters, "cyc_per_mma_med": round(float(np.median(c)) / iters, 1),
                                  "cyc_per_mma_max": round(float(c.max()) / iters, 1)}), flush=True)

for mode in (0, 7, 8, 15):
    for N in (64, 256):
        iters = 512
        for _ in range(2):
            A._check(L.astra_micro_mma_chain(128, N, iters, 1, mode, A._ptr(cyc), None, st))
            torch.cuda.synchronize()
        c = cyc[:1].cpu().numpy()
        print(json.dumps({"mode": mode, "M": 128, "N": N, "iters": iters, "cyc_per_mma": round(float(c[0]) / iters, 1)}), flush=True)
