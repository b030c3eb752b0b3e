"""Summarise a parity-metric log (ASTRA_PARITY_LOG written by tests/helpers.rel_err during
`pytest -m gpu`): per precision path and metric, the number of compared tensors and the worst
values as a multiple of the tensor tolerance (reading R18 / R18b in DESIGN.md)."""
import collections
import json
import sys

rows = [json.loads(l) for l in open(sys.argv[1])]
agg = collections.defaultdict(list)
for d in rows:
    tol = 1e-4 if "fp32" in d["test"] else 2e-2
    fam = "fp32 path (tol 1e-4)" if tol == 1e-4 else "bf16 path (tol 2e-2)"
    for k in ("l2", "max", "row", "col"):
        if k in d:
            agg[(fam, k)].append((d[k] / tol, d["test"].split("::")[-1], tuple(d["shape"])))
print(f"{len(rows)} compared tensors; values are metric / tol (row, col already divided by SLICE_FACTOR)")
for (fam, k), v in sorted(agg.items()):
    v.sort(reverse=True)
    print(f"{fam:22s} {k:4s} n={len(v):4d} worst: " + "; ".join(f"{a:.2f} {b[:48]} {list(c)}" for a, b, c in v[:3]))
