"""Summarise an ncu `--metrics gpu__time_duration.sum --csv` launch list per kernel."""
import collections
import csv
import sys


def summarise(path):
    lines = [l for l in open(path) if l.startswith('"')]
    rows = list(csv.reader(lines))
    hdr = rows[0]
    ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
    gi = hdr.index("Grid Size")
    agg = collections.defaultdict(lambda: [0, 0.0, ""])
    tot = 0.0
    for r in rows[1:]:
        try:
            v = float(r[vi].replace(",", ""))
        except ValueError:
            continue
        name = (r[ki].split("(")[0].replace("void ", "").replace("astra::", "")[:52] + " g" + r[gi].replace(" ", ""))[:70]
        agg[name][0] += 1
        agg[name][1] += v
        agg[name][2] = r[gi]
        tot += v
    out = []
    for k, (n, v, g) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        out.append(f"{k:70s} n={n:4d} total={v / 1e6:8.3f} ms avg={v / n / 1e3:9.2f} us "
                   f"share={v / tot * 100:5.1f}% grid={g}")
    out.append(f"total kernel time {tot / 1e6:.3f} ms over {sum(a[0] for a in agg.values())} launches")
    return "\n".join(out)


if __name__ == "__main__":
    print(summarise(sys.argv[1]))
