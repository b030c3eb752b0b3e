"""Summarise an ncu launch list (`--metrics gpu__time_duration.sum[,dram__bytes_read.sum,...] --csv`)
per kernel (name + grid): launches, total/avg device time, share of the step, DRAM bytes per launch."""
import collections
import csv
import sys


def summarise(path):
    lines = [l for l in open(path) if l.startswith('"')]
    rows = list(csv.reader(lines))
    hdr = rows[0]
    ki, vi, mi, gi, ii = (hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Name"),
                          hdr.index("Grid Size"), hdr.index("ID"))
    per_launch = collections.defaultdict(dict)
    names = {}
    for r in rows[1:]:
        try:
            v = float(r[vi].replace(",", ""))
        except ValueError:
            continue
        per_launch[r[ii]][r[mi]] = v
        names[r[ii]] = (r[ki].split("(")[0].replace("void ", "").replace("astra::", "")[:52] + " g"
                        + r[gi].replace(" ", ""))[:70]
    agg = collections.defaultdict(lambda: [0, 0.0, 0.0])
    tot = 0.0
    for i, m in per_launch.items():
        t = m.get("gpu__time_duration.sum", 0.0)
        b = m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
        a = agg[names[i]]
        a[0] += 1
        a[1] += t
        a[2] += b
        tot += t
    out = []
    for k, (n, t, b) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        extra = f" dram/launch={b / n / 1e6:8.2f} MB ({b / t:6.0f} GB/s)" if b else ""
        out.append(f"{k:70s} n={n:4d} total={t / 1e6:8.3f} ms avg={t / n / 1e3:9.2f} us share={t / tot * 100:5.1f}%"
                   + extra)
    out.append(f"total kernel time {tot / 1e6:.3f} ms over {len(per_launch)} launches")
    return "\n".join(out)


if __name__ == "__main__":
    print(summarise(sys.argv[1]))
