"""Per-kernel summary of an ncu launch list (--metrics gpu__time_duration.sum --csv): count, mean, total, share."""
import collections
import csv
import sys


def summarize(path):
    rows = list(csv.reader(ln for ln in open(path) if not ln.startswith("==")))
    h = rows[0]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}
    agg = collections.defaultdict(list)
    for r in rows[1:]:
        agg[r[ki].replace("(anonymous namespace)::", "").split("(")[0]].append(
            float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0))
    tot = sum(sum(v) for v in agg.values())
    out = ["| kernel | launches | mean µs | total µs | share |", "|---|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        out.append(f"| {k} | {len(v)} | {sum(v) / len(v):.1f} | {sum(v):.1f} | {sum(v) / tot:.1%} |")
    return "\n".join(out)


if __name__ == "__main__":
    print(summarize(sys.argv[1]))
