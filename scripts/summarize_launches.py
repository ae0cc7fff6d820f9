"""Summarise an ncu launch list (--metrics gpu__time_duration.sum) into a markdown
table: per kernel the launch count, mean duration and share of the listed time.
The list is cold-cache and serialised, so only the SHARES are meaningful."""
import csv
import sys
from collections import defaultdict

SCALE = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "second": 1e6, "s": 1e6}


def main(path, title):
    rows = [r for r in csv.reader(open(path)) if len(r) > 5]
    h = rows[0]
    ki, vi, ui, mi = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit"), h.index("Metric Name")
    agg = defaultdict(list)
    for r in rows[1:]:
        if r[mi] == "gpu__time_duration.sum":
            agg[r[ki].split("(")[0]].append(float(r[vi].replace(",", "")) * SCALE.get(r[ui], 1.0))
    tot = sum(sum(v) for v in agg.values()) or 1.0
    out = [f"# launch list: {title}", "", f"source: `{path.split('/')[-1]}` (ncu --metrics gpu__time_duration.sum --clock-control none)", "",
           "| kernel | launches | mean us | share |", "|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda x: -sum(x[1])):
        out.append(f"| `{k}` | {len(v)} | {sum(v) / len(v):.1f} | {100 * sum(v) / tot:.1f}% |")
    print("\n".join(out))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
