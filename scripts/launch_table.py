"""Per-kernel totals of an ncu --metrics gpu__time_duration.sum --csv launch list."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hdr]
ki, vi = h.index("Kernel Name"), h.index("Metric Value")
data = [(r[ki], float(r[vi].replace(",", ""))) for r in rows[hdr + 1:] if len(r) > vi]
agg = collections.defaultdict(list)
for k, v in data:
    agg[k.split("(")[0].split("<")[0].replace("void ", "")].append(v)
tot = sum(v for _, v in data)
for k, vs in sorted(agg.items(), key=lambda x: -sum(x[1]))[:int(sys.argv[2]) if len(sys.argv) > 2 else 12]:
    print(f"{k:28s} n={len(vs):5d} total_ms={sum(vs) / 1e6:9.2f} share={sum(vs) / tot:6.1%} "
          f"avg_us={sum(vs) / len(vs) / 1e3:8.1f}")
