"""Summarise ncu output into profiles/ (run here, on the CPU box).

    python scripts/ncu_summary.py TAG CONFIG launches.csv [full_capture.ncu-rep ...]

Writes profiles/<TAG>_<CONFIG>.md (launch-list shares per kernel + the key
counters of each full capture) and merges per-launch DRAM traffic of the
captured kernels into profiles/traffic.json (read by bench.py's roofline).
"""
import csv
import json
import os
import re
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 throughput %"),
    ("lts__t_sector_hit_rate.pct", "L2 hit rate %"),
    ("l1tex__t_sector_hit_rate.pct", "L1 hit rate %"),
    ("l1tex__throughput.avg.pct_of_peak_sustained_active", "L1 throughput %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active %"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
     "long-scoreboard stall / issue"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor pipe %"),
]

SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
         "ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3, "s": 1}


def short(name):
    m = re.search(r"(k_[A-Za-z0-9_]+)", name)
    return m.group(1) if m else name[:40]


def launches(path):
    text = open(path).read().splitlines()
    start = next(i for i, l in enumerate(text) if l.startswith('"ID"'))
    rows = list(csv.DictReader(text[start:]))
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", "")) * SCALE.get(r.get("Metric Unit", "ns"), 1e-9)
        k = short(r["Kernel Name"])
        agg[k][0] += 1
        agg[k][1] += v
    return agg


def capture(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = {"kernel": short(vals[hdr.index("Kernel Name")])}
        for key, label in KEYS:
            if key in hdr:
                i = hdr.index(key)
                d[label] = (vals[i], units[i])
        res.append(d)
    return res


def to_bytes(v):
    val, unit = v
    return float(val.replace(",", "")) * SCALE.get(unit, 1)


def main():
    tag, cfg, lcsv = sys.argv[1], sys.argv[2], sys.argv[3]
    reps = sys.argv[4:]
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    lines = [f"# ncu summary {tag} / {cfg}", "",
             f"Launch list: `ncu --metrics gpu__time_duration.sum --clock-control none` of "
             f"`scripts/prof_step.py {cfg} 2` (cold-cache, serialised: compare shares, not "
             "absolute times).", "", "| kernel | launches | total ms | share | avg us |",
             "|---|---|---|---|---|"]
    agg = launches(lcsv)
    tot = sum(t for _, t in agg.values())
    for k, (n, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        lines.append(f"| {k} | {n} | {t * 1e3:.2f} | {100 * t / tot:.1f}% | {1e6 * t / n:.1f} |")
    traffic_path = os.path.join(ROOT, "profiles", "traffic.json")
    traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
    l2_path = os.path.join(ROOT, "profiles", "l2.json")
    l2 = json.load(open(l2_path)) if os.path.exists(l2_path) else {}
    for rp in reps:
        for d in capture(rp):
            lines += ["", f"## `ncu --set full` capture: {d['kernel']} ({os.path.basename(rp)})", "",
                      "| counter | value |", "|---|---|"]
            for _, label in KEYS:
                if label in d:
                    lines.append(f"| {label} | {d[label][0]} {d[label][1]} |")
            if "DRAM read" in d and "DRAM write" in d:
                b = to_bytes(d["DRAM read"]) + to_bytes(d["DRAM write"])
                kind = ("frozen" if "wspmv" in d["kernel"] else "reverse" if "reverse" in d["kernel"]
                        else "forward" if "forward" in d["kernel"] else d["kernel"])
                traffic.setdefault(cfg, {})[kind] = b
                lines.append(f"| traffic (read + write) per launch | {b / 1e9:.3f} GB |")
            if "L2 hit rate %" in d:  # bench.py reports it for L2-resident configs
                l2.setdefault(cfg, {})[d["kernel"]] = float(d["L2 hit rate %"][0].replace(",", ""))
    with open(os.path.join(ROOT, "profiles", f"{tag}_{cfg}.md"), "w") as fh:
        fh.write("\n".join(lines) + "\n")
    with open(traffic_path, "w") as fh:
        json.dump(traffic, fh, indent=1)
    with open(l2_path, "w") as fh:
        json.dump(l2, fh, indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
