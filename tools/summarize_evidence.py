"""Summarise tools/ncu_evidence.sh into profiles/<tag>_kernel_evidence.md: per kernel (template instance),
launches, total time, time-weighted tensor-pipe utilisation and DRAM throughput (% of peak and TB/s).
usage: python tools/summarize_evidence.py <evidence.csv> <tag>"""
import csv
import os
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
hdr = rows[0]
ik, imn, iv = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
iid = hdr.index("ID")
per = defaultdict(dict)
for r in rows[1:]:
    try:
        per[(r[iid], r[ik])][r[imn]] = float(r[iv].replace(",", ""))
    except ValueError:
        pass
agg = defaultdict(lambda: [0, 0.0, 0.0, 0.0, 0.0])
for (_, name), m in per.items():
    t = m.get("gpu__time_duration.sum", 0.0)  # ns (or us, normalised below)
    a = agg[name.split("(")[0][:90]]
    a[0] += 1
    a[1] += t
    a[2] += t * m.get("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", 0.0)
    a[3] += t * m.get("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", 0.0)
    a[4] += m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
tot = sum(a[1] for a in agg.values())
unit = "ns" if tot > 1e6 else "us"
scale = 1e-6 if unit == "ns" else 1e-3  # -> ms
lines = ["# Per-kernel ncu evidence, " + sys.argv[2], "",
         "`bash tools/ncu_evidence.sh` on one B200: bench.py (ResNet50 top-5) at 4096 images, one step, every launch "
         "profiled with `--clock-control none` (serialised, cold-cache: compare utilisations, not absolute times). "
         "Tensor-pipe and DRAM columns are time-weighted means over the kernel's launches; TB/s = DRAM bytes / time.",
         "", "| kernel | launches | ms | share | tensor pipe % | DRAM % of peak | DRAM TB/s |", "|---|---|---|---|---|---|---|"]
for k, a in sorted(agg.items(), key=lambda x: -x[1][1]):
    ms = a[1] * scale
    tbs = a[4] / (a[1] * (1e-9 if unit == "ns" else 1e-6)) / 1e12 if a[1] else 0
    lines.append(f"| `{k}` | {a[0]} | {ms:.2f} | {100 * a[1] / tot:.1f} % | {a[2] / a[1]:.1f} | {a[3] / a[1]:.1f} | {tbs:.2f} |")
open(os.path.join(ROOT, "profiles", f"{sys.argv[2]}_kernel_evidence.md"), "w").write("\n".join(lines) + "\n")
print("\n".join(lines[:30]))
