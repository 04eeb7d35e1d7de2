"""Aggregate a VISTA_PROF_LOG file (per-launch CUDA-event records) by launch label."""
import sys
from collections import defaultdict
agg = defaultdict(lambda: [0, 0.0, 0.0, 0.0])
for line in open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/prof.tsv"):
    c, ms, fl, by, lab = line.rstrip("\n").split("\t")
    key = lab if lab else f"cls{c}"
    key = " ".join(w for w in key.split() if not w.startswith("M") and not w.startswith("tiles"))
    a = agg[key]; a[0] += 1; a[1] += float(ms); a[2] += float(fl); a[3] += float(by)
tot = sum(a[1] for a in agg.values())
n = int(sys.argv[2]) if len(sys.argv) > 2 else 16
for k, a in sorted(agg.items(), key=lambda x: -x[1][1])[:n]:
    tf = a[2] / (a[1] / 1e3) / 1e12 if a[2] else 0
    gb = a[3] / (a[1] / 1e3) / 1e9
    print(f"{a[1]:8.2f} ms {100 * a[1] / tot:5.1f}% n={a[0]:4d} {tf:7.1f} TF/s {gb:7.0f} GB/s  {k}")
print("total", round(tot, 2))
