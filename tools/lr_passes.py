"""Per-pass LR times from a VISTA_PROF_LOG file: the launch sequence of the largest-ld layer (stats, power,
ISTA, eval) and per-size totals.  usage: python tools/lr_passes.py prof.tsv"""
import collections
import sys

rows = [l.rstrip("\n").split("\t") for l in open(sys.argv[1])]
lr = [(float(r[1]), float(r[3])) for r in rows if r[0] == "5"]
by = collections.defaultdict(list)
for ms, b in lr:
    by[b].append(ms)
tot = 0.0
for b, v in sorted(by.items()):
    tot += sum(v)
    print(f"{b / 1e6:8.1f} MB  n={len(v):3d}  total {sum(v):6.2f} ms  mean {1e3 * sum(v) / len(v):6.1f} us  "
          f"min {1e3 * min(v):6.1f} us ({b / (min(v) * 1e-3) / 1e12:.2f} TB/s)")
big = max(by)
print("largest-layer sequence (us):", [round(ms * 1e3, 1) for ms, b in lr if b == big][:33])
print(f"lr total {tot:.2f} ms")
