"""Summarise an `ncu --metrics ... --csv` log of tools/layer_probe.py: last launch per probe shape."""
import csv
import sys

NAMES = ["c4_res", "c2_res", "c3_res", "c5_res", "a2_3x3", "a3_3x3", "a4_3x3", "r2_1x1", "r4_1x1"]


def load(path):
    rows = list(csv.reader(open(path)))
    hdr, out = None, {}
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr is None or len(r) < len(hdr):
            continue
        d = dict(zip(hdr, r))
        m = out.setdefault(int(d["ID"]), {"k": d["Kernel Name"]})
        m[d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
    return [out[i] for i in sorted(out)]


def main():
    names = sys.argv[2].split(",") if len(sys.argv) > 2 else NAMES
    L = load(sys.argv[1])
    per = len(L) // len(names)
    for i, nm in enumerate(names):
        m = L[i * per + per - 1]
        t = m["gpu__time_duration.sum"] / 1e6
        b = m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
        print(f"{nm:8s} {t:.4f} ms  dram {b / 1e6:8.1f} MB {b / t / 1e9:6.2f} TB/s  {m['k'][:40]}")


if __name__ == "__main__":
    main()
