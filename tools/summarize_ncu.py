"""Summarise the ncu captures of tools/profile_gpu.sh into profiles/ (committed evidence).

usage: python tools/summarize_ncu.py <capture dir> <round tag>
writes profiles/<tag>_launches.csv (trimmed launch list), profiles/<tag>_ncu_summary.md and
profiles/ncu_summary.json (read by bench.py for roofline.traffic).
"""
import csv
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def read_ncu_csv(path):
    rows = list(csv.reader(open(path)))
    hdr, out = None, []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            out.append(dict(zip(hdr, r)))
    return out


def short(name):
    name = name.replace("void ", "").replace("vista::", "")
    return name.split("(")[0]


def main():
    src, tag = sys.argv[1], sys.argv[2]
    prof = os.path.join(ROOT, "profiles")
    os.makedirs(prof, exist_ok=True)
    cmd = sys.argv[3] if len(sys.argv) > 3 else "bash tools/profile_gpu.sh"
    md = [f"# ncu evidence, {tag}", "",
          f"Command: `{cmd}` under gpurun on one B200 (bench.py default workload: ResNet50 top-5, 20k images; "
          "the launch list and the DRAM pass cover every step execution of that bench command, see the launch "
          "count). ncu times are cold-cache and serialised: compare shares, not absolutes.", ""]
    # ---- 1. launch list ----
    L = read_ncu_csv(os.path.join(src, "launches.csv"))
    with open(os.path.join(prof, f"{tag}_launches.csv"), "w", newline="") as f:
        w = csv.writer(f)
        w.writerow(["id", "kernel", "grid", "block", "gpu__time_duration.sum_ns"])
        for d in L:
            w.writerow([d["ID"], short(d["Kernel Name"]), d["Grid Size"], d["Block Size"], d["Metric Value"]])
    agg = defaultdict(lambda: [0, 0.0])
    for d in L:
        k = short(d["Kernel Name"])
        agg[k][0] += 1
        agg[k][1] += float(d["Metric Value"] or 0)
    tot = sum(v[1] for v in agg.values())
    md += ["## 1. Launch list (all kernels of the profiled step executions)", "",
           f"{len(L)} launches, {tot / 1e6:.1f} ms of device time.", "",
           "| kernel | launches | ms | share |", "|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        md.append(f"| `{k}` | {v[0]} | {v[1] / 1e6:.2f} | {100 * v[1] / tot:.1f} % |")
    # ---- 2. dram bytes per conv launch ----
    D = read_ncu_csv(os.path.join(src, "conv_dram.csv"))
    per = defaultdict(dict)
    for d in D:
        per[d["ID"]][d["Metric Name"]] = float(d["Metric Value"] or 0)
        per[d["ID"]]["grid"] = d["Grid Size"]
    n = len(per)
    t_ns = sum(v.get("gpu__time_duration.sum", 0) for v in per.values())
    rd = sum(v.get("dram__bytes_read.sum", 0) for v in per.values())
    wr = sum(v.get("dram__bytes_write.sum", 0) for v in per.values())
    md += ["", "## 2. DRAM traffic of every conv-class launch (conv_tc_kernel, res_chain_kernel, conv1_pool_kernel)", "",
           f"{n} launches, {t_ns / 1e6:.1f} ms, dram read {rd / 1e9:.1f} GB, "
           f"write {wr / 1e9:.1f} GB -> {(rd + wr) / n / 1e6:.2f} MB per launch on average, "
           f"{(rd + wr) / (t_ns * 1e-9) / 1e12:.2f} TB/s while running.", ""]
    summary = {"tag": tag, "dominant": {
        "kernel": "conv_tc_kernel", "launches": n, "dram_bytes_per_launch": (rd + wr) / n if n else None,
        "dram_read_bytes": rd, "dram_write_bytes": wr, "ncu_ms": t_ns / 1e6,
        "note": "dram__bytes_read.sum + dram__bytes_write.sum per launch, averaged over every conv-class launch "
                "(conv_tc, res_chain, conv1_pool) of the profiled bench step executions (ncu, --clock-control none)"}}
    # ---- 3. the --set full capture ----
    rep = os.path.join(src, "conv_full.ncu-rep")
    raw_csv = os.path.join(src, "conv_full.raw.csv")
    raw = None
    if os.path.exists(rep):
        raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    elif os.path.exists(raw_csv):  # the capture scripts export the raw page and delete the report
        raw = open(raw_csv).read()
    if raw:
        rows = list(csv.reader(raw.splitlines()))
        if len(rows) >= 3:
            hdr, units, vals = rows[0], rows[1], rows[2]
            want = ["Kernel Name", "Grid Size", "Block Size", "gpu__time_duration.sum", "dram__bytes_read.sum",
                    "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
                    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
                    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
                    "lts__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
                    "launch__shared_mem_per_block_dynamic", "sm__warps_active.avg.pct_of_peak_sustained_active"]
            md += ["", "## 3. `ncu --set full` on one launch of the top conv kernel (res4 3x3, CTA-pair im2col; 1024-image micro-batch)", "",
                   "| metric | value |", "|---|---|"]
            full = {}
            for w_ in want:
                if w_ in hdr:
                    i = hdr.index(w_)
                    md.append(f"| {w_} | {vals[i]} {units[i]} |")
                    full[w_] = vals[i]
            summary["full_capture"] = full
    open(os.path.join(prof, f"{tag}_ncu_summary.md"), "w").write("\n".join(md) + "\n")
    json.dump(summary, open(os.path.join(prof, "ncu_summary.json"), "w"), indent=1)
    print("\n".join(md))


if __name__ == "__main__":
    main()
