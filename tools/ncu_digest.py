"""Digest of `ncu --page raw --csv` exports: duration, DRAM / L2 / tensor-pipe / issue metrics per kernel."""
import csv
import sys

WANT = [
    ("gpu__time_duration.sum", "dur"),
    ("dram__bytes_read.sum", "dram_rd"),
    ("dram__bytes_write.sum", "dram_wr"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "dram%"),
    ("lts__t_bytes.sum", "l2_bytes"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "l2%"),
    ("lts__t_sector_hit_rate.pct", "l2hit%"),
    ("sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active", "hmma%"),
    ("sm__inst_executed_pipe_uma.avg.pct_of_peak_sustained_active", "uma%"),
    ("sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active", "tc%"),
    ("sm__issue_active.avg.pct_of_peak_sustained_active", "issue%"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed", "smem%"),
    ("sm__cycles_elapsed.avg.per_second", "clk"),
]


def digest(path):
    rows = list(csv.reader(open(path)))
    hdr = rows[0]
    units = rows[1]
    out = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        name = d.get("Kernel Name", "?")[:70]
        vals = {}
        for k, short in WANT:
            if k in d:
                vals[short] = d[k] + (units[hdr.index(k)] if units[hdr.index(k)] else "")
        out.append((name, vals))
    return out, hdr


if __name__ == "__main__":
    for p in sys.argv[1:]:
        res, hdr = digest(p)
        for name, vals in res:
            print(p, name)
            print("   ", vals)
        if "--list" in sys.argv:
            print([h for h in hdr if "tensor" in h or "pipe_tc" in h or "lts__t" in h][:60])
