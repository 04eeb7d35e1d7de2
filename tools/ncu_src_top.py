"""Top stall lines / opcode mix of an `ncu --page source --csv --print-source sass` export."""
import collections
import csv
import sys


def main(path, ntop=30):
    lines = open(path).read().split("\n")
    blocks, cur = [], None
    for l in lines:
        if l.startswith('"Kernel Name"'):
            cur = [l]
            blocks.append(cur)
            continue
        if cur is not None:
            cur.append(l)
    for b in blocks[:1]:
        print(b[0][:150])
        rows = list(csv.reader(b[1:]))
        hdr = rows[0]
        ix = {h: i for i, h in enumerate(hdr)}
        data = [r for r in rows[1:] if len(r) > 5]
        tot = sum(int(r[ix["Instructions Executed"]] or 0) for r in data)
        samp = sum(int(r[ix["Warp Stall Sampling (All Samples)"]] or 0) for r in data)
        print("total warp instr", tot, "samples", samp)
        op, st = collections.Counter(), collections.Counter()
        for r in data:
            s = r[ix["Source"]].strip().split()
            o = s[0] if not s[0].startswith("@") else s[1]
            op[o.split(".")[0]] += int(r[ix["Instructions Executed"]] or 0)
            st[o.split(".")[0]] += int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
        for k, v in op.most_common(15):
            print("  ", k, v, "%.1f%%" % (100 * v / max(tot, 1)), "stall%%=%.1f" % (100 * st[k] / max(samp, 1)))
        for i, r in enumerate(sorted(range(len(data)), key=lambda i: -int(data[i][ix["Warp Stall Sampling (All Samples)"]] or 0))[:ntop]):
            d = data[r]
            # show the line index so neighbours can be inspected
            print("   #%d" % r, d[ix["Warp Stall Sampling (All Samples)"]], d[ix["Instructions Executed"]], d[ix["Source"]].strip()[:90])


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 30)
