#!/usr/bin/env python
"""Group the per-instruction counts of an `ncu --page source --csv --print-source sass` export by
execution count (instructions that run equally often belong to the same loop level), for one kernel.

  python tools/sass_hist.py <sass.csv> [kernel_index] [units]     (units: candidates, for per-unit rates)
"""
import collections
import csv
import sys


def kernels(path):
    out, cur = [], None
    for row in csv.reader(open(path)):
        if row and row[0] == "Kernel Name":
            cur = {"name": row[1], "rows": []}
            out.append(cur)
        elif cur is not None and row and row[0] == "Address":
            cur["hdr"] = row
        elif cur is not None and row and row[0].startswith("0x"):
            cur["rows"].append(row)
    return out


def main():
    ks = kernels(sys.argv[1])
    k = ks[int(sys.argv[2]) if len(sys.argv) > 2 else 0]
    units = float(sys.argv[3]) if len(sys.argv) > 3 else 1.0
    h = k["hdr"]
    ie, ti, sm, src = (h.index(c) for c in ("Instructions Executed", "Thread Instructions Executed",
                                           "Warp Stall Sampling (All Samples)", "Source"))
    groups = collections.defaultdict(lambda: [0, 0, 0, 0])
    tot_w = tot_t = tot_s = 0
    for r in k["rows"]:
        w, t, s = int(r[ie]), int(r[ti]), int(r[sm])
        tot_w += w; tot_t += t; tot_s += s
        g = groups[w]
        g[0] += 1; g[1] += t; g[2] += s
    print(k["name"][:100])
    print("warp instr %d, thread instr %d (%.3f per unit), stall samples %d" % (tot_w, tot_t, tot_t / units, tot_s))
    print("%12s %6s %10s %8s %8s" % ("exec count", "instrs", "thr/unit", "warp%", "samples%"))
    for w, (n, t, s, _) in sorted(groups.items(), key=lambda kv: -kv[0] * kv[1][0])[:25]:
        print("%12d %6d %10.3f %7.1f%% %7.1f%%" % (w, n, t / units, 100.0 * w * n / tot_w, 100.0 * s / max(tot_s, 1)))


if __name__ == "__main__":
    main()
