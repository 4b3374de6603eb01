#!/usr/bin/env python
"""Per-source-line totals of an ncu source export (`ncu -i X.ncu-rep --page source --csv
--print-source cuda,sass`): warp instructions, thread instructions and stall samples by (file, line).

  python tools/ncu_lines.py <export.csv> [top]
"""
import csv
import sys


def main():
    path = sys.argv[1]
    top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
    rows, fname, hdr = [], None, None
    tot_w = tot_s = 0
    for r in csv.reader(open(path)):
        if not r:
            continue
        if r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr and r[0] and r[0].isdigit():
            d = dict(zip(hdr[2:], r[2:]))
            try:
                w = int(d.get("Instructions Executed", "0") or 0)
                t = int(d.get("Thread Instructions Executed", "0") or 0)
                s = int(d.get("# Samples", "0") or 0)
            except ValueError:
                continue
            if w or s:
                rows.append((w, t, s, fname, int(r[0]), r[1].strip()[:90]))
                tot_w += w
                tot_s += s
    rows.sort(reverse=True)
    print("total warp instr %d, samples %d" % (tot_w, tot_s))
    for w, t, s, f, ln, src in rows[:top]:
        print("%5.1f%% w %5.1f%% s  %-16s %4d  %s" % (100.0 * w / tot_w, 100.0 * s / max(tot_s, 1), f, ln, src))


if __name__ == "__main__":
    main()
