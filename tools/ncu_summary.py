#!/usr/bin/env python
"""Summarise ncu outputs into the text files committed under profiles/.

  python tools/ncu_summary.py launches <launches.csv>      per-kernel count, mean/total device time, share
  python tools/ncu_summary.py full <report.ncu-rep>        key metrics of a --set full capture
"""
import csv
import io
import re
import subprocess
import sys
from collections import OrderedDict


def launches(path):
    lines = [l for l in open(path) if l.startswith('"')]
    rows = list(csv.DictReader(io.StringIO("".join(lines))))
    agg = OrderedDict()
    for r in rows:
        if r["Metric Name"] != "gpu__time_duration.sum":
            continue
        name = re.sub(r"\(.*", "", r["Kernel Name"]).replace("void ", "")
        ns = float(r["Metric Value"].replace(",", ""))
        a = agg.setdefault(name, [0, 0.0, r["Grid Size"], r["Block Size"]])
        a[0] += 1
        a[1] += ns
    tot = sum(v[1] for v in agg.values())
    print("%-46s %6s %12s %12s %7s  %s" % ("kernel", "count", "mean_us", "total_us", "share", "grid x block"))
    for k, (n, t, g, b) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print("%-46s %6d %12.2f %12.1f %6.1f%%  %s x %s" % (k[:46], n, t / n / 1e3, t / 1e3, 100 * t / tot, g, b))
    print("total device time of listed launches: %.1f us (%d launches)" % (tot / 1e3, sum(v[0] for v in agg.values())))


KEYS = ["gpu__time_duration.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__inst_executed.sum",
        "smsp__inst_executed.avg.per_cycle_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__occupancy_limit_registers", "launch__grid_size",
        "launch__block_size", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_alu.sum", "sm__inst_executed_pipe_fma.sum", "sm__inst_executed_pipe_lsu.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "sm__cycles_elapsed.avg.per_second",
        "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_branch_resolving_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active"]


def full(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    for r in rows[2:]:
        print("kernel:", r[hdr.index("Kernel Name")][:120])
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k)
                print("  %-72s %s %s" % (k, r[i], units[i]))


def short(name):
    name = re.sub(r"\(.*", "", name).replace("void ", "").replace("ap::", "")
    name = name.replace("unsigned long long", "u64").replace("unsigned int", "u32").replace("(bool)", "")
    name = name.replace("(int)", "").replace(", 256>", ">").replace(" ", "")
    return name


def traffic(path):
    """JSON of dram read + write bytes per captured launch (bench.py's roofline `traffic`)."""
    import json
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = OrderedDict()
    for r in rows[2:]:
        b = 0.0
        for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            i = hdr.index(k)
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(units[i], 1)
            b += float(r[i].replace(",", "")) * scale
        name = short(r[hdr.index("Kernel Name")])
        if name.startswith("k_search_r1<8,"):
            name = name.split(",")[0] + "," + name.split(",")[1] + ">" if name.count(",") >= 2 else name
        key = name
        n = 2
        while key in res:
            key = "%s#%d" % (name, n)
            n += 1
        res[key] = int(b)
    res["source"] = "ncu --set full, one launch each (tools/profile_kernels.py)"
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    {"launches": launches, "full": full, "traffic": traffic}[sys.argv[1]](sys.argv[2])
