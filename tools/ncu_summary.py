#!/usr/bin/env python3
"""Summarise ncu outputs for profiles/: a launch list CSV (gpu__time_duration per launch) and/or a
--set full report of the update kernel. Usage:
  python tools/ncu_summary.py launches <launches.csv>
  python tools/ncu_summary.py report <prof.ncu-rep>"""
import collections
import csv
import io
import subprocess
import sys


def launches(path):
    lines = open(path).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    rows = list(csv.DictReader(io.StringIO("\n".join(lines[start:]))))
    d, cnt = collections.OrderedDict(), collections.Counter()
    for x in rows:
        if x.get("Metric Name") == "gpu__time_duration.sum":
            k = x["Kernel Name"].split("(")[0]
            d[k] = d.get(k, 0.0) + float(x["Metric Value"].replace(",", "")) / 1e6
            cnt[k] += 1
    tot = sum(d.values())
    print(f"{'ms':>10s} {'launches':>8s} {'share':>6s}  kernel")
    for k, v in sorted(d.items(), key=lambda t: -t[1]):
        print(f"{v:10.3f} {cnt[k]:8d} {100 * v / tot:5.1f}%  {k}")
    print(f"{tot:10.3f} total (cold-cache, serialised: compare shares, not absolutes)")


WANT = ["Kernel Name", "gpu__time_duration.sum", "launch__grid_size", "launch__block_size",
        "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__bytes_read.sum.per_second",
        "dram__cycles_active.avg.pct_of_peak_sustained_elapsed", "lts__t_requests_srcunit_tex_op_read.sum",
        "lts__t_sectors_srcunit_tex_op_read.sum", "lts__t_sectors_srcunit_tex_op_write.sum",
        "lts__t_sector_hit_rate.pct", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        # 32-B sector efficiency of the global loads / stores (useful bytes per sector moved; 32 = 100 %)
        "smsp__sass_average_data_bytes_per_sector_mem_global_op_ld.ratio",
        "smsp__sass_average_data_bytes_per_sector_mem_global_op_st.ratio",
        "l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum"]


def report(path):
    """path: a .ncu-rep, or the --page raw --csv export of one (*.csv)."""
    if path.endswith(".csv"):
        out = open(path).read()
    else:
        out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    for vals in rows[2:]:
        d = dict(zip(hdr, zip(vals, units)))
        for w in WANT:
            if w in d:
                print(f"{w:72s} {d[w][0]:>28s} {d[w][1]}")
        print()


if __name__ == "__main__":
    {"launches": launches, "report": report}[sys.argv[1]](sys.argv[2])
