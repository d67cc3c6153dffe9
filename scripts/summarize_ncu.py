#!/usr/bin/env python
"""Summaries of ncu output for profiles/ (run on the CPU box, no GPU needed).

  summarize_ncu.py rep  <file.ncu-rep> [...]   key metrics of each profiled launch
  summarize_ncu.py launches <launches.csv>      per-kernel share of a launch list
"""
import collections
import csv
import io
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "DRAM % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit rate"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 throughput %"),
    ("l1tex__throughput.avg.pct_of_peak_sustained_active", "L1/smem throughput %"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__shared_mem_per_block_dynamic", "dyn smem/block"),
    ("launch__occupancy_limit_registers", "occupancy limit (regs, blocks)"),
    ("launch__occupancy_limit_shared_mem", "occupancy limit (smem, blocks)"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("smsp__inst_executed.sum", "instructions executed"),
    ("smsp__warps_launched.sum", "warps launched"),
    ("l1tex__t_bytes_pipe_lsu_mem_local_op_ld.sum", "local (spill) load bytes"),
    ("l1tex__t_bytes_pipe_lsu_mem_local_op_st.sum", "local (spill) store bytes"),
    ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "stall long_scoreboard/issue"),
    ("smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio", "stall barrier/issue"),
    ("smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio", "stall short_scoreboard/issue"),
    ("smsp__average_warps_issue_stalled_wait_per_issue_active.ratio", "stall wait/issue"),
    ("smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio", "stall math_pipe/issue"),
    ("smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio", "stall mio_throttle/issue"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
]


def rep(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = {"kernel": vals[hdr.index("Kernel Name")]}
        for k, label in KEYS:
            if k in hdr:
                i = hdr.index(k)
                d[label] = f"{vals[i]} {units[i]}".strip()
        res.append(d)
    return res


def launches(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 5]
    hdr = rows[0]
    ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
    mi = hdr.index("Metric Name") if "Metric Name" in hdr else None
    agg = collections.defaultdict(list)
    for r in rows[1:]:
        if mi is not None and r[mi] != "gpu__time_duration.sum":
            continue   # launch lists may carry more metrics (dram bytes); time only here
        try:
            agg[r[ki]].append(float(r[vi].replace(",", "")))
        except ValueError:
            pass
    tot = sum(sum(v) for v in agg.values())
    lines = ["| kernel | launches | total us | mean us | share |", "|---|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        lines.append(f"| {k[:70]} | {len(v)} | {sum(v)/1e3:.1f} | {sum(v)/len(v)/1e3:.2f} | "
                     f"{sum(v)/tot:.3f} |")
    return "\n".join(lines)


if __name__ == "__main__":
    if sys.argv[1] == "rep":
        for p in sys.argv[2:]:
            print(f"### {p}\n")
            for d in rep(p):
                print("| metric | value |\n|---|---|")
                for k, v in d.items():
                    print(f"| {k} | {v} |")
                print()
    else:
        print(launches(sys.argv[2]))
