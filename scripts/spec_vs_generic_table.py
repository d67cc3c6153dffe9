#!/usr/bin/env python
"""Side-by-side ncu table of the specialized (JIT) and generic (AOT) variant of each
workload kernel from gpurun_out/sg_<w>_<v>_<tag>.ncu-rep (scripts/gpu/gpu_spec_vs_generic.sh).
  python scripts/spec_vs_generic_table.py <tag> > profiles/r01/ncu_spec_vs_generic_<tag>.md"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
TAG = sys.argv[1] if len(sys.argv) > 1 else "r01h"
# file name pattern: r01 captures are sg_<w>_<v>_<tag>.ncu-rep, r02's <w>_<v>_<tag>.ncu-rep
PAT = sys.argv[2] if len(sys.argv) > 2 else "sg_{w}_{v}_{tag}.ncu-rep"
# algorithmic bytes per launch: stencil 16 B/point, adam_run 28 B/param per
# run, xs 44 B of outputs + 4 B perm per lookup (+ the table, L2-resident), micro
# 2820 B/column
ALG = {"stencil": 16 * 256 ** 3, "adam_run": 28 * 10 ** 6, "xs": 48 * 10 ** 7,
       "micro": 2820 * 10 ** 6}
M = [("gpu__time_duration.sum", "duration (us)", 1e-3),
     ("dram__bytes_read.sum", "DRAM read (MB)", 1e-6),
     ("dram__bytes_write.sum", "DRAM write (MB)", 1e-6),
     ("launch__registers_per_thread", "registers/thread", 1),
     ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %", 1),
     ("smsp__inst_executed.sum", "warp instructions (M)", 1e-6),
     ("l1tex__t_requests_pipe_lsu_mem_local_op_ld.sum", "local-memory (spill) load requests", 1),
     ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %", 1),
     ("l1tex__throughput.avg.pct_of_peak_sustained_active", "L1/smem throughput %", 1),
     ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput %", 1)]


def raw(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv", "--print-units", "base"],
                         capture_output=True, text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return dict(zip(rows[0], rows[2]))


def num(s):
    return float(s.replace(",", ""))


peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
print(f"# Specialized (JIT, mode all) vs generic (nvcc AOT) kernels, ncu --set full, {TAG}\n")
print("One launch each at the BASELINE.json config, cold L2, `--clock-control none` "
      "(scripts/gpu/gpu_spec_vs_generic.sh).  Algorithmic GB/s = DESIGN.md §7 bytes per launch / "
      f"duration; HBM peak = MEASURED_PEAKS.json {peak} GB/s.\n")
for w in ("stencil", "adam_run", "xs", "micro"):
    d = {v: raw(os.path.join(ROOT, "gpurun_out", PAT.format(w=w, v=v, tag=TAG)))
         for v in ("jit", "aot")}
    print(f"## {w} ({d['jit']['Kernel Name']})\n")
    print("| metric | specialized | generic | generic / specialized |\n|---|---|---|---|")
    for k, label, sc in M:
        a, b = num(d["jit"][k]) * sc, num(d["aot"][k]) * sc
        print(f"| {label} | {a:.4g} | {b:.4g} | {b / a if a else float('nan'):.3f} |")
    ta, tb = num(d["jit"]["gpu__time_duration.sum"]), num(d["aot"]["gpu__time_duration.sum"])
    ga, gb = ALG[w] / ta, ALG[w] / tb   # bytes/ns = GB/s
    print(f"| algorithmic GB/s | {ga:.0f} | {gb:.0f} | {gb / ga:.3f} |")
    print(f"| fraction of HBM peak | {ga / peak:.3f} | {gb / peak:.3f} | |")
    da = (num(d['jit']['dram__bytes_read.sum']) + num(d['jit']['dram__bytes_write.sum'])) / ta
    db = (num(d['aot']['dram__bytes_read.sum']) + num(d['aot']['dram__bytes_write.sum'])) / tb
    print(f"| DRAM GB/s (measured bytes) | {da:.0f} | {db:.0f} | {db / da:.3f} |\n")
