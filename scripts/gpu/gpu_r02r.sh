#!/bin/bash
# r02r: micro_column with 32-bit indices -- timing, parity, ncu (spills)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in jit aot; do timeout 300 python scripts/profile_workloads.py --workload micro --variant $v --reps 8 2>&1 | tail -1; done | tee gpurun_out/r02r_micro.txt
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_full.py tests/test_gpu_ir.py -q -x -k micro 2>&1 | tail -2 | tee -a gpurun_out/r02r_micro.txt
for v in jit aot; do
  R="micro_column__jit"; [ $v = aot ] && R="^micro_column$"
  timeout 600 ncu --set full --clock-control none -k regex:$R -s 1 -c 1 -f -o gpurun_out/micro_${v}_r02r python scripts/profile_workloads.py --workload micro --variant $v --reps 3 > /dev/null 2>&1; echo ncu $v rc=$?
done
