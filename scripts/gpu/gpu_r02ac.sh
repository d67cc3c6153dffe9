#!/bin/bash
# r02ac: ncu of adam_step at n = 2^26 (CFG 1's HBM-bound shape), JIT and AOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in jit aot; do
  R="adam_step__jit"; [ $v = aot ] && R="^adam_step$"
  timeout 600 ncu --set full --clock-control none -k regex:$R -s 2 -c 1 -f -o gpurun_out/adam_step_2p26_${v}_r02ac python scripts/profile_workloads.py --workload adam --variant $v --reps 4 --n-adam 67108864 > gpurun_out/prof_adam_2p26_${v}.log 2>&1; echo ncu $v rc=$?
  timeout 300 python scripts/profile_workloads.py --workload adam --variant $v --reps 10 --n-adam 67108864 2>&1 | tail -1
done
