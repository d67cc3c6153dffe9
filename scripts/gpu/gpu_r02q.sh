#!/bin/bash
# r02q: final-state check -- GPU tests, smoke, bench line, ncu of the four JIT kernels
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q 2>&1 | tail -4 | tee gpurun_out/r02q_gpu_tests.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1 | cut -c1-200 | tee gpurun_out/r02q_smoke.txt
s=$(date +%s); timeout 1500 python bench.py > gpurun_out/bench_r02q.json 2> gpurun_out/bench_r02q.err; echo bench rc=$? wall=$(( $(date +%s) - s ))s
for w in stencil xs micro adam_run; do
  K=$w; case $w in xs) K=xs_lookup;; micro) K=micro_column;; stencil) K=stencil4_ws;; esac
  for v in jit aot; do
    R="${K}__jit"; [ $v = aot ] && R="^${K}$"
    STENCIL_ENTRY=stencil4_ws timeout 600 ncu --set full --clock-control none -k regex:$R -s 1 -c 1 -f -o gpurun_out/${w}_${v}_r02q python scripts/profile_workloads.py --workload $w --variant $v --reps 3 > /dev/null 2>&1; echo ncu $w $v rc=$?
  done
done
