#!/bin/bash
# r02e: full GPU suite + bench (suite key, 5-run rotated e2e) + XS breakdown + ncu of the 4 JIT kernels
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 | tee gpurun_out/r02e_gpu_tests.txt
timeout 300 python scripts/xs_step_breakdown.py 2>&1 | tail -4 | tee gpurun_out/r02e_xs_breakdown.txt
timeout 1500 python bench.py > gpurun_out/bench_r02e.json 2> gpurun_out/bench_r02e.err; echo bench rc=$?
tail -3 gpurun_out/bench_r02e.err
for w in xs micro adam_run stencil; do
  K=$w; case $w in xs) K=xs_lookup;; micro) K=micro_column;; stencil) K=stencil4_ws;; esac
  STENCIL_ENTRY=stencil4_ws timeout 600 ncu --set full --clock-control none --import-source on -k regex:${K}__jit -s 1 -c 1 -f -o gpurun_out/${w}_jit_r02e python scripts/profile_workloads.py --workload $w --variant jit --reps 3 > gpurun_out/prof_${w}_r02e.log 2>&1; echo ncu $w rc=$?
done
