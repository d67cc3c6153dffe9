#!/bin/bash
# r02av: the 13/16-material XS sort test (global bucket rows), the sanitizer skip, the
# launch list of a short bench command (the r02at one timed out under ncu: the default
# command runs ~40 000 launches), ncu --set full of the bench kernel (JIT + AOT) and of the
# XS step's kernels (JIT)
export PROTEUS_LINEINFO=1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -q -k "global_bucket_rows or sanitizer or xs_vs_oracle" 2>&1 | tail -4 | tee gpurun_out/r02av_tests.txt
CMD="python bench.py --steps 20 --warmup 3 --job-sweeps 20 --e2e-processes 0 --no-suite --cpu-seconds 1"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r02av.csv $CMD > gpurun_out/launches_r02av.log 2>&1; echo ncu-launch rc=$?
for v in jit aot; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:stencil4_ws -s 2 -c 1 -f -o gpurun_out/stencil_${v}_r02av python scripts/profile_workloads.py --workload stencil --variant $v --reps 3 > gpurun_out/prof_stencil_${v}_r02av.log 2>&1; echo ncu stencil $v rc=$?
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"xs_(bin|scan|scatter|lookup)" -s 4 -c 4 -f -o gpurun_out/xs_step_jit_r02av python scripts/profile_workloads.py --workload xs --variant jit --reps 2 > gpurun_out/prof_xs_jit_r02av.log 2>&1; echo ncu xs rc=$?
