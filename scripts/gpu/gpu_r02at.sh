#!/bin/bash
# r02at: validation after the per-block counting sort (dc6eb82) in a fresh container:
# GPU tests, smoke, default bench line, launch list of the bench command, ncu --set full of
# the bench kernel (JIT) and the XS sort kernels.
export PROTEUS_LINEINFO=1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02at_build.log 2>&1; echo build rc=$?
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -4 | tee gpurun_out/r02at_gpu_tests.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1 | cut -c1-160 | tee gpurun_out/r02at_smoke.txt
s=$(date +%s); timeout 1500 python bench.py > gpurun_out/bench_r02at.json 2> gpurun_out/bench_r02at.err; echo bench rc=$? wall=$(( $(date +%s) - s ))s
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r02at.csv python bench.py --steps 20 --warmup 3 --job-sweeps 20 --cpu-seconds 1 > /dev/null 2>&1; echo ncu-launch rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:stencil4_ws -s 2 -c 1 -f -o gpurun_out/stencil_jit_r02at python scripts/profile_workloads.py --workload stencil --variant jit --reps 3 > gpurun_out/prof_stencil_jit_r02at.log 2>&1; echo ncu stencil rc=$?
