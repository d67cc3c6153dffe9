#!/bin/bash
# bench + launch list + ncu full captures of the stencil (jit and aot)
set -x
export PROTEUS_LINEINFO=1   # ncu --import-source maps JIT kernels to their source
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
timeout 600 python bench.py > gpurun_out/bench_r01.json 2> gpurun_out/bench_r01.err; echo bench rc=$?
tail -3 gpurun_out/bench_r01.err
cat gpurun_out/bench_r01.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01.csv python bench.py --steps 20 --warmup 3 --job-sweeps 20 --cpu-seconds 1 > gpurun_out/bench_under_ncu.json 2>&1; echo ncu-launch rc=$?
for v in jit aot; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:stencil4 -s 2 -c 1 -f -o gpurun_out/stencil_${v}_r01 python scripts/profile_workloads.py --workload stencil --variant $v --reps 4 > gpurun_out/prof_stencil_${v}.log 2>&1; echo ncu-$v rc=$?
done
for w in adam xs micro; do for v in jit aot; do
  timeout 300 python scripts/profile_workloads.py --workload $w --variant $v --reps 5 2>&1 | tail -1
done; done
