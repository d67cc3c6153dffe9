#!/bin/bash
# One measurement pass: tests, bench line, launch list, ncu --set full per workload/variant.
# usage: bash scripts/gpu/gpu_round.sh TAG [workloads...]
TAG=${1:-r01}; shift
WL=${@:-stencil adam xs micro}
export PROTEUS_LINEINFO=1   # ncu --import-source maps JIT kernels to their source
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
timeout 900 python bench.py > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err; echo bench rc=$?
tail -2 gpurun_out/bench_${TAG}.err; cat gpurun_out/bench_${TAG}.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv python bench.py --steps 20 --warmup 3 --job-sweeps 20 --cpu-seconds 1 > /dev/null 2>&1; echo ncu-launch rc=$?
for w in $WL; do
  case $w in stencil) K=stencil4;; adam) K=adam_step;; xs) K=xs_lookup;; micro) K=micro_column;; esac
  for v in jit aot; do
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:$K -s 2 -c 1 -f -o gpurun_out/${w}_${v}_${TAG} python scripts/profile_workloads.py --workload $w --variant $v --reps 3 > gpurun_out/prof_${w}_${v}_${TAG}.log 2>&1; echo ncu $w $v rc=$?
    timeout 300 python scripts/profile_workloads.py --workload $w --variant $v --reps 8 2>&1 | tail -1
  done
done
