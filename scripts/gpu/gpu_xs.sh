#!/bin/bash
export PROTEUS_LINEINFO=1   # ncu --import-source maps JIT kernels to their source
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "xs" 2>&1 | tail -2
for w in xs xs_large; do
for v in jit aot; do
timeout 300 python scripts/profile_workloads.py --workload $w --variant $v --reps 6 2>&1 | tail -1
done
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/xs_launches.csv python scripts/profile_workloads.py --workload xs --variant jit --reps 4 > /dev/null 2>&1; echo ncu rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:xs_lookup -s 1 -c 1 -f -o gpurun_out/xs_jit_ws python scripts/profile_workloads.py --workload xs --variant jit --reps 2 > /dev/null 2>&1; echo ncu rc=$?
