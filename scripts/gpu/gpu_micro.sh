#!/bin/bash
export PROTEUS_LINEINFO=1   # ncu --import-source maps JIT kernels to their source
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "micro or spec_routines" 2>&1 | tail -2
timeout 600 ncu --set full --clock-control none --import-source on -k regex:micro_column -s 1 -c 1 -f -o gpurun_out/micro_jit_src python scripts/profile_workloads.py --workload micro --variant jit --reps 2 > gpurun_out/prof_micro.log 2>&1; echo ncu rc=$?
timeout 300 python scripts/profile_workloads.py --workload micro --variant jit --reps 8 2>&1 | tail -1
timeout 300 python scripts/profile_workloads.py --workload micro --variant aot --reps 8 2>&1 | tail -1
