#!/bin/bash
# r01h ncu captures: current xs step (launch list + full capture of xs_lookup), stencil4_ws bench kernel.
export PROTEUS_LINEINFO=1   # ncu --import-source maps JIT kernels to their source
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/xs_launches_r01h.csv python scripts/profile_workloads.py --workload xs --variant jit --reps 3 > /dev/null 2>&1; echo ncu-xs-list rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:xs_lookup -s 2 -c 1 -f -o gpurun_out/xs_jit_r01h python scripts/profile_workloads.py --workload xs --variant jit --reps 3 > /dev/null 2>&1; echo ncu-xs rc=$?
STENCIL_ENTRY=stencil4_ws timeout 600 ncu --set full --clock-control none --import-source on -k regex:stencil4_ws -s 2 -c 1 -f -o gpurun_out/stencil_ws_jit_r01h python scripts/profile_workloads.py --workload stencil --variant jit --reps 3 > /dev/null 2>&1; echo ncu-st rc=$?
timeout 300 python scripts/profile_workloads.py --workload xs --variant jit --reps 8 2>&1 | tail -1
