#!/bin/bash
# round-1 profiles after PDL + micro log_s rework: launch list of bench.py, ncu --set full of
# stencil4_ws (JIT) and micro_column (JIT, AOT)
export PROTEUS_LINEINFO=1   # ncu --import-source maps JIT kernels to their source
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01f.csv python bench.py --steps 20 --warmup 3 --job-sweeps 20 --cpu-seconds 1 > /dev/null 2>&1; echo ncu-launch rc=$?
STENCIL_ENTRY=stencil4_ws timeout 600 ncu --set full --clock-control none --import-source on -k regex:stencil4_ws -s 2 -c 1 -f -o gpurun_out/stencil_ws_jit_r01f python scripts/profile_workloads.py --workload stencil --variant jit --reps 3 > gpurun_out/prof_st.log 2>&1; echo ncu st rc=$?
for v in jit aot; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:micro_column -s 1 -c 1 -f -o gpurun_out/micro_${v}_r01f python scripts/profile_workloads.py --workload micro --variant $v --reps 2 > gpurun_out/prof_micro_$v.log 2>&1; echo ncu micro $v rc=$?
done
