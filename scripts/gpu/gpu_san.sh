#!/bin/bash
export PROTEUS_LINEINFO=1   # ncu --import-source maps JIT kernels to their source
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_sanitizer.py -m gpu -q 2>&1 | tail -3
for M in 0 3 4 5; do
MINB=$M CONFIGS="4,2,6;4,2,8;3,2,6;7,1,8" ZCS="3,4,8" timeout 900 python scripts/tune_stencil_ws.py > gpurun_out/tune_ws_minb$M.txt 2>&1; echo minb $M; tail -1 gpurun_out/tune_ws_minb$M.txt | cut -c1-200
done
timeout 900 python bench.py > gpurun_out/bench_chk.json 2> gpurun_out/bench_chk.err; echo bench rc=$?
tail -3 gpurun_out/bench_chk.err; cat gpurun_out/bench_chk.json
STENCIL_ENTRY=stencil4_ws timeout 600 ncu --set full --clock-control none --import-source on -k regex:stencil4_ws -s 2 -c 1 -f -o gpurun_out/stencil_ws_jit_r01e python scripts/profile_workloads.py --workload stencil --variant jit --reps 3 > gpurun_out/prof_ws_jit.log 2>&1; echo ncu rc=$?
