#!/bin/bash
# r02bi: validation of the r02 final kernels (den-folded adam_run + fallback, XS_PACK,
# XS_CA_LDG): every GPU test, smoke, the default bench line, the launch list of a short
# bench command
export PROTEUS_LINEINFO=1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02bi_build.log 2>&1; echo build rc=$?
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -4 | tee gpurun_out/r02bi_gpu_tests.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1 | cut -c1-200 | tee gpurun_out/r02bi_smoke.txt
s=$(date +%s); timeout 1500 python bench.py > gpurun_out/bench_r02bi.json 2> gpurun_out/bench_r02bi.err; echo bench rc=$? wall=$(( $(date +%s) - s ))s
s=$(date +%s); timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_r02bi_k20.json 2> gpurun_out/bench_r02bi_k20.err; echo bench k20 rc=$? wall=$(( $(date +%s) - s ))s
CMD="python bench.py --steps 20 --warmup 3 --job-sweeps 20 --e2e-processes 0 --no-suite --cpu-seconds 1"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r02bi.csv $CMD > gpurun_out/launches_r02bi.log 2>&1; echo ncu-launch rc=$?
