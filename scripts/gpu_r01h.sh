#!/bin/bash
# Re-entry verification: GPU tests, smoke, default bench line, launch list of the bench command.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -8
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -3
timeout 900 python bench.py > gpurun_out/bench_r01h.json 2> gpurun_out/bench_r01h.err; echo bench rc=$?
tail -3 gpurun_out/bench_r01h.err; cat gpurun_out/bench_r01h.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01h.csv python bench.py --steps 20 --warmup 3 --job-sweeps 20 --cpu-seconds 1 > /dev/null 2>&1; echo ncu-launch rc=$?
