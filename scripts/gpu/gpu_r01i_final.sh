#!/bin/bash
# r01i refresh: all GPU tests, smoke, CFG 1-5 suite, fresh-process e2e, bench line, ncu spec-vs-generic.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1 | cut -c1-120
timeout 2400 python bench_suite.py > gpurun_out/suite_r01i.jsonl 2> gpurun_out/suite_r01i.err; echo suite rc=$?
timeout 2400 python bench_suite.py --configs e2e:stencil,e2e:adam_run,e2e:xs,e2e:micro > gpurun_out/e2e_proc_r01i.jsonl 2> gpurun_out/e2e_proc_r01i.err; echo e2e rc=$?
timeout 900 python bench.py > gpurun_out/bench_r01i.json 2> gpurun_out/bench_r01i.err; echo bench rc=$?
timeout 300 python bench.py --workload adam --steps 300 --warmup 5 > gpurun_out/bench_adam_r01i.json 2>/dev/null; echo bench-adam rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01i.csv python bench.py --steps 20 --warmup 3 --job-sweeps 20 --cpu-seconds 1 --e2e-processes 0 > /dev/null 2>&1; echo ncu-launch rc=$?
TAG=r01i PROTEUS_LINEINFO=1 bash scripts/gpu/gpu_spec_vs_generic.sh 2>&1 | tail -8
