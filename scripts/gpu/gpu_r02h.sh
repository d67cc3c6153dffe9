#!/bin/bash
# r02h: end-to-end jobs incl. JIT in fresh processes (5 rotated runs): ~2 s AOT jobs (Table 2
# scale) and the default short jobs; ncu of xs_lookup (minBlocks 9); bench launch list
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 2400 python bench_suite.py --configs e2e:stencil@36000,e2e:adam_run@37000,e2e:xs@1500,e2e:micro@900 --runs 5 > gpurun_out/e2e_2s_r02h.jsonl 2> gpurun_out/e2e_2s_r02h.err; echo e2e2s rc=$?
timeout 1500 python bench_suite.py --configs e2e:adam_run,e2e:xs,e2e:micro --runs 5 > gpurun_out/e2e_short_r02h.jsonl 2> gpurun_out/e2e_short_r02h.err; echo e2eshort rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:xs_lookup__jit -s 1 -c 1 -f -o gpurun_out/xs_jit_r02h python scripts/profile_workloads.py --workload xs --variant jit --reps 3 > gpurun_out/prof_xs_r02h.log 2>&1; echo ncu xs rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r02h.csv python bench.py --steps 20 --warmup 3 --job-sweeps 20 --cpu-seconds 1 --e2e-processes 0 --no-suite > gpurun_out/bench_under_ncu_r02h.log 2>&1; echo ncu-launch rc=$?
