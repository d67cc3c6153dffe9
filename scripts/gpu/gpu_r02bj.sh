#!/bin/bash
# r02bj: bench.py repeats the W warm-up sweeps inside the clock sampler right before the
# timed region (short K started on a ramping clock): K = 20 lines, bench GPU tests
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for i in 1 2; do
  timeout 900 python bench.py --steps 20 --warmup 5 --no-suite --e2e-processes 0 > gpurun_out/bench_r02bj_k20_$i.json 2> gpurun_out/bench_r02bj_k20_$i.err; echo bench k20 rc=$?
  python -c "import json;d=json.load(open('gpurun_out/bench_r02bj_k20_$i.json'));print(d['value'],d['ms_per_step'],d['roofline']['frac'],d['clocks'])"
done
timeout 1800 python -m pytest tests -m gpu -q -k "bench" 2>&1 | tail -3 | tee gpurun_out/r02bj_tests.txt
