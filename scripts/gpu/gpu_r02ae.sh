#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for flags in "--no-e2e-jobs" ""; do
timeout 600 python bench.py --e2e-processes 0 --no-suite --cpu-seconds 1 $flags 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); s=d['speedup_vs_aot']; print('flags=$flags', d['ms_per_step'], s['aot_sweep_us'], s['jit_sweep_us'])"
done
