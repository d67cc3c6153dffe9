#!/bin/bash
# r02p: micro_column without the unused terminal-velocity recompute after the last substep
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
AB="-DMICRO_SKIP_LAST_VT=0;-DMICRO_SKIP_LAST_VT=1" timeout 900 python scripts/ab_micro.py 2>&1 | tee gpurun_out/r02p_ab_micro.txt
for v in jit aot; do timeout 300 python scripts/profile_workloads.py --workload micro --variant $v --reps 8 2>&1 | tail -1; done | tee -a gpurun_out/r02p_ab_micro.txt
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_full.py -q -x -k micro 2>&1 | tail -2 | tee -a gpurun_out/r02p_ab_micro.txt
