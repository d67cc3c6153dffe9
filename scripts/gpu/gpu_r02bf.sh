#!/bin/bash
# r02bf: adam_run with the per-block fallback for non-finite folded factors: Adam GPU tests
# (incl. lr = 0 and 1e-30) and the kernel time (must stay at ~0.0478 ms)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -q -k "adam" 2>&1 | tail -4 | tee gpurun_out/r02bf_tests.txt
AB="-DADAM_FOLD=1;-DADAM_FOLD=0" timeout 900 python scripts/ab_adam.py 2>&1 | tee gpurun_out/ab_adam_guard_r02bf.txt
MODE=none AB="-DADAM_FOLD=1" timeout 900 python scripts/ab_adam.py 2>&1 | sed 's/^/none /' | tee -a gpurun_out/ab_adam_guard_r02bf.txt
