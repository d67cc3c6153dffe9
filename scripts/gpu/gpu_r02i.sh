#!/bin/bash
# r02i: adam_run one-SFU-op reciprocal (ADAM_INV_RSQ) A/B + parity
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
AB="-DADAM_INV_RSQ=0;-DADAM_INV_RSQ=1;-DADAM_INV_RSQ=1 -DADAM_RCP_SPLIT=0" MINB=5 timeout 600 python scripts/ab_adam.py 2>&1 | tee gpurun_out/r02i_ab_adam.txt
AB="-DADAM_INV_RSQ=1" MINB=4 timeout 600 python scripts/ab_adam.py 2>&1 | tail -1 | tee -a gpurun_out/r02i_ab_adam.txt
AB="-DADAM_INV_RSQ=1" MINB=6 timeout 600 python scripts/ab_adam.py 2>&1 | tail -1 | tee -a gpurun_out/r02i_ab_adam.txt
AB="-DADAM_INV_RSQ=1" MINB=8 timeout 600 python scripts/ab_adam.py 2>&1 | tail -1 | tee -a gpurun_out/r02i_ab_adam.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "adam" 2>&1 | tail -3 | tee gpurun_out/r02i_adam_tests.txt
timeout 600 python bench.py --workload adam --steps 50 --warmup 5 2>/dev/null | tee gpurun_out/r02i_bench_adam.json
