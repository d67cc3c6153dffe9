#!/bin/bash
# r02n: stencil4_ws z-chunks in alternating march directions (WS_ALT) -- A/B, parity, ncu DRAM
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do for A in 0 1; do
echo "== WS_ALT=$A rep $rep" | tee -a gpurun_out/r02n2_alt.txt
EXTRA="-DWS_ALT=$A" CONFIGS="4,2,6;4,2,8" ZCS="4,6,8" timeout 600 python scripts/tune_stencil_ws.py 2>&1 | grep -v BEST | tee -a gpurun_out/r02n2_alt.txt
done; done
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_full.py tests/test_gpu_p2p.py -q -x -k "stencil or zslab or p2p or slab" 2>&1 | tail -4 | tee gpurun_out/r02n2_tests.txt
STENCIL_ENTRY=stencil4_ws timeout 600 ncu --set full --clock-control none -k regex:stencil4_ws__jit -s 1 -c 1 -f -o gpurun_out/stencil_alt_r02n2 python scripts/profile_workloads.py --workload stencil --variant jit --reps 3 > /dev/null 2>&1; echo ncu rc=$?
