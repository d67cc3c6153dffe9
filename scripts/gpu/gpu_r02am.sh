#!/bin/bash
# r02am: where xs_scatter's time goes (scripts/native/exp_scatter.cu)
mkdir -p gpurun_out
nvcc -arch=sm_100a -O3 -std=c++17 -Ipaper_conf_cgo_georgakoudispb25_b200/csrc/kernels -o /tmp/exp_scatter scripts/native/exp_scatter.cu && timeout 120 /tmp/exp_scatter | tee gpurun_out/exp_scatter_r02am.txt
