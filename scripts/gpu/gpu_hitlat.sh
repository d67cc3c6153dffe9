#!/bin/bash
# native in-memory-hit launch latency (no Python in the loop)
mkdir -p gpurun_out
g++ -O2 -std=c++17 -Iinclude scripts/native/hit_latency.cpp -o gpurun_out/hit_latency \
    -Lpaper_conf_cgo_georgakoudispb25_b200 -lproteus -Wl,-rpath,$PWD/paper_conf_cgo_georgakoudispb25_b200 -ldl || exit 1
for K in 1 16 256; do
  timeout 300 gpurun_out/hit_latency paper_conf_cgo_georgakoudispb25_b200/csrc/kernels/daxpy.cu $K 20000
done | tee gpurun_out/hit_latency.jsonl
