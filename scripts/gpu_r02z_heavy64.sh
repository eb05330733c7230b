#!/bin/bash
mkdir -p gpurun_out
O=gpurun_out/heavy64.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/heavy64.err; }
for rep in 1 2 3; do
for cfg in "c3" "c3 --dtype f32"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so build/libdasp_DASP_HEAVY_FIRST=0.so; do run "$lib" "$cfg"; done
done; done
echo done
