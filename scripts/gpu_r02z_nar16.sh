#!/bin/bash
# FP16 stencil (mid path) knobs: row-blocks per narrow/mid warp 4 / 16, interleaved narrow warps
mkdir -p gpurun_out
O=gpurun_out/nar16.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/nar16.err; }
for cfg in "c2 --dtype f16" "c2big --dtype f16" "c3 --dtype f16" "c3"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so build/libdasp_DASP_NARROW_RB=4.so build/libdasp_DASP_NARROW_RB=16.so build/libdasp_DASP_NARROW_IL=1.so; do run "$lib" "$cfg"; done
done
echo done
