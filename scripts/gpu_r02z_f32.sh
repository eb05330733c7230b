#!/bin/bash
mkdir -p gpurun_out
O=gpurun_out/f32.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/f32.err; }
for cfg in "c2 --dtype f32" "c2big --dtype f32" "c3 --dtype f32" "c5 --scale 0.05 --dtype f32"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "build/libdasp_DASP_PEEL_F32=1+DASP_WIDE_META_PF_F32=1.so" "build/libdasp_DASP_WIDE_META_PF_F32=1.so"; do run "$lib" "$cfg"; done
done
echo done
