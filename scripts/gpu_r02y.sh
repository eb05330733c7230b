#!/bin/bash
mkdir -p gpurun_out
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab20.jsonl
for cfg in "c3" "c3 --dtype f16" "c3 --dtype f32" "c5 --scale 0.05" "c6 --scale 20" "c1a"; do
  for lib in "" build/libdasp_DASP_NARROW_RB=4.so build/libdasp_DASP_NARROW_RB=16.so build/libdasp_DASP_SHORT_TPW_F64=1.so; do
    echo "# lib=$lib cfg=$cfg" >> gpurun_out/ab20.jsonl
    DASP_LIB=${lib:-paper_conf_sc_lu023_b200/libdasp.so} timeout 300 $B --config $cfg >> gpurun_out/ab20.jsonl 2>> gpurun_out/ab20.err
  done
done
echo done
