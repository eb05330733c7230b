#!/bin/bash
# round 2: heavy blocks first (DASP_HEAVY_FIRST) A/B, interleaved with the default library
mkdir -p gpurun_out
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab5.jsonl
for rep in 1 2; do
for cfg in "c3" "c3 --dtype f16" "c5 --scale 0.05" "c2big" "c2" "c6 --scale 20"; do
  for lib in "" build/libdasp_DASP_HEAVY_FIRST=1.so build/libdasp_DASP_HEAVY_FIRST=2.so build/libdasp_DASP_HEAVY_FIRST=4.so; do
    echo "# lib=$lib cfg=$cfg" >> gpurun_out/ab5.jsonl
    DASP_LIB=${lib:-paper_conf_sc_lu023_b200/libdasp.so} timeout 300 $B --config $cfg >> gpurun_out/ab5.jsonl 2>> gpurun_out/ab5.err
  done
done
done
echo done
