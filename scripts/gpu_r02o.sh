#!/bin/bash
mkdir -p gpurun_out
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab13.jsonl
for rep in 1 2; do
for cfg in "c3" "c3 --dtype f16" "c5 --scale 0.05" "c7" "c7 --dtype f16"; do
  for lib in "" build/libdasp_DASP_LONG_UPW2=1.so; do
    echo "# lib=$lib cfg=$cfg" >> gpurun_out/ab13.jsonl
    DASP_LIB=${lib:-paper_conf_sc_lu023_b200/libdasp.so} timeout 300 $B --config $cfg >> gpurun_out/ab13.jsonl 2>> gpurun_out/ab13.err
  done
done
done
echo done
