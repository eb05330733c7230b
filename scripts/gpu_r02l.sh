#!/bin/bash
# round 2: FP16 main kernel (CUDA-core) at 5 blocks / 48 registers with 2 or 3 short tiles per warp
mkdir -p gpurun_out
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub --dtype f16"
: > gpurun_out/ab10.jsonl
for rep in 1 2; do
for cfg in "c2" "c2big" "c3" "c5 --scale 0.05" "c6 --scale 20" "c7"; do
  for lib in "" build/libdasp_DASP_SHORT_TPW_F16=3.so "build/libdasp_DASP_MIN_BLOCKS_F16=5+DASP_SHORT_TPW_F16=3.so" "build/libdasp_DASP_MIN_BLOCKS_F16=5+DASP_SHORT_TPW_F16=2.so"; do
    echo "# lib=$lib cfg=$cfg" >> gpurun_out/ab10.jsonl
    DASP_LIB=${lib:-paper_conf_sc_lu023_b200/libdasp.so} timeout 300 $B --config $cfg >> gpurun_out/ab10.jsonl 2>> gpurun_out/ab10.err
  done
done
done
echo done
