#!/bin/bash
# round 2: LOOP_NUM (row-blocks per wide medium warp) re-check on the ragged configs
mkdir -p gpurun_out
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab7.jsonl
for cfg in "c3" "c3 --dtype f16" "c5 --scale 0.05"; do
  for r in 0 1 2 3 6 8; do
    echo "# rbw=$r cfg=$cfg" >> gpurun_out/ab7.jsonl
    timeout 300 $B --config $cfg --rbw $r >> gpurun_out/ab7.jsonl 2>> gpurun_out/ab7.err
  done
done
echo done
