#!/bin/bash
mkdir -p gpurun_out
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab15.jsonl
for cfg in "c3 --dtype f16" "c5 --scale 0.05 --dtype f16" "c2 --dtype f16" "c2big --dtype f16" "c6 --scale 20 --dtype f16" "c5 --scale 0.05" "c3 --dtype f32" "c5 --scale 0.05 --dtype f32" "c6 --scale 20"; do
  for pr in 0 8192 16384 32768; do
    echo "# panel=$pr cfg=$cfg" >> gpurun_out/ab15.jsonl
    timeout 300 $B --config $cfg --panel-rows $pr >> gpurun_out/ab15.jsonl 2>> gpurun_out/ab15.err
  done
done
echo done
