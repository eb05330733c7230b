#!/bin/bash
mkdir -p gpurun_out
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab19.jsonl
for cfg in "c2big" "c2" "c2big --dtype f16"; do
  for pr in 0 -1 1417176 2125764 524288; do
    echo "# panel=$pr cfg=$cfg" >> gpurun_out/ab19.jsonl
    timeout 300 $B --config $cfg --panel-rows $pr >> gpurun_out/ab19.jsonl 2>> gpurun_out/ab19.err
  done
done
echo done
