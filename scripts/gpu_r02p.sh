#!/bin/bash
# round 2: panel size re-check below the 1M-row default (rows of a row-block closer together ->
# their local x windows overlap in L1)
mkdir -p gpurun_out
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab14.jsonl
for cfg in "c5 --scale 0.05" "c3" "c3 --dtype f16" "c2"; do
  for pr in 0 4096 16384 65536 262144; do
    echo "# panel=$pr cfg=$cfg" >> gpurun_out/ab14.jsonl
    timeout 300 $B --config $cfg --panel-rows $pr >> gpurun_out/ab14.jsonl 2>> gpurun_out/ab14.err
  done
done
echo done
