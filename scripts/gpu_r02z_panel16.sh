#!/bin/bash
mkdir -p gpurun_out
O=gpurun_out/panel16.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
for cfg in "c3 --dtype f16" "c5 --scale 0.05 --dtype f16"; do
  for pr in 0 4096 16384 32768 65536; do echo "# panel=$pr cfg=$cfg" >> $O; timeout 300 $B --config $cfg --panel-rows $pr >> $O 2>> gpurun_out/panel16.err; done
done
echo done
