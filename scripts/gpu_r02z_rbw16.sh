#!/bin/bash
mkdir -p gpurun_out
O=gpurun_out/rbw16.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
for cfg in "c3 --dtype f16" "c5 --scale 0.05 --dtype f16" "c3"; do
  for r in 0 1 2 4 8; do echo "# rbw=$r cfg=$cfg" >> $O; timeout 300 $B --config $cfg --rbw $r >> $O 2>> gpurun_out/rbw16.err; done
done
echo done
