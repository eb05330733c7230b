#!/bin/bash
# tau sweep ("a customized parameter"): regular-block threshold
mkdir -p gpurun_out
O=gpurun_out/tau.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
for cfg in "c3" "c3 --dtype f16" "c5 --scale 0.05" "c2"; do
  for tau in 0.75 0.5 0.625 0.875 1.0; do echo "# tau=$tau cfg=$cfg" >> $O; timeout 300 $B --config $cfg --tau $tau >> $O 2>> gpurun_out/tau.err; done
done
echo done
