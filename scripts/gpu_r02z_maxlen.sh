#!/bin/bash
# MAX_LEN sweep ("an adjustable parameter"): rows longer than max_len go to the long-row
# (grouped, one-round-trip unit) path instead of the wide medium row-block path.
mkdir -p gpurun_out
O=gpurun_out/maxlen.jsonl
: > $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,power.limit --format=csv > gpurun_out/smi_maxlen.txt
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
for cfg in "c3" "c3 --dtype f16" "c3 --dtype f32" "c5 --scale 0.05" "c5 --scale 0.05 --dtype f16"; do
  for ml in 0 128 96 64 48 32; do
    echo "# max_len=$ml cfg=$cfg" >> $O
    timeout 300 $B --config $cfg --max-len $ml >> $O 2>> gpurun_out/maxlen.err
  done
done
echo done
