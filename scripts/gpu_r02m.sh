#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_m.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_m.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab11.jsonl
for cfg in "c2 --dtype f16" "c2big --dtype f16" "c3 --dtype f16" "c5 --scale 0.05 --dtype f16" "c6 --scale 20 --dtype f16" "c3" "c2"; do
  timeout 300 $B --config $cfg >> gpurun_out/ab11.jsonl 2>> gpurun_out/ab11.err
done
echo done
