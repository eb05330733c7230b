#!/bin/bash
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_r.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_r.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab16.jsonl
for cfg in "c3" "c3 --dtype f16" "c5 --scale 0.05" "c5 --scale 0.05 --dtype f16" "c5 --scale 0.05 --dtype f32" "c2" "c2 --dtype f16"; do
  timeout 300 $B --config $cfg >> gpurun_out/ab16.jsonl 2>> gpurun_out/ab16.err
done
timeout 1500 python bench.py --config c5 --steps 30 --warmup 3 --e2e-steps 0 --no-compare --no-graph --no-cpu-baseline --no-triad > gpurun_out/c5full_r.jsonl 2> gpurun_out/c5full_r.err; echo "c5 rc=$?"
echo done
