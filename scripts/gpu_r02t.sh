#!/bin/bash
mkdir -p gpurun_out
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab18.jsonl
for cfg in "c6 --scale 20 --dtype f32" "c6 --scale 20" "c6 --scale 20 --dtype f16" "c3 --dtype f32" "c3" "c5 --scale 0.05 --dtype f32"; do
  timeout 300 $B --config $cfg >> gpurun_out/ab18.jsonl 2>> gpurun_out/ab18.err
done
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "integer or occupancy or lens" > gpurun_out/pytest_t.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_t.log
echo done
