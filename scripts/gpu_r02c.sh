#!/bin/bash
# round 2: medium chunk units -- parity, A/B on / off on every config
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "units or integer or knobs or panels" > gpurun_out/pytest_units.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_units.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab3.jsonl
for cfg in "c3" "c3 --dtype f16" "c3 --dtype f32" "c5 --scale 0.05" "c5 --scale 0.05 --dtype f16" "c2" "c2big" "c2 --dtype f16" "c3 --variant mma" "c6 --scale 20" "c7"; do
  for u in "" "--no-medium-units"; do
    echo "# cfg=$cfg $u" >> gpurun_out/ab3.jsonl
    timeout 300 $B --config $cfg $u >> gpurun_out/ab3.jsonl 2>> gpurun_out/ab3.err
  done
done
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest all rc=$?"; tail -5 gpurun_out/pytest_gpu.log
echo done
