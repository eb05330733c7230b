#!/bin/bash
# Current build: GPU test suite + timings of the main configs (all dtypes) -> gpurun_out/quick.jsonl
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph"
: > gpurun_out/quick.jsonl
for cfg in ${CFGS:-"c2" "c2big" "c3" "c5 --scale 0.05" "c6 --scale 20"}; do for dt in f64 f16 f32; do
  timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/quick.jsonl 2>> gpurun_out/quick.err
done; done
echo done
