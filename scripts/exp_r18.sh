#!/bin/bash
# Ragged-chunk block-by-block layout (R18): full GPU suite + medium-heavy configs, all dtypes.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare"
: > gpurun_out/r18.jsonl
for cfg in c2 c2big c3 "c5 --scale 0.05" "c6 --scale 20"; do
 for dt in f64 f16 f32; do
  timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/r18.jsonl 2>> gpurun_out/r18.err
 done
done
echo done
