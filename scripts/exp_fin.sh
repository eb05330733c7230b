#!/bin/bash
# Long-row phase 2 + empty rows fused into the main kernel: full GPU suite, then the configs with long / empty rows.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare"
: > gpurun_out/fin.jsonl
for cfg in c3 c7 "c5 --scale 0.05" c1b c2; do
 for dt in f64 f16 f32; do
  timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/fin.jsonl 2>> gpurun_out/fin.err
 done
done
echo done
