#!/bin/bash
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 400 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare --no-gpu-build"
: > gpurun_out/split.jsonl
for sp in 0 1; do for cfg in "c3" "c6 --scale 20" "c5 --scale 0.05" "c2"; do for dt in f64 f16; do
  echo "{\"split\": $sp}" >> gpurun_out/split.jsonl
  DASP_SPLIT_SHORT=$sp timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/split.jsonl 2>> gpurun_out/split.err
done; done; done
echo done
