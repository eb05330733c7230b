#!/bin/bash
# A/B of the current build: GPU parity suite, then timings on the main configs (+ medium-only
# and short-only class timings of C3 / C5).  Output: gpurun_out/ab.jsonl
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph"
: > gpurun_out/ab.jsonl
for cfg in "c3" "c5 --scale 0.05" "c2" "c2big" "c6 --scale 20"; do for dt in f64 f16 f32; do
  timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/ab.jsonl 2>> gpurun_out/ab.err
done; done
for cfg in "c3" "c5 --scale 0.05"; do for dt in f64 f16; do for pc in 2 3; do
  echo "# class $pc" >> gpurun_out/ab.jsonl
  DASP_PROFILE_CLASS=$pc timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/ab.jsonl 2>> gpurun_out/ab.err
done; done; done
for v in mma; do timeout 300 $B --config c3 --variant $v >> gpurun_out/ab.jsonl 2>> gpurun_out/ab.err; done
echo done
