#!/bin/bash
# Per-class timing of the main kernel (DASP_PROFILE_CLASS: 2 = medium only, 3 = short only, 1 = long only)
# plus the co-scheduled vs separate comparison and the GPU test suite.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "co_schedule" > gpurun_out/pytest_cosched.log 2>&1; echo "pytest cosched rc=$?"; tail -3 gpurun_out/pytest_cosched.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph"
: > gpurun_out/class.jsonl
for cfg in "c3" "c5 --scale 0.05"; do for dt in f64 f16; do
  for pc in 1 2 3; do DASP_PROFILE_CLASS=$pc timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/class.jsonl 2>> gpurun_out/class.err; echo "# class $pc" >> gpurun_out/class.jsonl; done
  for cs in 0 1; do timeout 300 $B --config $cfg --dtype $dt --co-schedule $cs >> gpurun_out/class.jsonl 2>> gpurun_out/class.err; done
done; done
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
echo done
