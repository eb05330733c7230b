#!/bin/bash
# Overlap mode (main kernel capped at k blocks/SM + long kernel on a second stream) vs serial.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "overlap" > gpurun_out/pytest_ovl.log 2>&1; echo "pytest ovl rc=$?"; tail -3 gpurun_out/pytest_ovl.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph"
: > gpurun_out/overlap.jsonl
for cfg in "c3" "c5 --scale 0.05" "c7" "c1b"; do for dt in f64 f16 f32; do for k in 0 2 3; do
  echo "# overlap $k" >> gpurun_out/overlap.jsonl
  DASP_OVERLAP=$k timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/overlap.jsonl 2>> gpurun_out/overlap.err
done; done; done
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
echo done
