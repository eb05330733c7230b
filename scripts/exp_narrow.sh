#!/bin/bash
# A/B of the narrow medium path: previous build (exp/libdasp_old.so) vs this build with
# DASP_NARROW=0 / 1, on the configs with narrow row-blocks (C3, C5, C6 has none) and the stencils
# (no narrow row-blocks: register-allocation check).  Output: gpurun_out/narrow.jsonl
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/narrow.jsonl
for cfg in "c3" "c5 --scale 0.05" "c2" "c2big"; do for dt in f64 f32; do
  echo "# old" >> gpurun_out/narrow.jsonl
  DASP_LIB=$PWD/exp/libdasp_old.so timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/narrow.jsonl 2>> gpurun_out/narrow.err
  for nw in 0 1; do
    echo "# narrow $nw" >> gpurun_out/narrow.jsonl
    DASP_NARROW=$nw timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/narrow.jsonl 2>> gpurun_out/narrow.err
  done
done; done
for nw in 0 1; do
  echo "# narrow $nw class 2" >> gpurun_out/narrow.jsonl
  DASP_NARROW=$nw DASP_PROFILE_CLASS=2 timeout 300 $B --config c3 >> gpurun_out/narrow.jsonl 2>> gpurun_out/narrow.err
done
python scripts/show.py gpurun_out/narrow.jsonl
echo done
