#!/bin/bash
# mid narrow warps (two lanes per row): DASP_NARROW_MID=0/1, and DASP_NARROW=0 for reference
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 600 python -m pytest tests -m gpu -q -x -k narrow > gpurun_out/pytest_narrow.log 2>&1; echo "pytest narrow rc=$?"; tail -3 gpurun_out/pytest_narrow.log
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/narrow3.jsonl
for cfg in "c3" "c5 --scale 0.05"; do for dt in f64 f16 f32; do
  for mode in "DASP_NARROW=0" "DASP_NARROW_MID=0" "DASP_NARROW_MID=1"; do
    echo "# $mode" >> gpurun_out/narrow3.jsonl
    env $mode timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/narrow3.jsonl 2>> gpurun_out/narrow3.err
  done
done; done
for dt in f64 f16; do timeout 300 $B --config c2 --dtype $dt >> gpurun_out/narrow3.jsonl 2>> gpurun_out/narrow3.err; done
python scripts/show.py gpurun_out/narrow3.jsonl
echo done
