#!/bin/bash
# FP16 narrow path (DASP_NARROW=0/1) and the chunk software pipeline in FP64/FP32 (experiment build)
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/narrow2.jsonl
for cfg in "c3" "c5 --scale 0.05" "c2" "c2big"; do
  for nw in 0 1; do
    echo "# f16 narrow $nw" >> gpurun_out/narrow2.jsonl
    DASP_NARROW=$nw timeout 300 $B --config $cfg --dtype f16 >> gpurun_out/narrow2.jsonl 2>> gpurun_out/narrow2.err
  done
  for dt in f64 f32; do
    echo "# base" >> gpurun_out/narrow2.jsonl
    timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/narrow2.jsonl 2>> gpurun_out/narrow2.err
    echo "# chunk pipe" >> gpurun_out/narrow2.jsonl
    DASP_LIB=$PWD/build/libdasp_DASP_CHUNK_PIPE_F64=1+DASP_CHUNK_PIPE_F32=1.so timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/narrow2.jsonl 2>> gpurun_out/narrow2.err
  done
done
python scripts/show.py gpurun_out/narrow2.jsonl
echo done
