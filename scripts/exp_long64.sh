#!/bin/bash
# FP64 long kernel at 32 registers (DASP_LONG_MIN_BLOCKS=8) vs 40 (6); FP16/FP32 now at 32 (check)
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/long64.jsonl
for cfg in "c3" "c7" "c5 --scale 0.05"; do
  for lib in base "DASP_LONG_MIN_BLOCKS=8" base "DASP_LONG_MIN_BLOCKS=8"; do
    echo "# $lib" >> gpurun_out/long64.jsonl
    if [ $lib = base ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$PWD/build/libdasp_$lib.so; fi
    DASP_LIB=$L timeout 300 $B --config $cfg --dtype f64 >> gpurun_out/long64.jsonl 2>> gpurun_out/long64.err
  done
  for dt in f16 f32; do timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/long64.jsonl 2>> gpurun_out/long64.err; done
done
python scripts/show.py gpurun_out/long64.jsonl
echo done
