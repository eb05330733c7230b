#!/bin/bash
# FP16 / FP32 long kernel: two units per warp (UPW 2) at 64 / 48 registers, and 32 registers (8 blocks/SM)
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -k "long or parity_small or c1b" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/longf16.jsonl
for cfg in "c3" "c7" "c5 --scale 0.05"; do for dt in f16 f32; do
  for lib in base "DASP_LONG_UPW_F16=2+DASP_LONG_MIN_BLOCKS_F16=4" "DASP_LONG_UPW_F16=2+DASP_LONG_MIN_BLOCKS_F16=5" "DASP_LONG_MIN_BLOCKS_F16=8"; do
    echo "# $lib" >> gpurun_out/longf16.jsonl
    if [ $lib = base ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$PWD/build/libdasp_$lib.so; fi
    DASP_LIB=$L timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/longf16.jsonl 2>> gpurun_out/longf16.err
  done
done; done
python scripts/show.py gpurun_out/longf16.jsonl
echo done
