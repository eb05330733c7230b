#!/bin/bash
# short tiles per warp 3 / 4 (FP16, FP32) vs 2; small-matrix narrow warps (nrw 4 when LOOP_NUM 1)
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/tpw.jsonl
for cfg in c1a c1b; do for dt in f64 f16; do timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/tpw.jsonl 2>> gpurun_out/tpw.err; done; done
for cfg in "c3" "c6 --scale 20" "c5 --scale 0.05"; do
  for lib in base "DASP_SHORT_TPW_F16=3" "DASP_SHORT_TPW_F16=4"; do
    echo "# $lib" >> gpurun_out/tpw.jsonl
    if [ $lib = base ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$PWD/build/libdasp_$lib.so; fi
    DASP_LIB=$L timeout 300 $B --config $cfg --dtype f16 >> gpurun_out/tpw.jsonl 2>> gpurun_out/tpw.err
  done
  for lib in base "DASP_SHORT_TPW_F32=3"; do
    echo "# $lib" >> gpurun_out/tpw.jsonl
    if [ $lib = base ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$PWD/build/libdasp_$lib.so; fi
    DASP_LIB=$L timeout 300 $B --config $cfg --dtype f32 >> gpurun_out/tpw.jsonl 2>> gpurun_out/tpw.err
  done
done
python scripts/show.py gpurun_out/tpw.jsonl
echo done
