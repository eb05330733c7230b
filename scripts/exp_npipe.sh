#!/bin/bash
# narrow-path software pipeline (DASP_NARROW_PIPE) and the 85-register main kernel (MIN_BLOCKS=3)
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -k "narrow or parity_small or host" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/npipe.jsonl
for cfg in "c2" "c3" "c2big" "c5 --scale 0.05"; do for dt in f64 f16 f32; do
  for lib in base "DASP_NARROW_PIPE=1" "DASP_NARROW_PIPE=1+DASP_MIN_BLOCKS=3+DASP_MIN_BLOCKS_F16=3+DASP_MIN_BLOCKS_F32=3" "DASP_MIN_BLOCKS=3+DASP_MIN_BLOCKS_F16=3+DASP_MIN_BLOCKS_F32=3"; do
    echo "# $lib" >> gpurun_out/npipe.jsonl
    if [ $lib = base ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$PWD/build/libdasp_$lib.so; fi
    DASP_LIB=$L timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/npipe.jsonl 2>> gpurun_out/npipe.err
  done
done; done
python scripts/show.py gpurun_out/npipe.jsonl
echo done
