#!/bin/bash
# next-row-block metadata prefetch in the CUDA-core wide medium loop (this build) vs off
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -k "parity" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/metapf.jsonl
for cfg in "c2" "c2big" "c3" "c5 --scale 0.05"; do for dt in f64 f32; do
  for lib in off on off on; do
    echo "# metapf $lib" >> gpurun_out/metapf.jsonl
    if [ $lib = on ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$PWD/build/libdasp_DASP_META_PF=0.so; fi
    DASP_LIB=$L timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/metapf.jsonl 2>> gpurun_out/metapf.err
  done
done; done
python scripts/show.py gpurun_out/metapf.jsonl
echo done
