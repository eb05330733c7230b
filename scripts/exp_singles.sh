#!/bin/bash
# singles tile lane mapping: transposed (this build) vs 4 consecutive per lane (DASP_SINGLES_T=0)
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/singles.jsonl
for cfg in "c3" "c6 --scale 20" "c5 --scale 0.05"; do for dt in f64 f16 f32; do
  for lib in T0 T1 T0 T1; do
    echo "# singles $lib" >> gpurun_out/singles.jsonl
    if [ $lib = T1 ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$PWD/build/libdasp_DASP_SINGLES_T=0.so; fi
    DASP_LIB=$L timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/singles.jsonl 2>> gpurun_out/singles.err
  done
done; done
python scripts/show.py gpurun_out/singles.jsonl
echo done
