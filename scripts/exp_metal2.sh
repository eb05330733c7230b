#!/bin/bash
# wide warps L2-prefetch their metadata lines at warp start (this build) vs off
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -k "parity" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_gpu.log
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/metal2.jsonl
for cfg in "c2" "c2big" "c3" "c5 --scale 0.05"; do for dt in f64 f32 f16; do for lib in off on off on; do
  echo "# $lib" >> gpurun_out/metal2.jsonl
  if [ $lib = on ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$PWD/build/libdasp_DASP_META_L2PF=0.so; fi
  DASP_LIB=$L timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/metal2.jsonl 2>> gpurun_out/metal2.err
done; done; done
python scripts/show.py gpurun_out/metal2.jsonl | paste - - | awk '{print $2, $3, $4, $12, $13, $14, $15, $16, $17, $18}'
echo done
