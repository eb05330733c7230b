#!/bin/bash
# preferred shared-memory carveout for the main / long kernels: driver default vs 0 % (max L1) vs 50 %
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/carve.jsonl
for cfg in "c2" "c2 --dtype f16" "c2big" "c3" "c3 --dtype f16" "c5 --scale 0.05"; do for lib in base "DASP_CARVEOUT=0" "DASP_CARVEOUT=50" base; do
  echo "# $lib" >> gpurun_out/carve.jsonl
  if [ $lib = base ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$PWD/build/libdasp_$lib.so; fi
  DASP_LIB=$L timeout 300 $B --config $cfg >> gpurun_out/carve.jsonl 2>> gpurun_out/carve.err
done; done
python scripts/show.py gpurun_out/carve.jsonl | paste - - | awk '{print $2, $3, $4, $12, $13, $14, $15, $16, $17, $18}'
echo done
