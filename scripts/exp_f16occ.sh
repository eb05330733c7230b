#!/bin/bash
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 && make exp EXPVARS="DASP_MIN_BLOCKS_F16=5 DASP_MIN_BLOCKS_F16=6 DASP_MIN_BLOCKS=5" >> gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare"
: > gpurun_out/f16occ.jsonl
for lib in base "DASP_MIN_BLOCKS_F16=5" "DASP_MIN_BLOCKS_F16=6" "DASP_MIN_BLOCKS=5"; do
 if [ "$lib" = base ]; then L=paper_conf_sc_lu023_b200/libdasp.so; else L="build/libdasp_$lib.so"; fi
 for cfg in c2 c3 c7; do for dt in f64 f16; do for v in cudacore mma; do
  echo "{\"lib\": \"$lib\"}" >> gpurun_out/f16occ.jsonl
  DASP_LIB=$L timeout 300 $B --config $cfg --dtype $dt --variant $v >> gpurun_out/f16occ.jsonl 2>> gpurun_out/f16occ.err
 done; done; done
done
echo done
