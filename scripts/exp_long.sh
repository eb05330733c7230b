#!/bin/bash
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 && make exp EXPVARS="DASP_LONG_MIN_BLOCKS=6 DASP_LONG_MIN_BLOCKS_F16=8" >> gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare"
: > gpurun_out/long.jsonl
for lib in base "DASP_LONG_MIN_BLOCKS=6" "DASP_LONG_MIN_BLOCKS_F16=8"; do
 if [ "$lib" = base ]; then L=paper_conf_sc_lu023_b200/libdasp.so; else L="build/libdasp_$lib.so"; fi
 for cfg in c3 c7; do for dt in f64 f16; do
  echo "{\"lib\": \"$lib\"}" >> gpurun_out/long.jsonl
  DASP_LIB=$L timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/long.jsonl 2>> gpurun_out/long.err
 done; done
done
timeout 300 python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --config c2 >> gpurun_out/long.jsonl 2>> gpurun_out/long.err
echo done
