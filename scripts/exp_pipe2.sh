#!/bin/bash
mkdir -p gpurun_out
make -j8 all exp > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 600 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/pipe2.jsonl
for mode in direct pipe2 ns3 ns4; do
 case $mode in
  direct) E="DASP_PIPE=0";; pipe2) E="DASP_PIPE=1";;
  ns3) E="DASP_PIPE=1 DASP_LIB=build/libdasp_DASP_NSTAGE=3.so";; ns4) E="DASP_PIPE=1 DASP_LIB=build/libdasp_DASP_NSTAGE=4.so";;
 esac
 for cfg in "c2" "c3" "c7"; do for dt in f64 f16; do
  echo "{\"mode\": \"$mode\"}" >> gpurun_out/pipe2.jsonl
  env $E timeout 300 $B --config $cfg --dtype $dt --variant cudacore >> gpurun_out/pipe2.jsonl 2>> gpurun_out/pipe2.err
 done; done
done
echo done
