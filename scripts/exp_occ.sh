#!/bin/bash
mkdir -p gpurun_out
make -j8 all exp > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 100 --warmup 5 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/occ.jsonl
for mb in 4 5 6; do
 for cfg in "c3" "c2" "c6 --scale 20" "c7"; do
  for v in mma cudacore; do
   echo "{\"mb\": $mb, \"rbw\": 0}" >> gpurun_out/occ.jsonl
   DASP_LIB=build/libdasp_mb$mb.so timeout 300 $B --config $cfg --variant $v >> gpurun_out/occ.jsonl 2>> gpurun_out/occ.err
  done
 done
done
for rbw in 1 2 8; do
 for cfg in "c3" "c2"; do
   echo "{\"mb\": 5, \"rbw\": $rbw}" >> gpurun_out/occ.jsonl
   DASP_LIB=build/libdasp_mb5.so timeout 300 $B --config $cfg --rbw $rbw >> gpurun_out/occ.jsonl 2>> gpurun_out/occ.err
 done
done
echo done
