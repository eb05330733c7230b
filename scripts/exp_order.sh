#!/bin/bash
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 100 --warmup 5 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/order.jsonl
for lo in 0 1; do
 for cfg in "c3" "c7" "c2" "c6 --scale 20"; do
  for v in mma cudacore; do
   echo "{\"order\": $lo}" >> gpurun_out/order.jsonl
   DASP_LONG_ORDER=$lo timeout 300 $B --config $cfg --variant $v >> gpurun_out/order.jsonl 2>> gpurun_out/order.err
  done
 done
done
for cfg in "c3" "c2"; do for v in mma cudacore; do
   echo "{\"order\": 1}" >> gpurun_out/order.jsonl
   timeout 300 $B --config $cfg --variant $v --dtype f16 >> gpurun_out/order.jsonl 2>> gpurun_out/order.err
done; done
S="python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dasp_main -s 3 -c 1 -o gpurun_out/prof_c6 $S --config c6 --scale 20 > gpurun_out/ncu_c6.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dasp_main -s 3 -c 1 -o gpurun_out/prof_c3 $S --config c3 > gpurun_out/ncu_c3.log 2>&1
echo done
