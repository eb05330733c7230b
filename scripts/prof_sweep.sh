#!/bin/bash
# Per-config / per-variant bench sweep + ncu launch list + full captures of the main kernel.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
B="python bench.py --steps 200 --warmup 10 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep.jsonl
for cfg in "c3" "c2" "c7" "c6 --scale 20" "c2big"; do
  for v in mma cudacore; do
    timeout 300 $B --config $cfg --variant $v >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
  done
done
for cfg in "c3" "c2"; do
  for v in mma cudacore; do
    timeout 300 $B --config $cfg --dtype f16 --variant $v >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
  done
done
S="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3.csv $S > /dev/null 2>&1
for v in mma cudacore; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:dasp_main -s 3 -c 1 -o gpurun_out/prof_c3_f64_$v $S --variant $v > gpurun_out/ncu_c3_$v.log 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dasp_main -s 3 -c 1 -o gpurun_out/prof_c2_f64_mma $S --config c2 > gpurun_out/ncu_c2.log 2>&1
echo done
