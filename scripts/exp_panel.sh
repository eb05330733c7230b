#!/bin/bash
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
#timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_gpu.log
B="python bench.py --steps 100 --warmup 5 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/panel.jsonl
for cfg in "c3" "c2"; do
 for pr in -1 262144 1048576 2097152; do
  for v in mma cudacore; do
   echo "{\"panel\": $pr}" >> gpurun_out/panel.jsonl
   DASP_PANEL_ROWS=$pr timeout 300 $B --config $cfg --variant $v >> gpurun_out/panel.jsonl 2>> gpurun_out/panel.err
  done
 done
done
for cls in 1 2 3; do
  echo "{\"panel\": 0, \"cls\": $cls}" >> gpurun_out/panel.jsonl
  DASP_PROFILE_CLASS=$cls timeout 300 $B --config c3 >> gpurun_out/panel.jsonl 2>> gpurun_out/panel.err
done
S="python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline --config c3"
for cls in 1 2 3; do
 DASP_PROFILE_CLASS=$cls timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:dasp_main -s 3 -c 1 --csv $S > gpurun_out/ncu_pcls$cls.csv 2>/dev/null
done
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:dasp_main -s 3 -c 1 --csv $S > gpurun_out/ncu_pall.csv 2>/dev/null
echo done
