#!/bin/bash
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 300 python scripts/l2_probe.py > gpurun_out/l2_probe.txt 2>&1
B="python bench.py --steps 100 --warmup 5 --e2e-steps 0 --no-cpu-baseline --config c3"
: > gpurun_out/cls.jsonl
for pr in 0 65536 262144 1048576; do
 for cls in 0 1 2 3; do
  echo "{\"panel\": $pr, \"cls\": $cls}" >> gpurun_out/cls.jsonl
  DASP_PANEL_ROWS=$pr DASP_PROFILE_CLASS=$cls timeout 300 $B >> gpurun_out/cls.jsonl 2>> gpurun_out/cls.err
 done
done
S="python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline --config c3"
for cls in 1 2 3; do
 DASP_PROFILE_CLASS=$cls timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,sm__warps_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:dasp_main -s 3 -c 1 --csv $S > gpurun_out/ncu_cls$cls.csv 2>/dev/null
 DASP_PANEL_ROWS=262144 DASP_PROFILE_CLASS=$cls timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct --clock-control none -k regex:dasp_main -s 3 -c 1 --csv $S > gpurun_out/ncu_cls${cls}_p.csv 2>/dev/null
done
echo done
