#!/bin/bash
# Why does the 162^3 stencil reach a lower HBM fraction than 128^3?  panel / rbw sweep + DRAM bytes.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-compare --no-gpu-build"
: > gpurun_out/c2big.jsonl
for cfg in c2 c2big; do
 for pr in -1 262144 524288 1048576 2097152 4194304; do
   echo "{\"panel\": $pr, \"cfg\": \"$cfg\"}" >> gpurun_out/c2big.jsonl
   DASP_PANEL_ROWS=$pr timeout 300 $B --config $cfg >> gpurun_out/c2big.jsonl 2>> gpurun_out/c2big.err
 done
 for r in 1 2 8 16; do
   echo "{\"rbw\": $r, \"cfg\": \"$cfg\"}" >> gpurun_out/c2big.jsonl
   timeout 300 $B --config $cfg --rbw $r --no-triad >> gpurun_out/c2big.jsonl 2>> gpurun_out/c2big.err
 done
done
S="python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare --no-gpu-build"
for cfg in c2 c2big; do
 timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,sm__warps_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:dasp_main -s 3 -c 1 --csv $S --config $cfg > gpurun_out/ncu_$cfg.csv 2>/dev/null
done
echo done
