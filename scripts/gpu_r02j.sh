#!/bin/bash
# round 2: how much do x gathers cost on the stencils (no-x probe) and how many L2 requests do they make
mkdir -p gpurun_out
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab8.jsonl
for cfg in "c2" "c2 --dtype f16" "c2 --dtype f32" "c2big" "c2big --dtype f16" "c3" "c3 --dtype f16" "c5 --scale 0.05"; do
  for lib in "" build/libdasp_DASP_EXP_NOX=1.so; do
    echo "# lib=$lib cfg=$cfg" >> gpurun_out/ab8.jsonl
    DASP_LIB=${lib:-paper_conf_sc_lu023_b200/libdasp.so} timeout 300 $B --config $cfg >> gpurun_out/ab8.jsonl 2>> gpurun_out/ab8.err
  done
done
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_requests_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum,l1tex__t_sector_hit_rate.pct,lts__throughput.avg.pct_of_peak_sustained_elapsed
S="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare --no-gpu-build --no-graph --no-sub"
for cfg in "c2" "c2 --dtype f16" "c2 --dtype f32" "c5 --scale 0.05"; do
  echo "# $cfg" >> gpurun_out/ncu_stencil.csv
  timeout 600 ncu --metrics $M --clock-control none -k regex:dasp_ -s 4 -c 2 --csv $S --config $cfg >> gpurun_out/ncu_stencil.csv 2>> gpurun_out/ncu_stencil.err
done
echo done
