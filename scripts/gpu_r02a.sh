#!/bin/bash
# round 2, first check after the cleanup: GPU suite, new default bench line, C3 x-traffic probes
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab.jsonl
for lib in "" build/libdasp_DASP_EXP_NOX=1.so build/libdasp_DASP_LONG_ORDER=2.so "build/libdasp_DASP_LONG_ORDER=2+DASP_COL_BUCKETS=64.so" build/libdasp_DASP_LONG_ORDER=0.so build/libdasp_DASP_COL_BUCKETS=64.so; do
  for cfg in "c3" "c7"; do
    echo "# lib=$lib cfg=$cfg" >> gpurun_out/ab.jsonl
    DASP_LIB=${lib:-paper_conf_sc_lu023_b200/libdasp.so} timeout 300 $B --config $cfg >> gpurun_out/ab.jsonl 2>> gpurun_out/ab.err
  done
done
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum,dram__sectors_read.sum,lts__t_sector_hit_rate.pct,l1tex__t_sectors_pipe_lu_mem_global_op_ld.sum,l1tex__t_sector_hit_rate.pct
S="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare --no-gpu-build --no-graph --no-sub"
timeout 600 ncu --metrics $M --clock-control none -k regex:dasp_ -s 4 -c 2 --csv $S --config c3 > gpurun_out/ncu_c3_mem.csv 2> gpurun_out/ncu_c3_mem.err
DASP_LIB=build/libdasp_DASP_EXP_NOX=1.so timeout 600 ncu --metrics $M --clock-control none -k regex:dasp_ -s 4 -c 2 --csv $S --config c3 > gpurun_out/ncu_c3_mem_nox.csv 2>> gpurun_out/ncu_c3_mem.err
DASP_LIB=build/libdasp_DASP_LONG_ORDER=2.so timeout 600 ncu --metrics $M --clock-control none -k regex:dasp_ -s 4 -c 2 --csv $S --config c3 > gpurun_out/ncu_c3_mem_glob.csv 2>> gpurun_out/ncu_c3_mem.err
timeout 900 python bench.py > gpurun_out/bench.jsonl 2> gpurun_out/bench.err; echo "bench rc=$?"; tail -c 600 gpurun_out/bench.err
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -15 gpurun_out/pytest_gpu.log
echo done
