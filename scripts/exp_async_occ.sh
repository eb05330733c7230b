#!/bin/bash
# Occupancy of the cp.async medium build (did the shared-memory carveout take?), then C5 at full size.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
make exp EXPVARS="DASP_MED_ASYNC=1" -j8 >> gpurun_out/make.log 2>&1
S="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare --no-gpu-build"
M=launch__occupancy_limit_shared_mem,launch__occupancy_limit_registers,launch__shared_mem_config_size,sm__warps_active.avg.pct_of_peak_sustained_active,gpu__time_duration.sum
DASP_LIB=build/libdasp_DASP_MED_ASYNC=1.so timeout 600 ncu --metrics $M --clock-control none -k regex:dasp_main -s 3 -c 1 --csv $S > gpurun_out/ncu_async_occ.csv 2>/dev/null
timeout 600 ncu --metrics $M --clock-control none -k regex:dasp_main -s 3 -c 1 --csv $S > gpurun_out/ncu_base_occ.csv 2>/dev/null
bash scripts/c5_full.sh
