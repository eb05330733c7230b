#!/bin/bash
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
S="python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dasp_main -s 3 -c 1 -o gpurun_out/prof_c7 $S --config c7 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dasp_main -s 3 -c 1 -o gpurun_out/prof_c3b $S --config c3 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dasp_main -s 3 -c 1 -o gpurun_out/prof_c2f16 $S --config c2 --dtype f16 --variant cudacore > /dev/null 2>&1
echo done
