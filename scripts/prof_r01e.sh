#!/bin/bash
# r01e evidence at HEAD: launch list of the default bench command, full captures of the default
# command's main kernel (C2 FP64) and of C3's long / main kernels.
mkdir -p gpurun_out/r01e
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
S="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01e/launches_default_cmd.csv python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-triad > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dasp_main -s 3 -c 1 -o gpurun_out/r01e/prof_c2_f64_cudacore $S --config c2 > gpurun_out/r01e/ncu_c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"dasp_(main|long)_kernel" -s 6 -c 2 -o gpurun_out/r01e/prof_c3_f64_cudacore $S --config c3 > gpurun_out/r01e/ncu_c3.log 2>&1
ls -la gpurun_out/r01e
echo done
