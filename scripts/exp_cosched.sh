#!/bin/bash
# Co-scheduled long units (one launch) vs the separate long kernel: parity, then A/B timings.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "co_schedule" > gpurun_out/pytest_cosched.log 2>&1; echo "pytest cosched rc=$?"; tail -3 gpurun_out/pytest_cosched.log
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph"
: > gpurun_out/cosched.jsonl
for cfg in "c3" "c5 --scale 0.05" "c7" "c1b" "c2"; do for dt in f64 f16 f32; do for cs in 0 1; do
  timeout 300 $B --config $cfg --dtype $dt --co-schedule $cs >> gpurun_out/cosched.jsonl 2>> gpurun_out/cosched.err
done; done; done
S="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare --no-gpu-build --no-graph"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dasp_main -s 3 -c 1 -o gpurun_out/prof_c3_cosched $S --config c3 > /dev/null 2>&1
ncu -i gpurun_out/prof_c3_cosched.ncu-rep --page raw --csv > gpurun_out/prof_c3_cosched.raw.csv 2>/dev/null
ncu -i gpurun_out/prof_c3_cosched.ncu-rep --page source --csv > gpurun_out/prof_c3_cosched.source.csv 2>/dev/null
echo done
