#!/bin/bash
# L2 fetch granularity hint (cudaLimitMaxL2FetchGranularity) on the gather-heavy configs
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/l2fetch.jsonl
run() { echo "# $1 $2" >> gpurun_out/l2fetch.jsonl; env $1 timeout 300 $B $2 >> gpurun_out/l2fetch.jsonl 2>> gpurun_out/l2fetch.err; }
for cfg in "--config c3" "--config c3 --dtype f16" "--config c6 --scale 20" "--config c2" "--config c7" "--config c5 --scale 0.05"; do
  for m in A=1 DASP_L2_FETCH=32 DASP_L2_FETCH=64 DASP_L2_FETCH=128; do run $m "$cfg"; done
done
python scripts/show.py gpurun_out/l2fetch.jsonl
grep "granularity" gpurun_out/l2fetch.err | sort | uniq -c
echo done
