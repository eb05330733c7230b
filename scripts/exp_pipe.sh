#!/bin/bash
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
DASP_PIPE=1 timeout 600 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_pipe.log 2>&1; echo "pytest pipe rc=$?"; tail -15 gpurun_out/pytest_pipe.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/pipe.jsonl
for pipe in 0 1; do
for cfg in "c2" "c3" "c7" "c6 --scale 20"; do for dt in f64 f16; do for v in mma cudacore; do
  echo "{\"pipe\": $pipe}" >> gpurun_out/pipe.jsonl
  DASP_PIPE=$pipe timeout 300 $B --config $cfg --dtype $dt --variant $v >> gpurun_out/pipe.jsonl 2>> gpurun_out/pipe.err
done; done; done; done
echo done
