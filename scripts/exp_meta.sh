#!/bin/bash
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad"
: > gpurun_out/meta.jsonl
for cfg in "c2" "c3" "c7"; do for dt in f64 f16; do for v in mma cudacore; do
  echo "{\"rbw\": 0}" >> gpurun_out/meta.jsonl
  timeout 300 $B --config $cfg --dtype $dt --variant $v >> gpurun_out/meta.jsonl 2>> gpurun_out/meta.err
done; done; done
for rbw in 2 8 16; do for dt in f64 f16; do
  echo "{\"rbw\": $rbw}" >> gpurun_out/meta.jsonl
  timeout 300 $B --config c2 --dtype $dt --variant cudacore --rbw $rbw >> gpurun_out/meta.jsonl 2>> gpurun_out/meta.err
done; done
timeout 300 python bench.py --steps 1000 --e2e-steps 3 --no-cpu-baseline > gpurun_out/bench_triad.log 2>&1
echo done
