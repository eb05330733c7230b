#!/bin/bash
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "integer or random" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 400 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build"
: > gpurun_out/wmeta.jsonl
for cfg in c2 c3 c2big; do for dt in f64 f16 f32; do
  timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/wmeta.jsonl 2>> gpurun_out/wmeta.err
done; done
echo done
