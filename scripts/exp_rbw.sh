#!/bin/bash
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad"
: > gpurun_out/rbw.jsonl
for cfg in "c2" "c3" "c2big"; do for dt in f64 f16; do for v in mma cudacore; do for rbw in 2 4 8; do
  echo "{\"rbw\": $rbw}" >> gpurun_out/rbw.jsonl
  timeout 300 $B --config $cfg --dtype $dt --variant $v --rbw $rbw >> gpurun_out/rbw.jsonl 2>> gpurun_out/rbw.err
done; done; done; done
echo done
