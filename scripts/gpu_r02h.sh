#!/bin/bash
# round 2: the main kernel without the chunk-unit code (C2 regression check), heavy-first 0 / 4 / 16
mkdir -p gpurun_out
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab6.jsonl
for cfg in "c2" "c2big" "c3" "c3 --dtype f16" "c5 --scale 0.05" "c2 --dtype f32" "c6 --scale 20"; do
  for lib in "" build/libdasp_DASP_HEAVY_FIRST=0.so build/libdasp_DASP_HEAVY_FIRST=16.so; do
    echo "# lib=$lib cfg=$cfg" >> gpurun_out/ab6.jsonl
    DASP_LIB=${lib:-paper_conf_sc_lu023_b200/libdasp.so} timeout 300 $B --config $cfg >> gpurun_out/ab6.jsonl 2>> gpurun_out/ab6.err
  done
done
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_builder.py -m gpu -q -x > gpurun_out/pytest_h.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_h.log
echo done
