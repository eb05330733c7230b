#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -x > gpurun_out/pytest_s.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_s.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab17.jsonl
for cfg in "c3" "c3 --panel-rows 8192" "c3 --panel-rows 32768" "c3 --dtype f16" "c5 --scale 0.05" "c5 --scale 0.05 --dtype f16" "c2" "c2 --dtype f16" "c6 --scale 20" "c3 --dtype f32" "c3 --dtype f32 --panel-rows 8192"; do
  for lib in "" build/libdasp_DASP_PACK_WARPS=0.so; do
    echo "# lib=$lib cfg=$cfg" >> gpurun_out/ab17.jsonl
    DASP_LIB=${lib:-paper_conf_sc_lu023_b200/libdasp.so} timeout 300 $B --config $cfg >> gpurun_out/ab17.jsonl 2>> gpurun_out/ab17.err
  done
done
echo done
