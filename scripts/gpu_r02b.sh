#!/bin/bash
# round 2: per-warp phase trace of the main kernel (C3, C2, C6), FP16 spill-free variants, long order on C5
mkdir -p gpurun_out
for c in "c3" "c2" "c6 20" "c5 0.05"; do
  DASP_LIB=build/libdasp_DASP_EXP_TRACE=1.so timeout 300 python scripts/probe/warp_trace.py $c >> gpurun_out/warp_trace.jsonl 2>> gpurun_out/warp_trace.err
done
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab2.jsonl
for lib in "" build/libdasp_DASP_NARROW_PIPE_F16=0.so build/libdasp_DASP_CHUNK_PIPE_F16=0.so "build/libdasp_DASP_NARROW_PIPE_F16=0+DASP_CHUNK_PIPE_F16=0.so"; do
  for cfg in "c3 --dtype f16" "c2 --dtype f16" "c2big --dtype f16" "c3 --dtype f16 --variant mma" "c2 --dtype f16 --variant mma"; do
    echo "# lib=$lib cfg=$cfg" >> gpurun_out/ab2.jsonl
    DASP_LIB=${lib:-paper_conf_sc_lu023_b200/libdasp.so} timeout 300 $B --config $cfg >> gpurun_out/ab2.jsonl 2>> gpurun_out/ab2.err
  done
done
for lib in "" build/libdasp_DASP_LONG_ORDER=2.so; do
  for cfg in "c5 --scale 0.05" "c5 --scale 0.05 --dtype f16" "c3 --dtype f16" "c7 --dtype f16"; do
    echo "# lib=$lib cfg=$cfg" >> gpurun_out/ab2.jsonl
    DASP_LIB=${lib:-paper_conf_sc_lu023_b200/libdasp.so} timeout 300 $B --config $cfg >> gpurun_out/ab2.jsonl 2>> gpurun_out/ab2.err
  done
done
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "narrow" > gpurun_out/pytest_narrow.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_narrow.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -v > gpurun_out/pytest_fullsize.log 2>&1; echo "fullsize rc=$?"; tail -14 gpurun_out/pytest_fullsize.log
echo done
