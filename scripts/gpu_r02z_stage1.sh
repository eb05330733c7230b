#!/bin/bash
# x-window staging (TMA bulk copies into shared memory) first measurement + parity; PEEL FP64 /
# RAGGED_FIRST FP16 defaults
mkdir -p gpurun_out
O=gpurun_out/stage1.jsonl
: > $O
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "x_stage" > gpurun_out/stage1_pytest_stage.log 2>&1; echo "stage tests rc=$?"; tail -3 gpurun_out/stage1_pytest_stage.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/stage1_pytest_all.log 2>&1; echo "all gpu tests rc=$?"; tail -3 gpurun_out/stage1_pytest_all.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
for rep in 1 2; do
for cfg in "c2" "c2big" "c2 --dtype f32" "c2big --dtype f32"; do
  for xs in 1 0; do echo "# x_stage=$xs cfg=$cfg" >> $O; timeout 300 $B --config $cfg --x-stage $xs >> $O 2>> gpurun_out/stage1.err; done
done
done
for cfg in "c3" "c3 --dtype f16" "c5 --scale 0.05"; do echo "# cfg=$cfg" >> $O; timeout 300 $B --config $cfg >> $O 2>> gpurun_out/stage1.err; done
echo done
