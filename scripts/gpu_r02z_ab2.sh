#!/bin/bash
# A/B: CUDA-core wide medium path -- PEEL (chunk 0 + ragged + first irregular gathered in one round)
# vs RAGGED_FIRST (FP16) vs base
mkdir -p gpurun_out
O=gpurun_out/ab_peel.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
PEEL="build/libdasp_DASP_PEEL_F64=1+DASP_PEEL_F32=1+DASP_PEEL_F16=1.so"
RF16="build/libdasp_DASP_RAGGED_FIRST_F16=1.so"
DASP_LIB=$PEEL timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q > gpurun_out/ab_peel_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/ab_peel_pytest.log
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/ab_peel.err; }
for cfg in "c3" "c5 --scale 0.05" "c2" "c2big" "c3 --dtype f32" "c2 --dtype f32" "c1a" "c6 --scale 20"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "$PEEL"; do run "$lib" "$cfg"; done
done
for cfg in "c3 --dtype f16" "c5 --scale 0.05 --dtype f16" "c2 --dtype f16" "c2big --dtype f16"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "$PEEL" "$RF16"; do run "$lib" "$cfg"; done
done
echo done
