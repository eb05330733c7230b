#!/bin/bash
# A/B: FP64 main kernel at 3 blocks / 80 registers (24 warps per SM) with more work in flight per warp
mkdir -p gpurun_out
O=gpurun_out/mb3.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
L1="build/libdasp_DASP_MIN_BLOCKS=3.so"
L2="build/libdasp_DASP_MIN_BLOCKS=3+DASP_SHORT_TPW_F64=3+DASP_NARROW_PIPE_F64=1+DASP_PEEL_U2_F64=1.so"
L3="build/libdasp_DASP_PEEL_U2_F64=1.so"
DASP_LIB=$L2 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "f64 and not x_stage" > gpurun_out/mb3_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/mb3_pytest.log
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/mb3.err; }
for cfg in "c3" "c5 --scale 0.05" "c2" "c2big" "c6 --scale 20"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "$L1" "$L2" "$L3"; do run "$lib" "$cfg"; done
done
echo done
