#!/bin/bash
# A/B: L1-allocating irregular-tail loads on the narrow / mid path (lane = row: instructions revisit lines)
mkdir -p gpurun_out
O=gpurun_out/irrl1.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
L1="build/libdasp_DASP_NARROW_IRR_L1=1.so"
DASP_LIB=$L1 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "not x_stage" > gpurun_out/irrl1_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/irrl1_pytest.log
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/irrl1.err; }
for rep in 1 2; do
for cfg in "c3" "c3 --dtype f16" "c3 --dtype f32" "c5 --scale 0.05" "c2 --dtype f16" "c2big --dtype f16"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "$L1"; do run "$lib" "$cfg"; done
done
done
echo done
