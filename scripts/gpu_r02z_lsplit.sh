#!/bin/bash
# A/B: long units, lane holds elements l and l+32 of each group
mkdir -p gpurun_out
O=gpurun_out/lsplit.jsonl
: > $O
L="build/libdasp_DASP_LONG_SPLIT=1.so"
DASP_LIB=$L timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fuzz.py -q -x -k "not x_stage and not device_builder and (f64 or f32)"  > gpurun_out/lsplit_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/lsplit_pytest.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/lsplit.err; }
for rep in 1 2; do
for cfg in "c3" "c7" "c5 --scale 0.05" "c3 --dtype f32"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "$L"; do run "$lib" "$cfg"; done
done; done
echo done
