#!/bin/bash
# A/B: persistent long kernel (fixed grid, warps striding over the unit schedule)
mkdir -p gpurun_out
O=gpurun_out/persist.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
L8="build/libdasp_DASP_LONG_PERSIST=8.so"; L16="build/libdasp_DASP_LONG_PERSIST=16.so"; L6="build/libdasp_DASP_LONG_PERSIST=6+DASP_LONG_MIN_BLOCKS=6.so"
DASP_LIB=$L8 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "huge or c3s or lens" > gpurun_out/persist_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/persist_pytest.log
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/persist.err; }
for cfg in "c3" "c7" "c5 --scale 0.05" "c3 --dtype f16"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "$L8" "$L16" "$L6"; do run "$lib" "$cfg"; done
done
echo done
