#!/bin/bash
mkdir -p gpurun_out
O=gpurun_out/tpw3.jsonl
: > $O
L="build/libdasp_DASP_SHORT_TPW_OCC5=3.so"
DASP_LIB=$L timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fuzz.py -q -x -k "f16 and not device_builder" > gpurun_out/tpw3_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/tpw3_pytest.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/tpw3.err; }
for rep in 1 2; do
for cfg in "c3 --dtype f16" "c6 --scale 20 --dtype f16" "c2 --dtype f16"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "$L"; do run "$lib" "$cfg"; done
done; done
echo done
