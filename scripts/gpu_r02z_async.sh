#!/bin/bash
# A/B: register-free short-tile gathers (cp.async 8-byte copies into shared memory), TPW 2 / 3
mkdir -p gpurun_out
O=gpurun_out/async.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
A2="build/libdasp_DASP_SHORT_ASYNC_F64=1.so"
A3="build/libdasp_DASP_SHORT_ASYNC_F64=1+DASP_SHORT_TPW_F64=3.so"
for lib in $A2 $A3; do DASP_LIB=$lib timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "f64 and not x_stage" > gpurun_out/async_pytest.log 2>&1; echo "pytest $lib rc=$?"; tail -1 gpurun_out/async_pytest.log; done
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/async.err; }
for cfg in "c3" "c6 --scale 20" "c5 --scale 0.05" "c2"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "$A2" "$A3"; do run "$lib" "$cfg"; done
done
echo done
