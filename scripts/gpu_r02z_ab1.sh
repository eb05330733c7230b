#!/bin/bash
# A/B: CUDA-core wide medium path -- ragged chunk first (RF) and two chunks per round trip (U2)
mkdir -p gpurun_out
O=gpurun_out/ab_rf_u2.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
ALL=build/libdasp_DASP_RAGGED_FIRST_F64=1+DASP_RAGGED_FIRST_F32=1+DASP_RAGGED_FIRST_F16=1+DASP_CHUNK_U2_F64=1+DASP_CHUNK_U2_F32=1+DASP_CHUNK_U2_F16=1.so
DASP_LIB=$ALL timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q > gpurun_out/ab_rf_u2_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/ab_rf_u2_pytest.log
run() { # lib cfg
  echo "# lib=$1 cfg=$2" >> $O
  DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/ab_rf_u2.err
}
for rep in 1 2; do
for cfg in "c3" "c5 --scale 0.05" "c2" "c2big" "c3 --dtype f32" "c2 --dtype f32"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "build/libdasp_DASP_RAGGED_FIRST_F64=1+DASP_RAGGED_FIRST_F32=1.so" "build/libdasp_DASP_CHUNK_U2_F64=1+DASP_CHUNK_U2_F32=1+DASP_RAGGED_FIRST_F64=1+DASP_RAGGED_FIRST_F32=1.so"; do
    run "$lib" "$cfg"
  done
done
for cfg in "c3 --dtype f16" "c5 --scale 0.05 --dtype f16" "c2 --dtype f16"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "build/libdasp_DASP_RAGGED_FIRST_F16=1.so" "build/libdasp_DASP_RAGGED_FIRST_F16=1+DASP_CHUNK_U2_F16=1.so"; do
    run "$lib" "$cfg"
  done
done
done
echo done
