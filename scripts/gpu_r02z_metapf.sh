#!/bin/bash
# A/B: next-row-block / next-pass metadata prefetch in the wide and narrow medium paths
mkdir -p gpurun_out
O=gpurun_out/metapf.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
NP="build/libdasp_DASP_NARROW_META_PF_F64=1+DASP_NARROW_META_PF_F32=1.so"
WP="build/libdasp_DASP_WIDE_META_PF_F64=1+DASP_WIDE_META_PF_F32=1+DASP_WIDE_META_PF_F16=1.so"
BP="build/libdasp_DASP_WIDE_META_PF_F64=1+DASP_NARROW_META_PF_F64=1+DASP_WIDE_META_PF_F32=1+DASP_NARROW_META_PF_F32=1.so"
NP16="build/libdasp_DASP_NARROW_META_PF_F16=1.so"
DASP_LIB=$BP timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "not x_stage" > gpurun_out/metapf_pytest.log 2>&1; echo "pytest BP rc=$?"; tail -1 gpurun_out/metapf_pytest.log
DASP_LIB=$WP timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "f16 and not x_stage" >> gpurun_out/metapf_pytest.log 2>&1; echo "pytest WP f16 rc=$?"; tail -1 gpurun_out/metapf_pytest.log
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/metapf.err; }
for cfg in "c3" "c5 --scale 0.05" "c2" "c2big" "c3 --dtype f32" "c6 --scale 20"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "$NP" "$WP" "$BP"; do run "$lib" "$cfg"; done
done
for cfg in "c3 --dtype f16" "c5 --scale 0.05 --dtype f16" "c2 --dtype f16" "c2big --dtype f16"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "$WP" "$NP16"; do run "$lib" "$cfg"; done
done
echo done
