#!/bin/bash
# A/B: FP16 mid (two lanes per row) class upper bound 4K (default) / 3K / 2K slots: stencil rows of 27
# slots go to the wide warp-per-row-block path at 3K / 2K
mkdir -p gpurun_out
O=gpurun_out/mid16.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
M2="build/libdasp_DASP_MID_MUL_F16=2.so"; M3="build/libdasp_DASP_MID_MUL_F16=3.so"
DASP_LIB=$M3 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "f16 and not x_stage" > gpurun_out/mid16_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/mid16_pytest.log
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/mid16.err; }
for cfg in "c2 --dtype f16" "c2big --dtype f16" "c3 --dtype f16" "c5 --scale 0.05 --dtype f16"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "$M3" "$M2"; do run "$lib" "$cfg"; done
done
echo done
