#!/bin/bash
# main-kernel class split (build knob DASP_CLASS_MASK: 1 finish warps only, 3 + medium, 5 + short)
# and the no-x probe per class (DASP_EXP_NOX: every gather from a cache-resident window; wrong y)
mkdir -p gpurun_out
O=gpurun_out/classes.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
for cfg in "c3" "c3 --dtype f16" "c5 --scale 0.05"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so build/libdasp_DASP_CLASS_MASK=1.so build/libdasp_DASP_CLASS_MASK=3.so build/libdasp_DASP_CLASS_MASK=5.so build/libdasp_DASP_EXP_NOX=1.so "build/libdasp_DASP_CLASS_MASK=3+DASP_EXP_NOX=1.so" "build/libdasp_DASP_CLASS_MASK=5+DASP_EXP_NOX=1.so"; do
    echo "# lib=$lib cfg=$cfg" >> $O; DASP_LIB=$lib timeout 300 $B --config $cfg >> $O 2>> gpurun_out/classes.err
  done
done
echo done
