#!/bin/bash
mkdir -p gpurun_out
: > gpurun_out/warp_trace2.jsonl
for c in "c3" "c5 0.05" "c2"; do
  DASP_LIB=build/libdasp_DASP_EXP_TRACE=1.so timeout 300 python scripts/probe/warp_trace.py $c >> gpurun_out/warp_trace2.jsonl 2>> gpurun_out/warp_trace2.err
done
echo done
