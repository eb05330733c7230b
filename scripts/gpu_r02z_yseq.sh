#!/bin/bash
# probe: cost of the short class's output map + scattered y stores (outputs to consecutive y slots)
mkdir -p gpurun_out
O=gpurun_out/yseq.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/yseq.err; }
for cfg in "c3" "c6 --scale 20" "c3 --dtype f16"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so build/libdasp_DASP_EXP_SHORT_YSEQ=1.so build/libdasp_DASP_CLASS_MASK=5.so "build/libdasp_DASP_EXP_SHORT_YSEQ=1+DASP_CLASS_MASK=5.so"; do run "$lib" "$cfg"; done
done
echo done
