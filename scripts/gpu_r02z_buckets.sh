#!/bin/bash
# long-unit schedule: column buckets 4 / 16 (default) / 64 / 256 / 2048
mkdir -p gpurun_out
O=gpurun_out/buckets.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
for cfg in "c3" "c3 --dtype f16" "c5 --scale 0.05" "c7"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so build/libdasp_DASP_COL_BUCKETS=4.so build/libdasp_DASP_COL_BUCKETS=64.so build/libdasp_DASP_COL_BUCKETS=256.so build/libdasp_DASP_COL_BUCKETS=2048.so; do
    echo "# lib=$lib cfg=$cfg" >> $O; DASP_LIB=$lib timeout 300 $B --config $cfg >> $O 2>> gpurun_out/buckets.err
  done
done
echo done
