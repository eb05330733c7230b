#!/bin/bash
# round 2: main kernel at 5 / 6 blocks per SM (48 / 40 registers, spills) vs 4 (64, no spills)
mkdir -p gpurun_out
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab9.jsonl
for cfg in "c3" "c3 --dtype f16" "c5 --scale 0.05" "c2" "c2big" "c6 --scale 20" "c2 --dtype f16"; do
  for lib in "" "build/libdasp_DASP_MIN_BLOCKS=5+DASP_MIN_BLOCKS_F16=5.so" "build/libdasp_DASP_MIN_BLOCKS=6+DASP_MIN_BLOCKS_F16=6.so"; do
    echo "# lib=$lib cfg=$cfg" >> gpurun_out/ab9.jsonl
    DASP_LIB=${lib:-paper_conf_sc_lu023_b200/libdasp.so} timeout 300 $B --config $cfg >> gpurun_out/ab9.jsonl 2>> gpurun_out/ab9.err
  done
done
cd scripts/probe && timeout 1200 python hot_relabel.py c5 0.05 4096,65536,262144,1000000 > ../../gpurun_out/hot_relabel_c5.jsonl 2> ../../gpurun_out/hot_relabel_c5.err; cd ../..
echo done
