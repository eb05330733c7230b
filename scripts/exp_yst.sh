#!/bin/bash
# y store cache operator: plain / st.global.cs / st.global.cg (C3, C5: 100 MB+ of y against an L2-resident x)
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
DASP_LIB=$PWD/build/libdasp_DASP_Y_ST=1.so timeout 600 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -1
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/yst.jsonl
for cfg in "c3" "c5 --scale 0.05" "c3 --dtype f16" "c2" "c6 --scale 20"; do for lib in base "DASP_Y_ST=1" "DASP_Y_ST=2" base "DASP_Y_ST=1" "DASP_Y_ST=2"; do
  echo "# $lib" >> gpurun_out/yst.jsonl
  if [ $lib = base ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$PWD/build/libdasp_$lib.so; fi
  DASP_LIB=$L timeout 300 $B --config $cfg >> gpurun_out/yst.jsonl 2>> gpurun_out/yst.err
done; done
python scripts/show.py gpurun_out/yst.jsonl | paste - - | awk '{print $2, $3, $4, $12, $13, $14, $15, $16, $17, $18}'
echo done
