#!/bin/bash
# LOOP_NUM for the stencils (--rbw), FP64 short tiles per warp 3, FP16 stencil on the wide path
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/misc.jsonl
for cfg in c2 c2big; do for r in 8 6 10 12 8; do echo "# rbw $r" >> gpurun_out/misc.jsonl; timeout 300 $B --config $cfg --rbw $r >> gpurun_out/misc.jsonl 2>> gpurun_out/misc.err; done; done
for cfg in "c3" "c6 --scale 20" "c5 --scale 0.05"; do for lib in base "DASP_SHORT_TPW_F64=3" base "DASP_SHORT_TPW_F64=3"; do
  echo "# $lib" >> gpurun_out/misc.jsonl
  if [ $lib = base ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$PWD/build/libdasp_$lib.so; fi
  DASP_LIB=$L timeout 300 $B --config $cfg >> gpurun_out/misc.jsonl 2>> gpurun_out/misc.err
done; done
for cfg in c2 c2big; do for m in 1 0 1 0; do echo "# mid $m" >> gpurun_out/misc.jsonl; DASP_NARROW_MID=$m timeout 300 $B --config $cfg --dtype f16 >> gpurun_out/misc.jsonl 2>> gpurun_out/misc.err; done; done
python scripts/show.py gpurun_out/misc.jsonl | paste - - | awk '{print $2, $3, $4, $6, $14, $15, $16, $17, $18, $19}'
echo done
