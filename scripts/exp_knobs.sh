#!/bin/bash
# Medium/short knobs: small-pair row-blocks, chunk software pipeline, short tiles per warp.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
EV="DASP_SMALL_PAIR=0 DASP_CHUNK_PIPE=0 DASP_SHORT_TPW=1 DASP_SMALL_PAIR=0,DASP_CHUNK_PIPE=0,DASP_SHORT_TPW=1"
make exp EXPVARS="$EV" -j8 >> gpurun_out/make.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph"
: > gpurun_out/knobs.jsonl
run() { echo "# lib $1" >> gpurun_out/knobs.jsonl; DASP_LIB=$2 timeout 300 $B ${@:3} >> gpurun_out/knobs.jsonl 2>> gpurun_out/knobs.err; }
for cfg in "c2" "c3" "c2big" "c5 --scale 0.05" "c6 --scale 20"; do for dt in f64 f16 f32; do
  run base paper_conf_sc_lu023_b200/libdasp.so --config $cfg --dtype $dt
  for v in DASP_SMALL_PAIR=0 DASP_CHUNK_PIPE=0 DASP_SHORT_TPW=1 DASP_SMALL_PAIR=0+DASP_CHUNK_PIPE=0+DASP_SHORT_TPW=1; do
    run $v build/libdasp_$v.so --config $cfg --dtype $dt
  done
done; done
echo done
