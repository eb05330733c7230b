#!/bin/bash
# Per-dtype medium/short knob combinations for FP64 and FP32 (FP16 keeps SP1/CP1/TPW2).
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
L1=DASP_SMALL_PAIR_F64=0,DASP_SMALL_PAIR_F32=0,DASP_CHUNK_PIPE_F32=0
L2=DASP_SMALL_PAIR_F64=0,DASP_SHORT_TPW_F64=1,DASP_SMALL_PAIR_F32=0,DASP_CHUNK_PIPE_F32=0,DASP_SHORT_TPW_F32=1
L3=DASP_CHUNK_PIPE_F32=0
make exp EXPVARS="$L1 $L2 $L3" -j8 >> gpurun_out/make.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph"
: > gpurun_out/knobs2.jsonl
run() { echo "# lib $1" >> gpurun_out/knobs2.jsonl; DASP_LIB=$2 timeout 300 $B ${@:3} >> gpurun_out/knobs2.jsonl 2>> gpurun_out/knobs2.err; }
for cfg in "c2" "c3" "c2big" "c5 --scale 0.05" "c6 --scale 20"; do for dt in f64 f32; do
  run base paper_conf_sc_lu023_b200/libdasp.so --config $cfg --dtype $dt
  for v in $L1 $L2 $L3; do
    t=$(echo $v | tr , +)
    run $t build/libdasp_$t.so --config $cfg --dtype $dt
  done
done; done
echo done
