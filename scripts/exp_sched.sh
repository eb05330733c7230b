#!/bin/bash
# Dynamic (persistent, atomic work counter) main-kernel schedule vs the static grid; plus the
# two-row-blocks-in-flight builds at 3 blocks/SM.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
EV="DASP_PAIR_F16=2,DASP_MIN_BLOCKS_F16=3 DASP_PAIR_F32=2,DASP_MIN_BLOCKS_F32=3 DASP_PAIR_F64=2,DASP_MIN_BLOCKS=3"
make exp EXPVARS="$EV" -j8 >> gpurun_out/make.log 2>&1
DASP_SCHED=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_solvers.py -m gpu -q -x > gpurun_out/pytest_sched.log 2>&1; echo "pytest dyn rc=$?"; tail -2 gpurun_out/pytest_sched.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare"
: > gpurun_out/sched.jsonl
run() { echo "{\"tag\": \"$1\"}" >> gpurun_out/sched.jsonl; timeout 300 env ${@:2} >> gpurun_out/sched.jsonl 2>> gpurun_out/sched.err; }
for cfg in c2 c3 c2big "c6 --scale 20" "c5 --scale 0.05"; do
 for dt in f64 f16 f32; do
  run static DASP_SCHED=0 $B --config $cfg --dtype $dt
  run dyn DASP_SCHED=1 $B --config $cfg --dtype $dt
  run dyn-rbw4 DASP_SCHED=1 $B --config $cfg --dtype $dt --rbw 4
 done
done
for cfg in c2 c3; do
 run pairF16mb3 DASP_LIB=build/libdasp_DASP_PAIR_F16=2+DASP_MIN_BLOCKS_F16=3.so $B --config $cfg --dtype f16
 run pairF32mb3 DASP_LIB=build/libdasp_DASP_PAIR_F32=2+DASP_MIN_BLOCKS_F32=3.so $B --config $cfg --dtype f32
 run pairF64mb3 DASP_LIB=build/libdasp_DASP_PAIR_F64=2+DASP_MIN_BLOCKS=3.so $B --config $cfg --dtype f64
done
echo done
