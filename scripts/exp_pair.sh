#!/bin/bash
# Two row-blocks in flight per warp (DASP_PAIR_*) vs one; occupancy cap 4 or 3 blocks/SM.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
EV="DASP_PAIR_F16=2 DASP_PAIR_F16=2,DASP_MIN_BLOCKS_F16=3 DASP_PAIR_F32=2 DASP_PAIR_F32=2,DASP_MIN_BLOCKS_F32=3 DASP_PAIR_F64=2 DASP_PAIR_F64=2,DASP_MIN_BLOCKS=3"
make exp EXPVARS="$EV" -j8 >> gpurun_out/make.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "integer or random" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build"
: > gpurun_out/pair.jsonl
run() { echo "{\"lib\": \"$1\"}" >> gpurun_out/pair.jsonl; DASP_LIB=$2 timeout 300 $B ${@:3} >> gpurun_out/pair.jsonl 2>> gpurun_out/pair.err; }
for cfg in c2 c3 c2big; do
 for dt in f64 f16 f32; do run base paper_conf_sc_lu023_b200/libdasp.so --config $cfg --dtype $dt; done
 run F16=2 build/libdasp_DASP_PAIR_F16=2.so --config $cfg --dtype f16
 run F16=2,mb3 build/libdasp_DASP_PAIR_F16=2,DASP_MIN_BLOCKS_F16=3.so --config $cfg --dtype f16
 run F32=2 build/libdasp_DASP_PAIR_F32=2.so --config $cfg --dtype f32
 run F32=2,mb3 build/libdasp_DASP_PAIR_F32=2,DASP_MIN_BLOCKS_F32=3.so --config $cfg --dtype f32
 run F64=2 build/libdasp_DASP_PAIR_F64=2.so --config $cfg --dtype f64
 run F64=2,mb3 build/libdasp_DASP_PAIR_F64=2,DASP_MIN_BLOCKS=3.so --config $cfg --dtype f64
done
echo done
