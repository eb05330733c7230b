#!/bin/bash
# cp.async double-buffered medium row-blocks (DASP_MED_ASYNC=1) vs the register path.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
make exp EXPVARS="DASP_MED_ASYNC=1" -j8 >> gpurun_out/make.log 2>&1
L=build/libdasp_DASP_MED_ASYNC=1.so
DASP_LIB=$L timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x > gpurun_out/pytest_async.log 2>&1; echo "pytest async rc=$?"; tail -2 gpurun_out/pytest_async.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare"
: > gpurun_out/async.jsonl
run() { echo "{\"tag\": \"$1\"}" >> gpurun_out/async.jsonl; timeout 300 env ${@:2} >> gpurun_out/async.jsonl 2>> gpurun_out/async.err; }
for cfg in c2 c2big c3 "c5 --scale 0.05"; do
 for dt in f64 f16 f32; do
  run base DASP_LIB=paper_conf_sc_lu023_b200/libdasp.so $B --config $cfg --dtype $dt
  run async DASP_LIB=$L $B --config $cfg --dtype $dt
 done
done
run base-mma DASP_LIB=paper_conf_sc_lu023_b200/libdasp.so $B --config c2 --variant mma
run async-mma DASP_LIB=$L $B --config c2 --variant mma
for r in 2 4 16; do
 run async-rbw$r DASP_LIB=$L $B --config c2 --dtype f16 --rbw $r
 run async-rbw$r DASP_LIB=$L $B --config c2 --dtype f64 --rbw $r
done
echo done
