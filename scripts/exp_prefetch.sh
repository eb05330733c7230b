#!/bin/bash
# L2 prefetch of the next medium row-block (DASP_MED_PREFETCH) on vs off.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
make exp EXPVARS="DASP_MED_PREFETCH=0 ${EXTRA_EV}" -j8 >> gpurun_out/make.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph"
: > gpurun_out/prefetch.jsonl
run() { echo "# lib $1" >> gpurun_out/prefetch.jsonl; DASP_LIB=$2 timeout 300 $B ${@:3} >> gpurun_out/prefetch.jsonl 2>> gpurun_out/prefetch.err; }
for cfg in "c2" "c2big" "c3" "c5 --scale 0.05"; do for dt in f64 f32 f16; do
  run base paper_conf_sc_lu023_b200/libdasp.so --config $cfg --dtype $dt
  for v in DASP_MED_PREFETCH=0 ${EXTRA_EV}; do t=$(echo $v | tr , +); run $t build/libdasp_$t.so --config $cfg --dtype $dt; done
done; done
echo done
