#!/bin/bash
# A/B: PEEL + software-pipelined chunk loop (chunk ch+1 streams with chunk ch gathers)
mkdir -p gpurun_out
O=gpurun_out/pipe.jsonl
: > $O
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
P2="build/libdasp_DASP_PEEL_PIPE_F64=2.so"
P2N="build/libdasp_DASP_PEEL_PIPE_F64=2+DASP_WIDE_META_PF_F64=0.so"
P1N="build/libdasp_DASP_PEEL_PIPE_F64=1+DASP_WIDE_META_PF_F64=0.so"
DASP_LIB=$P2 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "f64 and not x_stage" > gpurun_out/pipe_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pipe_pytest.log
run() { echo "# lib=$1 cfg=$2" >> $O; DASP_LIB=$1 timeout 300 $B --config $2 >> $O 2>> gpurun_out/pipe.err; }
for rep in 1 2; do
for cfg in "c3" "c5 --scale 0.05" "c2" "c2big"; do
  for lib in paper_conf_sc_lu023_b200/libdasp.so "$P2" "$P2N" "$P1N"; do run "$lib" "$cfg"; done
done
done
echo done
