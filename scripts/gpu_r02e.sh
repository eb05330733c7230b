#!/bin/bash
# round 2: concurrent long / main kernels -- parity, A/B over blocks per SM; hot-x L1 probe (default cold policy)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "concurrent or units" > gpurun_out/pytest_conc.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_conc.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > gpurun_out/ab4.jsonl
for cfg in "c3" "c5 --scale 0.05" "c3 --dtype f16" "c3 --dtype f32" "c7" "c5 --scale 0.05 --dtype f16"; do
  for m in "--concurrent-long 0 --medium-units 0" "--concurrent-long 0 --medium-units 1" "--concurrent-long 1" "--concurrent-long 2" "--concurrent-long 3" "--concurrent-long 4"; do
    echo "# cfg=$cfg $m" >> gpurun_out/ab4.jsonl
    timeout 300 $B --config $cfg $m >> gpurun_out/ab4.jsonl 2>> gpurun_out/ab4.err
  done
done
cd scripts/probe && DASP_LIB=../../build/libdasp_DASP_EXP_HOT=1.so timeout 1200 python hot_l1.py c3 > ../../gpurun_out/hot_l1b.jsonl 2> ../../gpurun_out/hot_l1b.err; cd ../..
echo done
