#!/bin/bash
mkdir -p gpurun_out
O=gpurun_out/huge.jsonl
: > $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "huge or deterministic" > gpurun_out/huge_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/huge_pytest.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
for cfg in "c7" "c3" "c7 --dtype f16" "c5 --scale 0.05"; do echo "# cfg=$cfg" >> $O; timeout 300 $B --config $cfg >> $O 2>> gpurun_out/huge.err; done
echo done
