#!/bin/bash
# 16-bit medium columns: parity (col16 = bitwise int32 columns; fuzz) and A/B on the stencils / C3
mkdir -p gpurun_out
O=gpurun_out/col16.jsonl
: > $O
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fuzz.py -q -x -k "col16 or fuzz_bit" > gpurun_out/col16_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/col16_pytest.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
run() { echo "# col16=$1 cfg=$2" >> $O; timeout 300 $B --config $2 --col16 $1 >> $O 2>> gpurun_out/col16.err; }
for cfg in "c2" "c2big" "c2 --dtype f16" "c2big --dtype f16" "c2 --dtype f32" "c2big --dtype f32" "c3"; do
  for c in 1 2; do run $c "$cfg"; done
done
echo done
