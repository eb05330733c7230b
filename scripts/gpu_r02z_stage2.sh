#!/bin/bash
# x-window staging v2 (no block-wide wait on the entry load; tile map bulk-copied) A/B + parity;
# ncu source capture (cuda,sass) of the C3 FP64 main kernel at HEAD
mkdir -p gpurun_out
O=gpurun_out/stage2.jsonl
: > $O
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "x_stage or c2s" > gpurun_out/stage2_pytest.log 2>&1; echo "stage tests rc=$?"; tail -2 gpurun_out/stage2_pytest.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
for cfg in "c2" "c2big" "c2 --dtype f32"; do
  for xs in 1 0; do echo "# x_stage=$xs cfg=$cfg" >> $O; timeout 300 $B --config $cfg --x-stage $xs >> $O 2>> gpurun_out/stage2.err; done
done
S="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare --no-gpu-build --no-graph --no-sub"
P="ncu --set full --clock-control none --import-source on -k regex:dasp_main -s 3 -c 1"
timeout 900 $P -o gpurun_out/prof_c2_staged $S --config c2 --x-stage 0 > /dev/null 2>&1
timeout 900 $P -o gpurun_out/prof_c2_unstaged $S --config c2 --x-stage 1 > /dev/null 2>&1
timeout 900 $P -o gpurun_out/prof_c3_main $S --config c3 > /dev/null 2>&1
for r in gpurun_out/prof_c2_staged gpurun_out/prof_c2_unstaged gpurun_out/prof_c3_main; do
  ncu -i $r.ncu-rep --page raw --csv > $r.raw.csv 2>/dev/null
  ncu -i $r.ncu-rep --page source --csv --print-source cuda,sass > $r.source.csv 2>/dev/null
  ncu -i $r.ncu-rep --page details --csv > $r.details.csv 2>/dev/null
done
ls -la gpurun_out/
echo done
