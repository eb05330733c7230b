#!/bin/bash
# Quick round check: build, smoke, GPU tests, default bench line, reference arm, short sweep,
# launch lists and ncu --set full captures (summarised on the box) of the C2 / C3 FP64 kernels.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/smi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.log 2> gpurun_out/bench.err; echo "bench rc=$?"; cat gpurun_out/bench.log
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_ref.log 2> gpurun_out/bench_ref.err; echo "ref rc=$?"; cat gpurun_out/bench_ref.log
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph"
: > gpurun_out/sweep.jsonl
for cfg in "c2big" "c3" "c6 --scale 20" "c5 --scale 0.05"; do for dt in f64 f16 f32; do
  timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
done; done
S="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare --no-gpu-build --no-graph"
for cfg in c2 c3; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$cfg.csv $S --config $cfg > /dev/null 2>&1
done
P="ncu --set full --clock-control none --import-source on -k regex:dasp_(main|long) -s 3 -c 2"
timeout 900 $P -o gpurun_out/prof_c2_f64_cudacore $S > /dev/null 2>&1
timeout 900 $P -o gpurun_out/prof_c3_f64_cudacore $S --config c3 > /dev/null 2>&1
timeout 900 $P -o gpurun_out/prof_c6_f64_cudacore $S --config c6 --scale 20 > /dev/null 2>&1
echo '{}' > gpurun_out/ncu_traffic.json
NCU_TRAFFIC=gpurun_out/ncu_traffic.json python scripts/ncu_summary.py gpurun_out/ncu_summary.md \
  c2/f64/cudacore=gpurun_out/prof_c2_f64_cudacore.ncu-rep c3/f64/cudacore=gpurun_out/prof_c3_f64_cudacore.ncu-rep \
  c6/f64/cudacore=gpurun_out/prof_c6_f64_cudacore.ncu-rep > gpurun_out/ncu_summary.log 2>&1
for r in gpurun_out/*.ncu-rep; do
  ncu -i $r --page source --csv > ${r%.ncu-rep}.source.csv 2>/dev/null
  ncu -i $r --page raw --csv > ${r%.ncu-rep}.raw.csv 2>/dev/null
done
[ "$(du -sm gpurun_out | cut -f1)" -gt 55 ] && rm -f gpurun_out/prof_c6_f64_cudacore.ncu-rep
[ "$(du -sm gpurun_out | cut -f1)" -gt 55 ] && rm -f gpurun_out/prof_c2_f64_cudacore.ncu-rep
[ "$(du -sm gpurun_out | cut -f1)" -gt 55 ] && rm -f gpurun_out/*.source.csv
du -sh gpurun_out
echo done
