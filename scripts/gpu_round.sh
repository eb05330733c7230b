#!/bin/bash
# Round check: build, smoke, GPU tests, default bench line, class/dtype sweep, ncu evidence.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.log 2> gpurun_out/bench.err; echo "bench rc=$?"; cat gpurun_out/bench.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep.jsonl
for cfg in "c2" "c3" "c2big" "c7" "c6 --scale 20"; do for dt in f64 f16; do for v in mma cudacore; do
  timeout 300 $B --config $cfg --dtype $dt --variant $v >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
done; done; done
S="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv $S > /dev/null 2>&1
for v in mma cudacore; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:dasp_main -s 3 -c 1 -o gpurun_out/prof_c2_f64_$v $S --variant $v > /dev/null 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dasp_main -s 3 -c 1 -o gpurun_out/prof_c2_f16_mma $S --dtype f16 > /dev/null 2>&1
echo done
