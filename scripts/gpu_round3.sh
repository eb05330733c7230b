#!/bin/bash
# Round evidence (r01d): build, smoke, GPU tests, default bench line, reference arm, config sweep (all
# dtypes), launch lists (incl. the default bench command), ncu --set full of the main/long kernels
# (summarised on the box), CG.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.log 2> gpurun_out/bench.err; echo "bench rc=$?"; cat gpurun_out/bench.log
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_ref.log 2> gpurun_out/bench_ref.err; echo "ref rc=$?"
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-graph --no-library"
: > gpurun_out/sweep.jsonl
for cfg in "c2" "c2big" "c3" "c7" "c6 --scale 20" "c5 --scale 0.05" "c1a" "c1b"; do for dt in f64 f16 f32; do
  timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
done; done
timeout 300 python bench.py --steps 200 --warmup 5 --e2e-steps 3 --no-cpu-baseline --no-triad --iterate --config c5 --scale 0.05 >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
timeout 300 python bench.py --steps 200 --warmup 5 --e2e-steps 3 --no-cpu-baseline --no-triad --iterate --halo --config c2 >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
timeout 300 python bench.py --steps 200 --warmup 5 --e2e-steps 3 --no-cpu-baseline --no-triad --iterate --fused --config c2 >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches_default_cmd.csv python bench.py --steps 3 --warmup 3 --e2e-steps 2 --cpu-budget-s 1 > /dev/null 2>&1
S="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare --no-gpu-build --no-graph --no-library"
for cfg in c2 c3 c2big; do
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches_$cfg.csv $S --config $cfg > /dev/null 2>&1
done
P="ncu --set full --clock-control none --import-source on -k regex:dasp_(main|long) -s 3 -c 2"
timeout 900 $P -o gpurun_out/prof_c2_f64_cudacore $S > /dev/null 2>&1
timeout 900 $P -o gpurun_out/prof_c2_f64_mma $S --variant mma > /dev/null 2>&1
timeout 900 $P -o gpurun_out/prof_c2big_f64_cudacore $S --config c2big > /dev/null 2>&1
timeout 900 $P -o gpurun_out/prof_c3_f64_cudacore $S --config c3 > /dev/null 2>&1
timeout 900 $P -o gpurun_out/prof_c3_f64_mma $S --config c3 --variant mma > /dev/null 2>&1
timeout 900 $P -o gpurun_out/prof_c2_f16_cudacore $S --dtype f16 > /dev/null 2>&1
timeout 900 $P -o gpurun_out/prof_c2_f16_mma $S --dtype f16 --variant mma > /dev/null 2>&1
timeout 900 $P -o gpurun_out/prof_c2_f32_cudacore $S --dtype f32 > /dev/null 2>&1
timeout 900 $P -o gpurun_out/prof_c3_f16_cudacore $S --config c3 --dtype f16 > /dev/null 2>&1
# STREAM triad under ncu with the same clock control (the 75% target's denominator)
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:elementwise --log-file gpurun_out/triad_ncu.csv python -c "
import torch; n=1<<28
b=torch.rand(n,dtype=torch.float64,device='cuda'); c=torch.rand(n,dtype=torch.float64,device='cuda'); a=torch.empty_like(b)
for _ in range(5): torch.add(b,c,alpha=3.0,out=a)
torch.cuda.synchronize()" > /dev/null 2>&1
echo '{}' > gpurun_out/ncu_traffic.json
NCU_TRAFFIC=gpurun_out/ncu_traffic.json python scripts/ncu_summary.py gpurun_out/ncu_summary.md \
  c2/f64/cudacore=gpurun_out/prof_c2_f64_cudacore.ncu-rep c2/f64/mma=gpurun_out/prof_c2_f64_mma.ncu-rep \
  c2big/f64/cudacore=gpurun_out/prof_c2big_f64_cudacore.ncu-rep c3/f64/cudacore=gpurun_out/prof_c3_f64_cudacore.ncu-rep \
  c3/f64/mma=gpurun_out/prof_c3_f64_mma.ncu-rep c2/f16/cudacore=gpurun_out/prof_c2_f16_cudacore.ncu-rep \
  c2/f16/mma=gpurun_out/prof_c2_f16_mma.ncu-rep \
  c2/f32/cudacore=gpurun_out/prof_c2_f32_cudacore.ncu-rep c3/f16/cudacore=gpurun_out/prof_c3_f16_cudacore.ncu-rep \
  > gpurun_out/ncu_summary.log 2>&1
for r in gpurun_out/*.ncu-rep; do
  case $r in *prof_c2_f64_cudacore*|*prof_c3_f64_cudacore*) ;; *) rm -f $r ;; esac
done
[ "$(du -sm gpurun_out | cut -f1)" -gt 55 ] && rm -f gpurun_out/prof_c3_f64_cudacore.ncu-rep
du -sh gpurun_out
timeout 600 python scripts/cg_bench.py > gpurun_out/cg.jsonl 2> gpurun_out/cg.err; echo "cg rc=$?"; cat gpurun_out/cg.jsonl
echo done
