#!/bin/bash
# end-of-round evidence at HEAD: smoke, GPU suite, default bench line (1000 steps) and the driver's form,
# reference arm, config sweep, launch list of the default command, ncu --set full of C3 FP64 / FP16, C2+
O=gpurun_out/r02b_final3
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,power.limit --format=csv > $O/smi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1800 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 $O/pytest_gpu.log
timeout 900 python bench.py > $O/bench.jsonl 2> $O/bench.err; echo "bench rc=$?"
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench_driver_form.jsonl 2> $O/bench_driver_form.err; echo "bench20 rc=$?"
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > $O/bench_ref.jsonl 2> $O/bench_ref.err; echo "ref rc=$?"
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-sub"
: > $O/sweep.jsonl
for cfg in "c2" "c2big" "c3" "c5 --scale 0.05" "c6 --scale 20" "c7"; do for dt in f64 f16 f32; do
  timeout 300 $B --config $cfg --dtype $dt >> $O/sweep.jsonl 2>> $O/sweep.err
done; done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_default_cmd.csv \
  python bench.py --steps 20 --warmup 3 --e2e-steps 2 --no-cpu-baseline --no-triad --no-gpu-build > /dev/null 2>&1; echo "launches rc=$?"
S="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare --no-gpu-build --no-graph --no-sub"
P="ncu --set full --clock-control none --import-source on -k regex:dasp_(main|long) -s 3 -c 2"
timeout 900 $P -o $O/prof_c3_f64_cudacore $S --config c3 > /dev/null 2>&1
timeout 900 $P -o $O/prof_c3_f16_cudacore $S --config c3 --dtype f16 > /dev/null 2>&1
timeout 900 $P -o $O/prof_c2big_f64_cudacore $S --config c2big > /dev/null 2>&1
timeout 900 $P -o $O/prof_c2_f64_cudacore $S --config c2 > /dev/null 2>&1
echo '{}' > $O/ncu_traffic.json
NCU_TRAFFIC=$O/ncu_traffic.json python scripts/ncu_summary.py $O/ncu_summary.md \
  c3/f64/cudacore=$O/prof_c3_f64_cudacore.ncu-rep c3/f16/cudacore=$O/prof_c3_f16_cudacore.ncu-rep \
  c2big/f64/cudacore=$O/prof_c2big_f64_cudacore.ncu-rep c2/f64/cudacore=$O/prof_c2_f64_cudacore.ncu-rep > $O/ncu_summary.log 2>&1
for r in $O/*.ncu-rep; do ncu -i $r --page raw --csv > ${r%.ncu-rep}.raw.csv 2>/dev/null; done
rm -f $O/*.ncu-rep
du -sh $O
echo done
