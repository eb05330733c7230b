#!/bin/bash
# round 2 evidence run: smoke, GPU suite, default bench line, reference arm, ncu (launch list of the
# default command, --set full captures of C3 FP64 / FP16 and C2+), L2 gather ceiling, sanitizers
mkdir -p gpurun_out/r02f
O=gpurun_out/r02f
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 600 python scripts/probe/l2peak.py > $O/l2peak.jsonl 2> $O/l2peak.err; echo "l2peak rc=$?"
timeout 900 python bench.py > $O/bench.jsonl 2> $O/bench.err; echo "bench rc=$?"
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > $O/bench_ref.jsonl 2> $O/bench_ref.err; echo "ref rc=$?"
S="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare --no-gpu-build --no-graph --no-sub"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_default_cmd.csv python bench.py --steps 20 --warmup 3 --e2e-steps 2 --no-cpu-baseline --no-triad --no-gpu-build > /dev/null 2>&1; echo "launches rc=$?"
P="ncu --set full --clock-control none --import-source on -k regex:dasp_(main|long) -s 3 -c 2"
timeout 900 $P -o $O/prof_c3_f64_cudacore $S --config c3 > /dev/null 2>&1
timeout 900 $P -o $O/prof_c3_f16_cudacore $S --config c3 --dtype f16 > /dev/null 2>&1
timeout 900 $P -o $O/prof_c2big_f64_cudacore $S --config c2big > /dev/null 2>&1
timeout 900 $P -o $O/prof_c3_f64_mma $S --config c3 --variant mma > /dev/null 2>&1
echo '{}' > $O/ncu_traffic.json
NCU_TRAFFIC=$O/ncu_traffic.json python scripts/ncu_summary.py $O/ncu_summary.md \
  c3/f64/cudacore=$O/prof_c3_f64_cudacore.ncu-rep c3/f16/cudacore=$O/prof_c3_f16_cudacore.ncu-rep \
  c2big/f64/cudacore=$O/prof_c2big_f64_cudacore.ncu-rep c3/f64/mma=$O/prof_c3_f64_mma.ncu-rep > $O/ncu_summary.log 2>&1
for r in $O/*.ncu-rep; do ncu -i $r --page raw --csv > ${r%.ncu-rep}.raw.csv 2>/dev/null; done
rm -f $O/prof_c3_f64_mma.ncu-rep $O/prof_c2big_f64_cudacore.ncu-rep
timeout 2400 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest_gpu.log
bash scripts/sanitize.sh
mv gpurun_out/sanitize_*.log $O/ 2>/dev/null
du -sh $O
echo done
