#!/bin/bash
# HEAD check: smoke, GPU suite, default bench line (short), launch list of the default command
O=gpurun_out/r02b_head
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,power.limit --format=csv > $O/smi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest_gpu.log
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench_driver_form.jsonl 2> $O/bench_driver_form.err; echo "bench rc=$?"
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.jsonl 2> $O/bench_ref.err; echo "ref rc=$?"
echo done
