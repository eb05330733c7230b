#!/bin/bash
# probe: hot-column compaction on C3 (scripts/probe/hot_relabel.py)
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 1200 python scripts/probe/hot_relabel.py c3 > gpurun_out/hot_relabel.jsonl 2> gpurun_out/hot_relabel.err
echo "rc=$?"; cat gpurun_out/hot_relabel.jsonl; tail -5 gpurun_out/hot_relabel.err
