#!/bin/bash
# C5 at full size (62.5M rows, ~4e9 nnz, FP64) on ONE B200: the whole packed matrix (~48 GB)
# resident in HBM.  Host builder (the device builder would need the CSR and the plan on the GPU
# at once), 2 e2e steps, oracle baseline on a bounded row sample.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
( while true; do nvidia-smi --query-gpu=memory.used --format=csv,noheader >> gpurun_out/c5_mem.log; free -g | awk 'NR==2{print "host_used_gb", $3}' >> gpurun_out/c5_mem.log; sleep 10; done ) &
MON=$!
timeout 1500 python bench.py --config c5 --steps 30 --warmup 3 --no-gpu-build --e2e-steps 2 --no-compare ${EXTRA} \
  > gpurun_out/c5_full.jsonl 2> gpurun_out/c5_full.err
echo "bench rc=$?"
kill $MON
cat gpurun_out/c5_full.jsonl | head -c 3000
