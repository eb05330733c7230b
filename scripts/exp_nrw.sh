#!/bin/bash
# row-blocks per narrow / mid warp (DASP_NRW 4 / 8 / 16 / 32)
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 600 python -m pytest tests -m gpu -q -x -k narrow > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/nrw.jsonl
for a in "--config c2 --dtype f16" "--config c2big --dtype f16" "--config c3 --dtype f16" "--config c3 --dtype f64" "--config c3 --dtype f32"; do
  for n in 8 4 16 32 8; do
    echo "# nrw $n" >> gpurun_out/nrw.jsonl
    DASP_NRW=$n timeout 300 $B $a >> gpurun_out/nrw.jsonl 2>> gpurun_out/nrw.err
  done
done
python scripts/show.py gpurun_out/nrw.jsonl | paste - - | awk '{print $2, $3, $4, $13, $14, $15}'
echo done
