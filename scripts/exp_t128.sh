#!/bin/bash
# 128-thread blocks for the main / long kernels: A = 56 registers (9 blocks, 36 warps/SM), B = 64
# registers (8 blocks, 32 warps/SM: same occupancy, finer block granularity) vs the 256-thread build
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/t128.jsonl
for cfg in "c2" "c2big" "c3" "c5 --scale 0.05" "c6 --scale 20"; do for dt in f64 f16 f32; do
  for lib in base t128A t128B; do
    echo "# $lib" >> gpurun_out/t128.jsonl
    if [ $lib = base ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$PWD/build/libdasp_$lib.so; fi
    DASP_LIB=$L timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/t128.jsonl 2>> gpurun_out/t128.err
  done
done; done
DASP_LIB=$PWD/build/libdasp_t128B.so timeout 900 python -m pytest tests -m gpu -q -x -k "parity or narrow" > gpurun_out/pytest_t128B.log 2>&1; echo "pytest B rc=$?"; tail -1 gpurun_out/pytest_t128B.log
python scripts/show.py gpurun_out/t128.jsonl | paste - - | awk '{print $2, $3, $4, $10, $12, $13, $14, $15, $16, $17, $18, $19}'
echo done
