#!/bin/bash
# group-staged medium kernel (DASP_MED_GROUP=1) on the stencils vs the default main kernel
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 600 python -m pytest tests -m gpu -q -x -k "med_group" > gpurun_out/pytest_mg.log 2>&1; echo "pytest mg rc=$?"; tail -3 gpurun_out/pytest_mg.log
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/mg.jsonl
for cfg in c2 c2big; do for dt in f64 f32; do for m in 0 1 0 1; do
  echo "# mg $m" >> gpurun_out/mg.jsonl
  DASP_MED_GROUP=$m timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/mg.jsonl 2>> gpurun_out/mg.err
done; done; done
python scripts/show.py gpurun_out/mg.jsonl | paste - - | awk '{print $2, $3, $4, $5, $8, $14, $15}'
tail -5 gpurun_out/mg.err
echo done
