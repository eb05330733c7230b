#!/bin/bash
# narrow / mid warps interleaved per block (DASP_NARROW_IL) and the long-unit order (DASP_LONG_ORDER 0/1/2)
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/il2.jsonl
run() { echo "# $1 $3" >> gpurun_out/il2.jsonl; env $1 timeout 300 $B $2 >> gpurun_out/il2.jsonl 2>> gpurun_out/il2.err; }
for dt in f64 f16 f32; do
  for m in DASP_NARROW_IL=0 DASP_NARROW_IL=1 DASP_NARROW_IL=0 DASP_NARROW_IL=1; do run $m "--config c3 --dtype $dt"; done
done
for m in DASP_NARROW_IL=0 DASP_NARROW_IL=1 DASP_NARROW_IL=0 DASP_NARROW_IL=1; do run $m "--config c2 --dtype f16"; done
for m in DASP_NARROW_IL=0 DASP_NARROW_IL=1; do run $m "--config c5 --scale 0.05 --dtype f64"; done
for cfg in "c3" "c7"; do for dt in f64 f16; do
  for m in DASP_LONG_ORDER=0 DASP_LONG_ORDER=1 DASP_LONG_ORDER=2 DASP_LONG_ORDER=0 DASP_LONG_ORDER=1 DASP_LONG_ORDER=2; do run $m "--config $cfg --dtype $dt"; done
done; done
python scripts/show.py gpurun_out/il2.jsonl | paste - - | awk '{print $2, $3, $4, $6, $8, $10, $14, $15, $16, $17, $18, $19}'
echo done
