#!/bin/bash
# panel lookup from the kernel parameter space (this build; DASP_PARAM_PANELS=0 = blk_word load) vs the previous commit
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
B="python bench.py --steps 500 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/ppan.jsonl
for cfg in "c2" "c3" "c2big" "c5 --scale 0.05" "c6 --scale 20"; do for dt in f64 f32 f16; do
  for mode in old new off old new off; do
    echo "# $mode" >> gpurun_out/ppan.jsonl
    case $mode in old) E="DASP_LIB=$PWD/exp/libdasp_old.so";; new) E="A=1";; off) E="DASP_PARAM_PANELS=0";; esac
    env $E timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/ppan.jsonl 2>> gpurun_out/ppan.err
  done
done; done
python scripts/show.py gpurun_out/ppan.jsonl | paste - - | awk '{print $2, $3, $4, $6, $10, $14, $15, $16, $17, $18, $19}'
echo done
