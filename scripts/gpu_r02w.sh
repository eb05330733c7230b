#!/bin/bash
# variant justification (north_star (3)): ncu of the MMA (DMMA / HMMA) and CUDA-core variants of the
# same format, tensor-pipe vs FMA-pipe utilisation and DRAM bandwidth
O=gpurun_out/r02_variants
mkdir -p $O
S="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-triad --no-compare --no-gpu-build --no-graph --no-sub"
P="ncu --set full --clock-control none -k regex:dasp_(main|long) -s 3 -c 2"
for v in mma cudacore; do
  for c in "c2" "c2 --dtype f16" "c3 --dtype f16" "c2big"; do
    tag=$(echo "$c" | tr -d ' -' | sed 's/dtype//')
    timeout 900 $P -o $O/prof_${tag}_$v $S --config $c --variant $v > /dev/null 2>&1
  done
done
echo '{}' > $O/ncu_traffic.json
NCU_TRAFFIC=$O/ncu_traffic.json python scripts/ncu_summary.py $O/ncu_summary.md \
  c2/f64/mma=$O/prof_c2_mma.ncu-rep c2/f64/cudacore=$O/prof_c2_cudacore.ncu-rep \
  c2/f16/mma=$O/prof_c2f16_mma.ncu-rep c2/f16/cudacore=$O/prof_c2f16_cudacore.ncu-rep \
  c3/f16/mma=$O/prof_c3f16_mma.ncu-rep c3/f16/cudacore=$O/prof_c3f16_cudacore.ncu-rep \
  c2big/f64/mma=$O/prof_c2big_mma.ncu-rep c2big/f64/cudacore=$O/prof_c2big_cudacore.ncu-rep > $O/ncu_summary.log 2>&1
rm -f $O/*.ncu-rep
echo done
