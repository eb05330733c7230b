#!/bin/bash
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
B="python bench.py --steps 200 --warmup 10 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/xpol.jsonl
for cfg in "c3" "c2" "c7" "c6 --scale 20"; do
 for xm in 0 1; do for apw in 0 1; do for v in mma cudacore; do
  echo "{\"xmode\": $xm, \"apw\": $apw}" >> gpurun_out/xpol.jsonl
  DASP_XMODE=$xm DASP_X_APW=$apw timeout 300 $B --config $cfg --variant $v >> gpurun_out/xpol.jsonl 2>> gpurun_out/xpol.err
 done; done; done
done
python -c "import torch; p=torch.cuda.get_device_properties(0); print(p)" >> gpurun_out/xpol.err
nvidia-smi -q | grep -i -A3 "persist" >> gpurun_out/xpol.err
echo done
