#!/bin/bash
# C3 x-locality knobs: long-unit order, panel size, persisting L2 window over x (main + long kernel)
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
python -c "import torch; p=torch.cuda.get_device_properties(0); print(p.L2_cache_size, getattr(p,'persisting_l2_cache_max_size',None))" > gpurun_out/l2x_props.txt 2>&1
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library --config c3"
: > gpurun_out/l2x.jsonl
run() { echo "# $1" >> gpurun_out/l2x.jsonl; env $2 timeout 300 $B $3 >> gpurun_out/l2x.jsonl 2>> gpurun_out/l2x.err; }
run base "A=1" ""
run long_order0 "DASP_LONG_ORDER=0" ""
run panel_global "A=1" "--panel-rows -1"
run panel_4M "A=1" "--panel-rows 4194304"
run panel_256K "A=1" "--panel-rows 262144"
run apw "DASP_X_APW=1" ""
run apw_hit0.5 "DASP_X_APW=1 DASP_X_APW_HIT=0.5" ""
run apw_hit0.25 "DASP_X_APW=1 DASP_X_APW_HIT=0.25" ""
run f16_base "A=1" "--dtype f16"
run f16_apw "DASP_X_APW=1" "--dtype f16"
python scripts/show.py gpurun_out/l2x.jsonl
cat gpurun_out/l2x_props.txt
echo done
