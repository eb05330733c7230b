#!/bin/bash
# e2e A/B: host->device by SM loads (default) vs copy engine (DASP_H2D_SM=0), plus the host-path parity tests
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "spmv_host" 2>&1 | tail -3
B="python bench.py --steps 200 --warmup 10 --e2e-steps 80 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/h2d_ab.jsonl
for cfg in "c2" "c2 --dtype f16" "c3" "c2big"; do for m in 1 0 1 0; do
  echo "# DASP_H2D_SM=$m $cfg" >> gpurun_out/h2d_ab.jsonl
  DASP_H2D_SM=$m timeout 300 $B --config $cfg >> gpurun_out/h2d_ab.jsonl 2>> gpurun_out/h2d_ab.err
done; done
python - <<'PY'
import json
for l in open("gpurun_out/h2d_ab.jsonl"):
    if l.startswith("#"): tag = l.strip(); continue
    try: d = json.loads(l)
    except Exception: continue
    e = d["e2e"]; print(tag, "value", round(d["value"], 1), "e2e", round(e["value"], 1), e["ms_per_step"], "single", round(e["single_call"]["value"], 1))
PY
echo done
