#!/bin/bash
# dasp_spmv_host_stream check: parity tests, then the e2e leg of bench on c2 / c3 / c2 f16.
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 600 python -m pytest tests -m gpu -q -x -k "host" > gpurun_out/pytest_host.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_host.log
B="python bench.py --steps 200 --warmup 10 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-graph --no-library"
: > gpurun_out/e2e.jsonl
for a in "--config c2" "--config c2 --dtype f16" "--config c3" "--config c2big"; do
  timeout 300 $B $a >> gpurun_out/e2e.jsonl 2>> gpurun_out/e2e.err
done
python - <<'PY'
import json
for l in open("gpurun_out/e2e.jsonl"):
    d = json.loads(l); e = d["e2e"]
    print(d["config"]["workload"], d["dtype"], round(d["value"], 1), "e2e", round(e["value"], 1), e["ms_per_step"], "single", e.get("single_call"))
PY
echo done
