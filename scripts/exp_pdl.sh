#!/bin/bash
# programmatic dependent launch (DASP_PDL=1) between consecutive SpMV kernels: parity + A/B
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
L1=$PWD/build/libdasp_DASP_PDL=1.so
DASP_LIB=$L1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_solvers.py -q -x 2>&1 | tail -2
B="python bench.py --steps 1000 --warmup 20 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-compare --no-library"
: > gpurun_out/pdl.jsonl
for cfg in "c2" "c2 --dtype f16" "c3" "c1a" "c6" "c2big"; do for lib in base pdl base pdl; do
  echo "# $lib $cfg" >> gpurun_out/pdl.jsonl
  if [ $lib = base ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$L1; fi
  DASP_LIB=$L timeout 300 $B --config $cfg >> gpurun_out/pdl.jsonl 2>> gpurun_out/pdl.err
done; done
python - <<'PY'
import json
for l in open("gpurun_out/pdl.jsonl"):
    if l.startswith("#"): tag = l.strip(); continue
    try: d = json.loads(l)
    except Exception: continue
    r = d["roofline"]; g = d.get("cuda_graph") or {}
    print(tag, "step_ms %.5f" % d["ms_per_step"], "kern_ms %.5f" % r["avg_launch_ms"], "graph_ms", g.get("ms_per_step", g.get("error")))
PY
echo done
