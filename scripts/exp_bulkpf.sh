#!/bin/bash
# L2 bulk prefetch of the next row-block's regular region (DASP_BULK_PF=1, this build) vs off
mkdir -p gpurun_out
make -j8 all > gpurun_out/make.log 2>&1 || { tail -30 gpurun_out/make.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -k "parity" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
B="python bench.py --steps 300 --warmup 10 --e2e-steps 0 --no-cpu-baseline --no-triad --no-gpu-build --no-graph --no-library"
: > gpurun_out/bulkpf.jsonl
for cfg in "c2" "c2big" "c3" "c5 --scale 0.05"; do for dt in f64 f32 f16; do
  for lib in on off; do
    echo "# pf $lib" >> gpurun_out/bulkpf.jsonl
    if [ $lib = on ]; then L=$PWD/paper_conf_sc_lu023_b200/libdasp.so; else L=$PWD/build/libdasp_DASP_BULK_PF=0.so; fi
    DASP_LIB=$L timeout 300 $B --config $cfg --dtype $dt >> gpurun_out/bulkpf.jsonl 2>> gpurun_out/bulkpf.err
  done
done; done
python scripts/show.py gpurun_out/bulkpf.jsonl
python - <<'PY'
import json
for l in open("gpurun_out/bulkpf.jsonl"):
    if l.startswith("{"):
        d = json.loads(l); vc = d.get("variant_compare") or {}
        print(d["config"]["workload"], d["dtype"], {k: round(v["ms_per_step"], 4) for k, v in vc.items()})
PY
echo done
