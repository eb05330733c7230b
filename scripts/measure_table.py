#!/usr/bin/env python3
"""Markdown table of bench JSON lines (one per line; non-bench lines skipped).

    python scripts/measure_table.py profiles/r01/sweep_configs.jsonl [...]
"""
import json
import sys


def main():
    print("| workload | dtype | GFLOPS | ms/step | kernels: avg ms (alg GB/s) | dominant | frac of peak | CSR-equiv GB/s |")
    print("|---|---|---|---|---|---|---|---|")
    for path in sys.argv[1:]:
        for line in open(path):
            try:
                d = json.loads(line)
            except ValueError:
                continue
            if "value" not in d or "roofline" not in d:
                continue
            r = d["roofline"]
            ks = "; ".join(f"{k.replace('dasp_', '').replace('_kernel', '')} {v['avg_ms']:.4f} ({v['alg_gbs']:.0f})"
                           for k, v in r["kernels"].items() if v.get("alg_gbs"))
            par = d["config"].get("parallelism", "")
            wl = d["config"]["workload"] + (" (iterate" + (", halo" if "halo" in par else "") + ")" if " + " in par else "")
            print(f"| {wl} | {d['dtype']} | {d['value']:.1f} | {d['ms_per_step']:.4f} | {ks} | "
                  f"{r['kernel'].replace('dasp_', '')} | {r['frac']:.3f} | {d['effective_gbs']:.0f} |")


if __name__ == "__main__":
    main()
