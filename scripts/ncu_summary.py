#!/usr/bin/env python3
"""Summarise Nsight Compute reports of dasp_main_kernel into profiles/ (markdown + traffic JSON).

    python scripts/ncu_summary.py OUT.md KEY=REPORT.ncu-rep [KEY=REPORT.ncu-rep ...]
    NCU_TRAFFIC=path  overrides where the traffic JSON is merged (default profiles/ncu_traffic.json)

KEY is "<workload>/<dtype>/<variant>"; traffic is stored per "<KEY>/<kernel>" (bench.py's lookup
key for roofline.traffic); every dasp_* kernel captured in the report is summarised.
profiles/ncu_traffic.json receives dram__bytes_read.sum + dram__bytes_write.sum per launch.
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

WANT = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit %"),
    ("l1tex__t_sector_hit_rate.pct", "L1 hit %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "LSU pipe inst %"),
    ("sm__inst_executed_pipe_tensor_subpipe_dmma.avg.pct_of_peak_sustained_active", "tensor DMMA inst %"),
    ("sm__inst_executed_pipe_tensor_subpipe_hmma.avg.pct_of_peak_sustained_active", "tensor HMMA inst %"),
    ("TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed", "tensor pipe cycles active %"),
    ("TPC.TriageCompute.sm__pipe_fp64_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed", "FP64 pipe cycles active %"),
    ("sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "FMA pipe inst %"),
    ("sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active", "FP64 pipe inst %"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("lts__t_sectors_srcunit_tex_op_read.sum", "L2 read sectors from L1 (streams + x gathers)"),
    ("lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum", "L2 read sector misses"),
    ("lts__t_requests_srcunit_tex_op_read.sum", "L2 read requests from L1"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 (LTS) throughput % of peak"),
    ("lts__t_sectors.sum.pct_of_peak_sustained_elapsed", "L2 sectors % of peak"),
    ("l1tex__throughput.avg.pct_of_peak_sustained_elapsed", "L1 throughput % of peak"),
]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        res.append({h[i]: (u[i], r[i]) for i in range(len(h))})
    return res


def to_bytes(unit, v):
    f = float(v.replace(",", ""))
    return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)


def main():
    out_md = sys.argv[1]
    traffic_path = os.environ.get("NCU_TRAFFIC", os.path.join(ROOT, "profiles", "ncu_traffic.json"))
    traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
    lines = ["# ncu summaries (dasp_main_kernel / dasp_long_kernel, `--set full --clock-control none`, one launch each)", ""]
    for arg in sys.argv[2:]:
        key, rep = arg.split("=", 1)
        for k, d in enumerate(raw(rep)):
            kname = d.get("Kernel Name", ("", ""))[1]
            kern = next((n for n in ("dasp_main_kernel", "dasp_long_kernel") if n in kname), None)
            if kern is None:
                continue
            lines.append(f"## {key} — {kern}  ({os.path.basename(rep)})")
            lines.append("")
            lines.append("| metric | value |")
            lines.append("|---|---|")
            for m, name in WANT:
                if m in d:
                    lines.append(f"| {name} (`{m}`) | {d[m][1]} {d[m][0]} |")
            stalls = sorted(((float(v[1].replace(",", "") or 0), m) for m, v in d.items()
                             if m.startswith("smsp__pcsamp_warps_issue_stalled_") and not m.endswith("not_issued")),
                            reverse=True)[:6]
            lines.append("| top stall samples | " + ", ".join(f"{m.split('stalled_')[1]} {int(c)}" for c, m in stalls) + " |")
            rd = to_bytes(*d["dram__bytes_read.sum"])
            wr = to_bytes(*d["dram__bytes_write.sum"])
            traffic[f"{key}/{kern}"] = rd + wr
            sec = d.get("lts__t_sectors_srcunit_tex_op_read.sum")
            dur = d.get("gpu__time_duration.sum")
            if sec and dur:
                ns = float(dur[1].replace(",", "")) * {"ns": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6}.get(dur[0], 1)
                traffic[f"{key}/{kern}/l2_read_sectors"] = float(sec[1].replace(",", ""))
                traffic[f"{key}/{kern}/l2_read_Gsectors_per_s"] = float(sec[1].replace(",", "")) / ns
            req = d.get("lts__t_requests_srcunit_tex_op_read.sum")
            if req:
                traffic[f"{key}/{kern}/l2_read_requests"] = float(req[1].replace(",", ""))
            lines.append("")
    with open(out_md, "w") as f:
        f.write("\n".join(lines) + "\n")
    with open(traffic_path, "w") as f:
        json.dump(traffic, f, indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
