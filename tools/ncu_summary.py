#!/usr/bin/env python3
"""Summarise ncu output for profiles/: (1) a launch list CSV (--metrics gpu__time_duration.sum) into
per-kernel counts / total time / share of the step, (2) a --set full report (.ncu-rep) into the
metrics the roofline needs (duration, dram bytes read+write, DRAM throughput %, achieved occupancy,
registers, smem, top stall reasons).

usage: python tools/ncu_summary.py --launches gpurun_out/X_launches.csv --report gpurun_out/X_prof.ncu-rep
"""
import argparse
import csv
import io
import re
import subprocess
from collections import defaultdict

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic", "launch__grid_size",
        "launch__block_size", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
        "lts__t_bytes.sum", "l1tex__t_bytes.sum", "smsp__inst_executed.sum",
        "lts__t_sector_hit_rate.pct", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active"]


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    out = []
    for r in rows:
        if "Kernel Name" in r and "Metric Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d.get("Metric Name") == "gpu__time_duration.sum":
                unit = d.get("Metric Unit", "ns")
                v = float(d["Metric Value"].replace(",", ""))
                ns = v * {"ns": 1, "usecond": 1e3, "us": 1e3, "msecond": 1e6, "ms": 1e6, "nsecond": 1}.get(unit, 1)
                out.append((d["Kernel Name"], ns))
    agg = defaultdict(lambda: [0, 0.0])
    for k, ns in out:
        name = re.sub(r"\(.*", "", k)[:90]
        agg[name][0] += 1
        agg[name][1] += ns
    tot = sum(v[1] for v in agg.values()) or 1
    lines = [f"launches: {len(out)}, total kernel time {tot / 1e6:.3f} ms (cold-cache, serialised)", "",
             "| kernel | launches | total ms | mean us | share |", "|---|---|---|---|---|"]
    for k, (n, ns) in sorted(agg.items(), key=lambda x: -x[1][1]):
        lines.append(f"| `{k}` | {n} | {ns / 1e6:.3f} | {ns / n / 1e3:.1f} | {ns / tot:.1%} |")
    return "\n".join(lines)


def report(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    if not rows:
        return "(empty report)"
    hdr = rows[0]
    units = rows[1] if len(rows) > 1 else []
    lines = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        name = re.sub(r"\(.*", "", d.get("Kernel Name", "?"))
        lines.append(f"### {name} (id {d.get('ID', '?')}, grid {d.get('launch__grid_size', '?')}, "
                     f"block {d.get('launch__block_size', '?')})")
        for k in KEYS:
            if k in d:
                lines.append(f"- `{k}` = {d[k]} {u.get(k, '')}")
        try:
            dur_ns = float(d["gpu__time_duration.sum"].replace(",", ""))
            unit = u.get("gpu__time_duration.sum", "ns")
            dur_s = dur_ns * {"ns": 1e-9, "nsecond": 1e-9, "usecond": 1e-6, "us": 1e-6, "msecond": 1e-3, "ms": 1e-3}.get(unit, 1e-9)

            def byt(k):
                v = float(d[k].replace(",", ""))
                return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6,
                            "GB": 1e9}.get(u.get(k, "byte"), 1)
            tb = byt("dram__bytes_read.sum") + byt("dram__bytes_write.sum")
            lines.append(f"- DRAM traffic {tb / 1e6:.1f} MB in {dur_s * 1e6:.1f} us = {tb / dur_s / 1e9:.0f} GB/s")
        except Exception:  # noqa: BLE001
            pass
        stall = sorted(((float(d[k].replace(",", "") or 0), k) for k in d
                        if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued")),
                       reverse=True)[:5]
        if stall:
            lines.append("- top stall samples: " + ", ".join(f"{k.replace('smsp__pcsamp_warps_issue_stalled_', '')} {v:.0f}"
                                                           for v, k in stall))
        lines.append("")
    src = subprocess.run(["ncu", "-i", path, "--page", "details", "--csv"], capture_output=True, text=True).stdout
    stall = [ln for ln in src.splitlines() if "Stall" in ln or "Warp Cycles" in ln][:20]
    if stall:
        lines.append("details (stall-related rows):")
        lines += ["    " + s[:200] for s in stall]
    return "\n".join(lines)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--launches")
    ap.add_argument("--report")
    a = ap.parse_args()
    if a.launches:
        print("## Launch list\n")
        print(launches(a.launches))
        print()
    if a.report:
        print("## ncu --set full\n")
        print(report(a.report))


if __name__ == "__main__":
    main()
