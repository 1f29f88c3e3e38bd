#!/usr/bin/env python3
"""Copy/compute overlap of pipelined launches from the CUDA driver's own activity records (CUPTI, via
torch.profiler/Kineto): the nsys-style timeline that nsys (not in this image) would give. Unlike
tools/timeline.py (PP_OPT_TRACE: a timing event around every op, which perturbs the schedule), CUPTI
activity tracing timestamps every memcpy and kernel the library issues with no extra work on the
streams, so the timed launch runs the unmodified schedule (eager or CUDA-graph replay).

Writes the Chrome trace (open in chrome://tracing or Perfetto; the library's H2D / kernel / D2H ops
appear on their own CUDA streams) and prints one JSON line of overlap statistics per profiled launch:
H2D-busy, D2H-busy, both-busy fractions of the launch span, kernel time nested inside copy-busy time,
and the copy bytes CUPTI saw (checked against pp_query's counts).

usage: python tools/cupti_timeline.py --c 2 --S 3 --policy 1 [--graph 1] --out gpurun_out/t.json
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
from torch.profiler import ProfilerActivity, profile  # noqa: E402

import paper_conf_ipps_cuissf17_b200 as pp  # noqa: E402
import synth  # noqa: E402

sys.path.insert(0, os.path.join(ROOT, "tools"))
from timeline import intersect, length, union  # noqa: E402


def kind_of(ev):
    cat, name = ev.get("cat", ""), ev.get("name", "")
    if cat == "gpu_memcpy":
        if "HtoD" in name:
            return "H2D"
        if "DtoH" in name:
            return "D2H"
        return None
    if cat == "kernel":
        return "KER"
    return None


def launch_stats(ops):
    t0 = min(o[1] for o in ops)
    t1 = max(o[2] for o in ops)
    span = t1 - t0
    h = union([(a, b) for k, a, b, _ in ops if k == "H2D"])
    d = union([(a, b) for k, a, b, _ in ops if k == "D2H"])
    ker = union([(a, b) for k, a, b, _ in ops if k == "KER"])
    cp = union(h + d)
    hb = sum(n for k, _, _, n in ops if k == "H2D")
    db = sum(n for k, _, _, n in ops if k == "D2H")
    return {"span_ms": span / 1e3, "h2d_busy_frac": length(h) / span, "d2h_busy_frac": length(d) / span,
            "both_busy_frac": length(intersect(h, d)) / span, "kernel_ms": length(ker) / 1e3,
            "kernel_inside_copy_frac": length(intersect(ker, cp)) / max(1e-9, length(ker)),
            "h2d_bytes": hb, "d2h_bytes": db,
            "h2d_gbs_while_busy": hb / (length(h) * 1e-6) / 1e9 if h else None,
            "d2h_gbs_while_busy": db / (length(d) * 1e-6) / 1e9 if d else None,
            "n_h2d": sum(1 for o in ops if o[0] == "H2D"), "n_d2h": sum(1 for o in ops if o[0] == "D2H"),
            "n_kernels": sum(1 for o in ops if o[0] == "KER"),
            "h2d_gap_us_median": gap_median(ops, "H2D"), "d2h_gap_us_median": gap_median(ops, "D2H")}


def gap_median(ops, kind):
    """Median idle time between consecutive copies of one direction (us): the copy engine's gap."""
    iv = sorted((a, b) for k, a, b, _ in ops if k == kind)
    g = sorted(iv[i + 1][0] - iv[i][1] for i in range(len(iv) - 1))
    return g[len(g) // 2] if g else None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--shape", default=None, help="nz,ny,nx (default n,n,n)")
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    ap.add_argument("--budget", type=float, default=0, help="device ring budget in bytes (0 = none)")
    ap.add_argument("--c", type=int, default=2)
    ap.add_argument("--S", type=int, default=3)
    ap.add_argument("--policy", type=int, default=1)
    ap.add_argument("--graph", type=int, default=0)
    ap.add_argument("--launches", type=int, default=2)
    ap.add_argument("--persistent", type=int, default=0, help="PP_OPT_PERSISTENT (one resident kernel)")
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    nz, ny, nx = [int(x) for x in a.shape.split(",")] if a.shape else (a.n, a.n, a.n)
    n = nz
    dt = torch.float64 if a.dtype == "f64" else torch.float32
    A0 = torch.empty((nz, ny, nx), dtype=dt, pin_memory=True)
    An = torch.empty_like(A0).pin_memory()
    synth.fill(A0, "random", seed=synth.SEED_A, nx=nx, ny=ny)
    c0 = 1.0 / 6.0 if dt == torch.float64 else float(torch.tensor(1.0, dtype=dt) / 6)
    r = pp.Region(0)
    r.map("to", A0, -1, 3)
    r.map("from", An)
    r.pipeline(a.c, a.S)
    if a.budget:
        r.mem_limit(int(a.budget))
    r.set_option(pp.PP_OPT_STREAM_POLICY, a.policy)
    r.set_option(pp.PP_OPT_GRAPH, a.graph)
    r.set_option(pp.PP_OPT_PERSISTENT, a.persistent)
    for _ in range(2):
        r.launch(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
    lib_ms = []
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
        for _ in range(a.launches):
            r.launch(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
            lib_ms.append(r.query()["last_ms"])
        torch.cuda.synchronize()
    q = r.query()
    r.close()
    out = a.out or os.path.join(ROOT, "gpurun_out", f"cupti_c{a.c}S{a.S}p{a.policy}g{a.graph}.json")
    os.makedirs(os.path.dirname(out), exist_ok=True)
    prof.export_chrome_trace(out)
    with open(out) as f:
        trace = json.load(f)
    evs = trace["traceEvents"] if isinstance(trace, dict) else trace
    ops = []
    for ev in evs:
        k = kind_of(ev)
        if k is None or ev.get("ph") != "X":
            continue
        nb = int(ev.get("args", {}).get("bytes", 0) or 0)
        ops.append((k, float(ev["ts"]), float(ev["ts"]) + float(ev["dur"]), nb))
    ops.sort(key=lambda o: o[1])
    # split into launches: each launch moves exactly q["h2d_bytes"] in; cut at the op where the
    # cumulative H2D bytes cross a multiple of it and the previous launch's last D2H has ended
    per = q["h2d_bytes"]
    launches, cur, hb = [], [], 0
    for o in ops:
        if o[0] == "H2D" and hb >= per and cur:
            launches.append(cur)
            cur, hb = [], 0
        cur.append(o)
        if o[0] == "H2D":
            hb += o[3]
    if cur:
        launches.append(cur)
    for i, ops_i in enumerate(launches):
        st = launch_stats(ops_i)
        st.update({"launch": i, "shape": [nz, ny, nx], "dtype": a.dtype, "c": q["chunk_size"], "S": q["num_streams"],
                   "policy": a.policy, "graph": a.graph, "persistent": a.persistent, "ring_bytes": q["ring_bytes"],
                   "library_ms": lib_ms[i] if i < len(lib_ms) else None,
                   "expected_h2d_bytes": q["h2d_bytes"], "expected_d2h_bytes": q["d2h_bytes"],
                   "source": "CUPTI activity records (torch.profiler / Kineto)", "trace": os.path.relpath(out, ROOT)})
        print(json.dumps(st), flush=True)


if __name__ == "__main__":
    main()
