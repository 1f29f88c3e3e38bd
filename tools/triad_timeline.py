#!/usr/bin/env python3
"""CUPTI timeline (torch.profiler) of configs[0]'s pipelined triad: where the ~250 us of one launch go.

Prints, per profiled launch, every device op (H2D / kernel / D2H: start, end in us from the launch's
first CUDA runtime call) and the host-side runtime calls (cudaMemcpy*/cudaLaunchKernel/event/stream
calls: count and total us), so the fill, the per-copy gaps and the host enqueue cost can be read off.

usage: python tools/triad_timeline.py [--merge 1] [--graph 0] [--policy 1] [--launches 3]
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


def kind_of(ev):
    name = ev.get("name", "")
    cat = ev.get("cat", "")
    if cat in ("gpu_memcpy", "Memcpy") or name.startswith("Memcpy"):
        return "H2D" if "HtoD" in name else ("D2H" if "DtoH" in name else "CPY")
    if cat == "kernel":
        return "KER"
    if cat == "cuda_runtime" or cat == "cuda_driver":
        return "API"
    return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1 << 20)
    ap.add_argument("--chunks", type=int, default=4)
    ap.add_argument("--S", type=int, default=2)
    ap.add_argument("--policy", type=int, default=1)
    ap.add_argument("--graph", type=int, default=0)
    ap.add_argument("--merge", type=int, default=1)
    ap.add_argument("--launches", type=int, default=3)
    a = ap.parse_args()
    n = a.n
    ab = torch.empty(2 * n, dtype=torch.float32, pin_memory=True)
    A, B = ab[:n], ab[n:]
    C = torch.empty(n, dtype=torch.float32, pin_memory=True)
    synth.fill(A, "random", seed=synth.SEED_A)
    synth.fill(B, "random", seed=synth.SEED_B)
    r = pp.Region(0)
    r.map("to", A)
    r.map("to", B)
    r.map("from", C)
    r.pipeline(n // a.chunks, a.S)
    r.set_option(pp.PP_OPT_STREAM_POLICY, a.policy)
    r.set_option(pp.PP_OPT_GRAPH, a.graph)
    r.set_option(pp.PP_OPT_MERGE_COPIES, a.merge)
    for _ in range(5):
        r.launch(0, n, "triad", s=3.0)
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
        for _ in range(a.launches):
            r.launch(0, n, "triad", s=3.0)
        torch.cuda.synchronize()
    r.close()
    out = os.path.join(ROOT, "gpurun_out", "triad_timeline_trace.json")
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
        ops.append((k, float(ev["ts"]), float(ev["ts"]) + float(ev.get("dur", 0)), ev.get("name", "")[:40],
                    int(ev.get("args", {}).get("bytes", 0) or 0)))
    ops.sort(key=lambda o: o[1])
    # a launch starts at a runtime call that follows the previous launch's last D2H
    dev = [o for o in ops if o[0] != "API"]
    api = [o for o in ops if o[0] == "API"]
    per_launch = len(dev) // a.launches if a.launches else 0
    res = []
    for i in range(a.launches):
        d = dev[i * per_launch:(i + 1) * per_launch]
        if not d:
            continue
        t_prev_end = dev[i * per_launch - 1][2] if i else -1e18
        calls = [x for x in api if t_prev_end < x[1] <= d[-1][2]]
        t0 = calls[0][1] if calls else d[0][1]
        names = {}
        for x in calls:
            nm = x[3]
            c, tot = names.get(nm, (0, 0.0))
            names[nm] = (c + 1, tot + (x[2] - x[1]))
        res.append({"launch": i, "span_us": round(d[-1][2] - t0, 1),
                    "first_device_op_us": round(d[0][1] - t0, 1),
                    "ops": [(k, round(s - t0, 1), round(e - t0, 1), nb) for k, s, e, _, nb in d],
                    "api": {k: (c, round(t, 1)) for k, (c, t) in sorted(names.items(), key=lambda kv: -kv[1][1])}})
    for x in res:
        print(json.dumps(x))


if __name__ == "__main__":
    main()
