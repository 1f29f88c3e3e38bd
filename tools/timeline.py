#!/usr/bin/env python3
"""Copy/compute overlap timeline of one pipelined launch (nsys is not in this image: the library's
PP_OPT_TRACE records a CUDA timing event before and after every op on the op's own stream).

Writes a Chrome-trace JSON (open in chrome://tracing or Perfetto) and prints overlap statistics:
H2D-busy, D2H-busy, both-busy fractions of the launch, kernel time nested inside copy-busy time,
and the idle gaps of each copy direction.

usage: python tools/timeline.py --c 2 --S 3 --policy 0 --out profiles/r1_timeline_c2S3.json
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_cuissf17_b200 as pp  # noqa: E402
import synth  # noqa: E402


def union(iv):
    iv = sorted(iv)
    out = []
    for a, b in iv:
        if out and a <= out[-1][1]:
            out[-1][1] = max(out[-1][1], b)
        else:
            out.append([a, b])
    return out


def length(iv):
    return sum(b - a for a, b in iv)


def intersect(x, y):
    i = j = 0
    out = []
    while i < len(x) and j < len(y):
        a = max(x[i][0], y[j][0])
        b = min(x[i][1], y[j][1])
        if a < b:
            out.append([a, b])
        if x[i][1] < y[j][1]:
            i += 1
        else:
            j += 1
    return out


def stats(recs, total_ms):
    h = union([(r["start_ms"], r["end_ms"]) for r in recs if r["kind"] == "H2D"])
    d = union([(r["start_ms"], r["end_ms"]) for r in recs if r["kind"] == "D2H"])
    k = union([(r["start_ms"], r["end_ms"]) for r in recs if r["kind"] == "KER"])
    cp = union(h + d)
    both = intersect(h, d)
    hb = sum(r["bytes"] for r in recs if r["kind"] == "H2D")
    db = sum(r["bytes"] for r in recs if r["kind"] == "D2H")
    gaps_h = [h[i + 1][0] - h[i][1] for i in range(len(h) - 1)]
    gaps_d = [d[i + 1][0] - d[i][1] for i in range(len(d) - 1)]
    return {"launch_ms": total_ms, "h2d_busy_frac": length(h) / total_ms, "d2h_busy_frac": length(d) / total_ms,
            "both_busy_frac": length(both) / total_ms, "kernel_ms": length(k),
            "kernel_inside_copy_frac": length(intersect(k, cp)) / max(1e-9, length(k)),
            "h2d_gbs_while_busy": hb / (length(h) * 1e-3) / 1e9 if h else None,
            "d2h_gbs_while_busy": db / (length(d) * 1e-3) / 1e9 if d else None,
            "h2d_gap_ms": sum(gaps_h), "d2h_gap_ms": sum(gaps_d),
            "first_d2h_start_ms": d[0][0] if d else None, "last_h2d_end_ms": h[-1][1] if h else None}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--c", type=int, default=2)
    ap.add_argument("--S", type=int, default=3)
    ap.add_argument("--policy", type=int, default=0)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    n = a.n
    A0 = torch.empty((n, n, n), dtype=torch.float64, pin_memory=True)
    An = torch.empty_like(A0).pin_memory()
    synth.fill(A0, "random", seed=synth.SEED_A, nx=n, ny=n)
    c0 = 1.0 / 6.0
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(a.c, a.S)
        r.set_option(pp.PP_OPT_STREAM_POLICY, a.policy)
        r.launch(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)          # warm
        r.set_option(pp.PP_OPT_TRACE, 1)
        r.launch(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
        recs = r.trace()
        q = r.query()
    st = stats(recs, q["last_ms"])
    st.update({"c": a.c, "S": a.S, "policy": a.policy, "ring_planes": q["ring_planes"], "nchunks": q["nchunks"]})
    print(json.dumps(st))
    if a.out:
        ev = []
        lanes = {"H2D": 1, "KER": 2, "D2H": 3}
        for t in recs:
            ev.append({"name": f"{t['kind']} j{t['chunk']} [{t['p0']},{t['p1']})", "ph": "X", "pid": 0,
                       "tid": lanes[t["kind"]] * 100 + t["stream"], "ts": t["start_ms"] * 1e3,
                       "dur": (t["end_ms"] - t["start_ms"]) * 1e3, "args": {"bytes": t["bytes"]}})
        json.dump({"traceEvents": ev, "otherData": st}, open(a.out, "w"))


if __name__ == "__main__":
    main()
