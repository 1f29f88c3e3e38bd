#!/usr/bin/env python3
"""Chunk-size x stream-count x buffer-budget sweep on the 512^3 fp64 stencil vs the naive offload
(BASELINE.json configs[4]; the paper's Figs. 4, 7, 8 axes on synthetic data). One JSON line per cell:
e2e GB/s, ms, speedup vs naive, ring (device) bytes and HBM saved, resolved chunk/streams.

usage: python tools/sweep.py [--n 512] [--dtype f64] [--reps 3] [--quick] > gpurun_out/sweep.jsonl
"""
import argparse
import itertools
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_ipps_cuissf17_b200 as pp  # noqa: E402
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--dtype", default="f64")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--chunks", default="1,2,4,8,16,32,64,128,510")
    ap.add_argument("--streams", default="1,2,3,4,6,8")
    ap.add_argument("--policies", default="0,1")
    ap.add_argument("--graphs", default="0,1")
    ap.add_argument("--budgets", default="full-overlap")
    ap.add_argument("--persistent", default="0", help="PP_OPT_PERSISTENT values to sweep (0,1)")
    a = ap.parse_args()
    n = a.n
    dt = torch.float64 if a.dtype == "f64" else torch.float32
    es = 8 if a.dtype == "f64" else 4
    plane = n * n * es
    A0 = torch.empty((n, n, n), dtype=dt, pin_memory=True)
    An = torch.empty((n, n, n), dtype=dt, pin_memory=True)
    synth.fill(A0, "random", seed=synth.SEED_A, nx=n, ny=n)
    c0 = 1.0 / 6.0
    c1 = c0 / 6.0
    lo, hi = 1, n - 1

    def timeit(fn, reps):
        fn()
        torch.cuda.synchronize()
        t = []
        for _ in range(reps):
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            e1.record()
            torch.cuda.synchronize()
            t.append(e0.elapsed_time(e1))
        return sorted(t)[len(t) // 2]

    link = pp.pp_probe_link(0, 256 << 20, 5)
    print(json.dumps({"link": link}), flush=True)
    with pp.Region(0) as rn:
        rn.map("to", A0, -1, 3)
        rn.map("from", An)
        t_naive = timeit(lambda: rn.naive(lo, hi, "stencil7", c0=c0, c1=c1), a.reps)
        qn = rn.query()
    print(json.dumps({"naive_ms": t_naive, "naive_bytes": qn["naive_bytes"],
                      "phase_ms": [qn["naive_h2d_ms"], qn["naive_kernel_ms"], qn["naive_d2h_ms"]]}), flush=True)
    chunks = [int(x) for x in a.chunks.split(",")]
    streams = [int(x) for x in a.streams.split(",")]
    policies = [int(x) for x in a.policies.split(",")]
    graphs = [int(x) for x in a.graphs.split(",")]
    budgets = a.budgets.split(",")
    persist = [int(x) for x in a.persistent.split(",")]
    if a.quick:
        chunks, streams = [1, 2, 4, 8, 16], [2, 3, 4]
    for c, S, pol, g, b, pe in itertools.product(chunks, streams, policies, graphs, budgets, persist):
        if pe and g:
            continue                               # the persistent kernel is not graph-captured
        with pp.Region(0) as r:
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.pipeline(c, S)
            r.set_option(pp.PP_OPT_STREAM_POLICY, pol)
            r.set_option(pp.PP_OPT_GRAPH, g)
            r.set_option(pp.PP_OPT_PERSISTENT, pe)
            if b == "min":
                r.set_option(pp.PP_OPT_RING_EXTRA, 0)
            elif b.startswith("planes"):
                r.mem_limit(int(b[6:]) * plane)
            t0 = time.perf_counter()
            ms = timeit(lambda: r.launch(lo, hi, "stencil7", c0=c0, c1=c1), a.reps)
            q = r.query()
        byt = q["h2d_bytes"] + q["d2h_bytes"]
        print(json.dumps({"c": c, "S": S, "policy": pol, "graph": g, "persistent": pe, "budget": b, "ms": ms,
                          "e2e_gbs": byt / (ms * 1e-3) / 1e9, "speedup": t_naive / ms,
                          "chunk": q["chunk_size"], "streams": q["num_streams"], "nchunks": q["nchunks"],
                          "ring_bytes": q["ring_bytes"], "hbm_saved": 1 - q["ring_bytes"] / qn["naive_bytes"],
                          "ring_planes": q["ring_planes"], "wall_s": time.perf_counter() - t0}), flush=True)


if __name__ == "__main__":
    main()
