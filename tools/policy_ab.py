#!/usr/bin/env python3
"""Interleaved A/B of schedules at the configs[1] workload (512^3 fp64): every rep runs each schedule
once, in rotating order, so box-to-box and drift effects hit all alike. Prints median/min ms.

usage: policy_ab.py [reps] [c:S:policy[:graph[:ring_extra[:mirror]]]] ...]"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ipps_cuissf17_b200 as pp  # noqa: E402
import synth  # noqa: E402

SCHEDS = [(2, 3, 0), (2, 3, 1), (2, 3, 2), (2, 3, 3), (2, 3, 4), (6, 1, 1), (3, 2, 1), (3, 2, 3), (4, 1, 1)]


def parse(spec):
    f = [int(x) for x in spec.split(":")]
    return (f + [0, -1, 1][len(f) - 3:])[:6]


def main():
    reps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
    scheds = [parse(s) for s in sys.argv[2:]] or [list(s) + [0, -1, 1] for s in SCHEDS]
    n = 512
    A0 = torch.empty((n, n, n), dtype=torch.float64, pin_memory=True)
    An = torch.empty_like(A0).pin_memory()
    synth.fill(A0, "random", seed=synth.SEED_A, nx=n, ny=n)
    c0 = 1.0 / 6.0
    regions = []
    for c, S, pol, graph, extra, mirror in scheds:
        r = pp.Region(0)
        r.set_option(pp.PP_OPT_MIRROR, mirror)
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(c, S)
        r.set_option(pp.PP_OPT_STREAM_POLICY, pol)
        r.set_option(pp.PP_OPT_GRAPH, graph)
        r.set_option(pp.PP_OPT_RING_EXTRA, extra)
        r.launch(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
        regions.append(r)
    times = [[] for _ in scheds]
    for rep in range(reps):
        order = list(range(len(scheds)))
        order = order[rep % len(order):] + order[:rep % len(order)]
        for i in order:
            regions[i].launch(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
            times[i].append(regions[i].query()["last_ms"])
    for (c, S, pol, graph, extra, mirror), t, r in zip(scheds, times, regions):
        q = r.query()
        print(json.dumps({"c": c, "S": S, "policy": pol, "graph": graph, "ring_extra": extra, "mirror": mirror,
                          "n_h2d": q["n_h2d"], "n_d2h": q["n_d2h"],
                          "ring_planes": q["ring_planes"], "ring_bytes": q["ring_bytes"],
                          "median_ms": statistics.median(t), "min_ms": min(t), "max_ms": max(t)}),
              flush=True)
        r.close()


if __name__ == "__main__":
    main()
