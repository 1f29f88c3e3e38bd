#!/usr/bin/env python3
"""Interleaved timing of the configs[1] headline schedule (c = 6, one chunk in flight, per-stage
streams) and the literal c = 2, S = 3 schedule; run under different PP_* environment settings."""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ipps_cuissf17_b200 as pp  # noqa: E402
import synth  # noqa: E402


def main():
    n = 512
    A0 = torch.empty((n, n, n), dtype=torch.float64, pin_memory=True)
    An = torch.empty_like(A0).pin_memory()
    synth.fill(A0, "random", seed=synth.SEED_A, nx=n, ny=n)
    c0 = 1.0 / 6.0
    regs = []
    for c, S in ((6, 1), (2, 3)):
        r = pp.Region(0)
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(c, S)
        r.launch(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
        regs.append((c, S, r, []))
    for _ in range(10):
        for c, S, r, t in regs:
            r.launch(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
            t.append(r.query()["last_ms"])
    env = {k: v for k, v in os.environ.items() if k.startswith("PP_")}
    for c, S, r, t in regs:
        print(json.dumps({"env": env, "c": c, "S": S, "median_ms": statistics.median(t), "min_ms": min(t)}))
        r.close()


if __name__ == "__main__":
    main()
