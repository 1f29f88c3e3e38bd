#!/usr/bin/env python3
"""Interleaved A/B at configs[1] (512^3 fp64, c = 6, one chunk in flight, 28 MiB ring): host arrays
from torch.pin_memory (cudaHostAlloc) against anonymous mappings advised for 2 MiB transparent huge
pages and page-locked by pp_map (cudaHostRegister; hostmem.alloc_host). Prints median/min ms."""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_cuissf17_b200 as pp  # noqa: E402
from paper_conf_ipps_cuissf17_b200 import hostmem  # noqa: E402
import synth  # noqa: E402


def main():
    n = 512
    reps = int(sys.argv[1]) if len(sys.argv) > 1 else 12
    scheds = [(6, 1), (2, 3)]
    arrays = {}
    A = hostmem.alloc_host((n, n, n), np.float64)
    B = hostmem.alloc_host((n, n, n), np.float64)
    synth.fill(A, "random", seed=synth.SEED_A, nx=n, ny=n)
    B[:] = 0
    arrays["thp+register"] = (A, B)
    tA = torch.empty((n, n, n), dtype=torch.float64, pin_memory=True)
    tB = torch.zeros_like(tA).pin_memory()
    synth.fill(tA, "random", seed=synth.SEED_A, nx=n, ny=n)
    arrays["torch pin_memory"] = (tA, tB)
    c0 = 1.0 / 6.0
    regs = []
    for name, (x, y) in arrays.items():
        for c, S in scheds:
            r = pp.Region(0)
            r.map("to", x, -1, 3)
            r.map("from", y)
            r.pipeline(c, S)
            r.launch(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
            regs.append((name, c, S, r, []))
    for rep in range(reps):
        for name, c, S, r, t in regs[rep % len(regs):] + regs[:rep % len(regs)]:
            r.launch(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
            t.append(r.query()["last_ms"])
    for name, c, S, r, t in regs:
        print(json.dumps({"host": name, "c": c, "S": S, "median_ms": statistics.median(t), "min_ms": min(t)}), flush=True)
        r.close()


if __name__ == "__main__":
    main()
