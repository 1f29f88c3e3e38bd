#!/usr/bin/env python3
"""NEXT-1 fused-level depth A/B on the configs[1] array: T sweeps per pass with PP_OPT_FUSE = L, the
chunk size / chunks in flight picked by pp_autotune (budget = free HBM); per-pass time, launches, ring
bytes; every output bit-identical across L (and to L = 1).

usage: python tools/temporal_fuse_ab.py [--T 64] [--L 1,2,3,4]
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--T", type=int, default=64)
    ap.add_argument("--L", default="1,2,3,4")
    ap.add_argument("--reps", type=int, default=5)
    a = ap.parse_args()
    n = 512
    A0 = torch.empty((n, n, n), dtype=torch.float64, pin_memory=True)
    synth.fill(A0, "random", seed=synth.SEED_A, nx=n, ny=n)
    ref = None
    for L in [int(x) for x in a.L.split(",")]:
        An = torch.empty_like(A0).pin_memory()
        with pp.Region(0) as r:
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.pipeline(0, 3)
            r.set_option(pp.PP_OPT_SWEEPS, a.T)
            r.set_option(pp.PP_OPT_FUSE, L)
            tune = r.autotune(1, n - 1, "stencil7", trials=4, c0=1 / 6, c1=1 / 36)
            ms = []
            for _ in range(a.reps):
                r.launch(1, n - 1, "stencil7", c0=1 / 6, c1=1 / 36)
                ms.append(r.query()["last_ms"])
            q = r.query()
        if ref is None:
            ref = An.clone()
        same = bool(torch.equal(An[1:n - 1].view(torch.int64), ref[1:n - 1].view(torch.int64)))
        print(json.dumps({"T": a.T, "L": L, "ms_best": min(ms), "ms_median": sorted(ms)[len(ms) // 2],
                          "chunk": q["chunk_size"], "streams": q["num_streams"], "graph": tune["graph"],
                          "launches": q["n_kernels"], "ring_bytes": q["ring_bytes"], "identical": same}), flush=True)


if __name__ == "__main__":
    main()
