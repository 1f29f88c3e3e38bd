#!/usr/bin/env python3
"""Device-side cost of T Jacobi sweeps of the 512^3 stencil with PP_OPT_FUSE = L levels per kernel pass
(pp_naive's T-sweep baseline: whole arrays resident in HBM, ceil(T/L) launches ping-ponging two device
arrays; the kernel phase is timed with CUDA events). Effective GB/s = T x the single-sweep algorithmic
bytes ((iters+2) + iters planes) per second of kernel time, i.e. what T unfused sweeps would have to
move to match.

usage: python tools/fuse_probe.py [--n 512] [--dtype f64] [--T 12] [--fuse 1,2,3,4] [--reps 5]
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
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--dtype", default="f64")
    ap.add_argument("--T", type=int, default=12)
    ap.add_argument("--fuse", default="1,2,3,4")
    ap.add_argument("--reps", type=int, default=5)
    a = ap.parse_args()
    n = a.n
    dt = torch.float64 if a.dtype == "f64" else torch.float32
    es = 8 if a.dtype == "f64" else 4
    A0 = torch.empty((n, n, n), dtype=dt, pin_memory=True)
    An = torch.empty_like(A0).pin_memory()
    synth.fill(A0, "random", seed=synth.SEED_A, nx=n, ny=n)
    c0 = 1.0 / 6.0
    sweep_bytes = (2 * n - 2) * n * n * es
    for L in [int(x) for x in a.fuse.split(",")]:
        with pp.Region(0) as r:
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.set_option(pp.PP_OPT_SWEEPS, a.T)
            r.set_option(pp.PP_OPT_FUSE, L)
            r.naive(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
            ks = []
            for _ in range(a.reps):
                r.naive(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
                ks.append(r.query()["naive_kernel_ms"])
            launches = r.query()["n_kernels"]
        best = min(ks)
        print(json.dumps({"dtype": a.dtype, "n": n, "T": a.T, "fuse": L, "launches": launches,
                          "variant": os.environ.get("PP_FUSE_VARIANT", "default"),
                          "kernel_ms": best, "ms_per_sweep": best / a.T,
                          "effective_gbs": a.T * sweep_bytes / (best * 1e-3) / 1e9,
                          "sweeps_per_s": a.T / (best * 1e-3)}), flush=True)


if __name__ == "__main__":
    main()
