#!/usr/bin/env python3
"""Per-launch cost of the stencil kernels on resident (HBM) arrays, by chunk size and kernel path,
with the op trace giving each kernel's device interval.

usage: python tools/kernel_probe.py [--n 512] [--dtype f64]
"""
import argparse
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
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=512)
    ap.add_argument("--dtype", default="f64")
    ap.add_argument("--paths", default="tma,generic")
    ap.add_argument("--chunks", default="510,64,16,8,4,2,1")
    ap.add_argument("--kernel", default="stencil7", choices=["stencil7", "conv3d"])
    a = ap.parse_args()
    n = a.n
    dt = torch.float64 if a.dtype == "f64" else torch.float32
    es = 8 if a.dtype == "f64" else 4
    A0 = torch.empty((n, n, n), dtype=dt, pin_memory=True)
    synth.fill(A0, "random", seed=synth.SEED_A, nx=n, ny=n)
    dA = A0.cuda()
    dN = torch.empty_like(dA)
    c0 = 1.0 / 6.0
    plane = n * n * es
    paths = [{"tma": pp.KPATH_TMA, "generic": pp.KPATH_GENERIC}[x] for x in a.paths.split(",")]
    for path in paths:
        for c in [int(x) for x in a.chunks.split(",")]:
            with pp.Region(0) as r:
                r.map("to", dA, -1, 3)
                r.map("from", dN)
                r.pipeline(c, 1)
                r.set_option(pp.PP_OPT_KERNEL_PATH, path)
                kargs = {"c0": c0, "c1": c0 / 6} if a.kernel == "stencil7" else {}
                for _ in range(3):
                    r.launch(1, n - 1, a.kernel, **kargs)
                ms = []
                for _ in range(5):
                    r.launch(1, n - 1, a.kernel, **kargs)
                    ms.append(r.query()["last_ms"])
                r.set_option(pp.PP_OPT_TRACE, 1)
                r.launch(1, n - 1, a.kernel, **kargs)
                tr = [t for t in r.trace() if t["kind"] == "KER"]
            durs = [t["end_ms"] - t["start_ms"] for t in tr]
            gaps = [tr[i + 1]["start_ms"] - tr[i]["end_ms"] for i in range(len(tr) - 1)]
            byts = (n + (n - 2)) * plane
            best = min(ms)
            print(json.dumps({"kernel": a.kernel, "path": "tma" if path == pp.KPATH_TMA else "generic", "c": c,
                              "variant": os.environ.get("PP_TMA_VARIANT", "default"), "launches": len(tr),
                              "total_ms": best, "gbs": byts / (best * 1e-3) / 1e9,
                              "kernel_us_median": statistics.median(durs) * 1e3,
                              "kernel_us_max": max(durs) * 1e3,
                              "gap_us_median": statistics.median(gaps) * 1e3 if gaps else None}), flush=True)


if __name__ == "__main__":
    main()
