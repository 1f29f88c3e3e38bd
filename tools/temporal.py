#!/usr/bin/env python3
"""Multi-sweep temporal blocking on the 512^3 fp64 stencil: T Jacobi sweeps
streamed through the host link once (PP_OPT_SWEEPS = T) vs T separate pipelined sweeps vs the naive
offload of T sweeps (copy in, T kernels, copy out). One JSON line per T: ms, sweeps/s, the effective
link-equivalent GB/s (T x the bytes a single sweep moves, per second), device ring bytes."""
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
    ap.add_argument("--chunk", type=int, default=8)
    ap.add_argument("--streams", type=int, default=2)
    ap.add_argument("--Ts", default="1,2,4,8,16,32")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--graph", type=int, default=0)
    ap.add_argument("--fuse", type=int, default=1)
    ap.add_argument("--no-naive", action="store_true")
    a = ap.parse_args()
    n = a.n
    A0 = torch.empty((n, n, n), dtype=torch.float64, pin_memory=True)
    An = torch.empty_like(A0).pin_memory()
    synth.fill(A0, "random", seed=synth.SEED_A, nx=n, ny=n)
    c0 = 1.0 / 6.0
    single = None
    for T in [int(x) for x in a.Ts.split(",")]:
        with pp.Region(0) as r:
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.pipeline(a.chunk, a.streams)
            r.set_option(pp.PP_OPT_SWEEPS, T)
            r.set_option(pp.PP_OPT_GRAPH, a.graph)
            r.set_option(pp.PP_OPT_FUSE, min(a.fuse, T))
            r.launch(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
            ms = []
            for _ in range(a.reps):
                r.launch(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
                ms.append(r.query()["last_ms"])
            q = r.query()
            nv = [float("nan")]
            if not a.no_naive:
                r.naive(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
                nv = []
                for _ in range(a.reps):
                    r.naive(1, n - 1, "stencil7", c0=c0, c1=c0 / 6)
                    nv.append(r.query()["last_ms"])
        best = min(ms)
        if T == 1:
            single = best
        byt = q["h2d_bytes"] + q["d2h_bytes"]
        print(json.dumps({"T": T, "fuse": a.fuse, "graph": a.graph, "replayed": q["graph_replayed"], "chunk": q["chunk_size"], "streams": q["num_streams"], "ms": best,
                          "sweeps_per_s": T / (best * 1e-3), "effective_gbs": T * byt / (best * 1e-3) / 1e9,
                          "link_gbs": byt / (best * 1e-3) / 1e9, "ring_bytes": q["ring_bytes"],
                          "kernels": q["n_kernels"], "T_separate_sweeps_ms": T * single if single else None,
                          "speedup_vs_T_separate": (T * single / best) if single else None,
                          "naive_T_sweeps_ms": min(nv), "speedup_vs_naive": min(nv) / best}), flush=True)


if __name__ == "__main__":
    main()
