#!/usr/bin/env python3
"""2-D block regions (the paper's matmul-style non-contiguous transfers,
P:L376-385): triad c = a + s*b over [R][C] fp32 arrays pipelined along the COLUMN
dimension (split_dim = 1: each chunk is a column block of R rows, moved with cudaMemcpy2DAsync into
pitched [R][ring][block] rings) against the same arrays split along rows (contiguous 1-D copies),
same bytes, same chunk bytes. Prints one JSON line per case: ms, GB/s over the link, copies issued.

usage: python tools/block2d_probe.py [--rows 4096] [--cols 65536] [--chunk-mib 16] [--streams 3]
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
    ap.add_argument("--rows", type=int, default=4096)
    ap.add_argument("--cols", type=int, default=65536)
    ap.add_argument("--chunk-mib", type=float, default=16)
    ap.add_argument("--streams", type=int, default=3)
    ap.add_argument("--reps", type=int, default=7)
    a = ap.parse_args()
    R, C = a.rows, a.cols
    arrs = []
    for seed in (synth.SEED_A, synth.SEED_B):
        t = torch.empty((R, C), dtype=torch.float32, pin_memory=True)
        synth.fill(t, "random", seed=seed, nx=C, ny=R)
        arrs.append(t)
    out = torch.empty((R, C), dtype=torch.float32, pin_memory=True)
    chunk_bytes = a.chunk_mib * (1 << 20)
    cases = [("row blocks (split_dim 0, contiguous copies)", 0, max(1, int(chunk_bytes // (C * 4))), R),
             ("column blocks (split_dim 1, cudaMemcpy2DAsync)", 1, max(1, int(chunk_bytes // (R * 4))), C)]
    res = []
    for name, dim, c, n in cases:
        with pp.Region(0) as r:
            r.map("to", arrs[0], split_dim=dim)
            r.map("to", arrs[1], split_dim=dim)
            r.map("from", out, split_dim=dim)
            r.pipeline(c, a.streams)
            r.launch(0, n, "triad", s=3.0)
            ts = []
            for _ in range(a.reps):
                r.launch(0, n, "triad", s=3.0)
                ts.append(r.query()["last_ms"])
            q = r.query()
        ms = statistics.median(ts)
        res.append({"case": name, "rows": R, "cols": C, "chunk": c, "streams": a.streams, "nchunks": q["nchunks"],
                    "copies": q["n_h2d"] + q["n_d2h"], "ring_bytes": q["ring_bytes"], "ms": ms, "min_ms": min(ts),
                    "gbs": (q["h2d_bytes"] + q["d2h_bytes"]) / (ms * 1e-3) / 1e9})
    for x in res:
        print(json.dumps(x), flush=True)


if __name__ == "__main__":
    main()
