#!/usr/bin/env python3
"""Row a4 (pageable host arrays): configs[1] (512^3 fp64 stencil) from PAGEABLE host arrays (numpy,
4 KiB pages) through the four host-memory paths, against pinned (cudaHostAlloc) arrays:
  register  PP_OPT_AUTO_PIN = 1: cudaHostRegister in place at pp_map (its time reported apart)
  driver    PP_OPT_AUTO_PIN = 0, PP_OPT_BOUNCE = 0: the CUDA driver's pageable copies
  bounce    PP_OPT_AUTO_PIN = 0, PP_OPT_BOUNCE = 1: the library's pinned bounce ring + host workers
  pinned    torch pinned tensors (the paper's cudaHostAlloc)
Schedules: the bench's headline (c = 6, one chunk in flight, 28 MiB ring) and c = 16, S = 3. Every
output is checked bit for bit against the pinned run. One JSON line per (mode, schedule).

usage: python tools/pageable_ab.py [--reps 5]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_cuissf17_b200 as pp  # noqa: E402
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--n", type=int, default=512)
    a = ap.parse_args()
    n = a.n
    c0 = 1.0 / 6.0
    c1 = c0 / 6.0
    A_pin = torch.empty((n, n, n), dtype=torch.float64, pin_memory=True)
    synth.fill(A_pin, "random", seed=synth.SEED_A, nx=n, ny=n)
    ref = None
    for sched in ((6, 1), (16, 3)):
        for mode in ("pinned", "register", "driver", "bounce", "bounce4", "bounce15"):
            if mode == "pinned":
                A, B = A_pin, torch.empty_like(A_pin).pin_memory()
            else:
                A = np.empty((n, n, n), dtype=np.float64)
                A[...] = A_pin.numpy()
                B = np.empty_like(A)
            t = time.perf_counter()
            with pp.Region(0) as r:
                r.set_option(pp.PP_OPT_AUTO_PIN, 1 if mode == "register" else 0)
                r.set_option(pp.PP_OPT_BOUNCE, {"bounce": 1, "bounce4": 4, "bounce15": 15}.get(mode, 0))
                r.map("to", A, -1, 3)
                r.map("from", B)
                map_s = time.perf_counter() - t
                r.pipeline(*sched)
                r.set_option(pp.PP_OPT_STREAM_POLICY, 1)
                r.launch(1, n - 1, "stencil7", c0=c0, c1=c1)
                ms = []
                for _ in range(a.reps):
                    t = time.perf_counter()
                    r.launch(1, n - 1, "stencil7", c0=c0, c1=c1)
                    ms.append((time.perf_counter() - t) * 1e3)
                q = r.query()
            out = B.numpy() if isinstance(B, torch.Tensor) else B
            if ref is None:
                ref = out.copy()
            same = bool(np.array_equal(out[1:n - 1].view(np.uint64), ref[1:n - 1].view(np.uint64)))
            print(json.dumps({"mode": mode, "chunk": q["chunk_size"], "streams": q["num_streams"],
                              "pinned": q["pinned"], "map_s": map_s, "ms_best": min(ms),
                              "ms_median": sorted(ms)[len(ms) // 2],
                              "gbs": (q["h2d_bytes"] + q["d2h_bytes"]) / (min(ms) * 1e-3) / 1e9,
                              "bit_identical_to_pinned": same}), flush=True)


if __name__ == "__main__":
    main()
