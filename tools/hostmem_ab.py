#!/usr/bin/env python3
"""configs[1] end to end (512^3 fp64 stencil, c = 6, S = 1, 28 MiB ring) from host arrays of three
kinds, interleaved: torch pinned (cudaHostAlloc), 2 MiB-page anonymous memory page-locked in place
(hostmem.alloc_host + cudaHostRegister through pp_map), and 4 KiB-page anonymous memory page-locked in
place. Does the host page size change the copy engines' per-copy cost? CUDA events, median of --reps.

usage: python tools/hostmem_ab.py [--reps 15] [--rounds 2]
"""
import argparse
import json
import mmap
import os
import statistics
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_cuissf17_b200 as pp  # noqa: E402
import synth  # noqa: E402
from paper_conf_ipps_cuissf17_b200 import hostmem  # noqa: E402


def small_pages(shape):
    n = int(np.prod(shape)) * 8
    m = mmap.mmap(-1, n, flags=mmap.MAP_PRIVATE | mmap.MAP_ANONYMOUS)
    try:
        m.madvise(mmap.MADV_NOHUGEPAGE)
    except (AttributeError, OSError):
        pass
    return np.frombuffer(m, dtype=np.float64).reshape(shape)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=15)
    ap.add_argument("--rounds", type=int, default=2)
    ap.add_argument("--c", type=int, default=6)
    a = ap.parse_args()
    n = 512
    shape = (n, n, n)
    kinds = {
        "torch_pinned": lambda: torch.empty(shape, dtype=torch.float64, pin_memory=True).numpy(),
        "hugepage_registered": lambda: hostmem.alloc_host(shape, np.float64),
        "4k_registered": lambda: small_pages(shape),
    }
    arrays = {}
    for k, f in kinds.items():
        A0, An = f(), f()
        synth.fill(A0, "random", seed=synth.SEED_A, nx=n, ny=n)
        An[:] = 0
        arrays[k] = (A0, An)
    c0, c1 = 1.0 / 6.0, 1.0 / 36.0
    for rnd in range(a.rounds):
        for k, (A0, An) in arrays.items():
            with pp.Region(0) as r:
                r.map("to", A0, -1, 3)
                r.map("from", An)
                r.pipeline(a.c, 1)
                r.mem_limit(28 << 20)
                r.launch(1, n - 1, "stencil7", c0=c0, c1=c1)
                ts = []
                for _ in range(a.reps):
                    e0 = torch.cuda.Event(enable_timing=True)
                    e1 = torch.cuda.Event(enable_timing=True)
                    e0.record()
                    r.launch(1, n - 1, "stencil7", c0=c0, c1=c1)
                    e1.record()
                    torch.cuda.synchronize()
                    ts.append(e0.elapsed_time(e1))
                q = r.query()
            print(json.dumps({"round": rnd, "host": k, "median_ms": statistics.median(ts), "min_ms": min(ts),
                              "pinned_by_map": bool(q["pinned"][0]), "ring_planes": q["ring_planes"][:2]}), flush=True)


if __name__ == "__main__":
    main()
