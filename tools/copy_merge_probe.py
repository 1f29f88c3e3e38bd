#!/usr/bin/env python3
"""Does one 2-D copy of two equally spaced 1 MiB pieces cost less than two 1 MiB copies? (configs[0]
triad: a and b of a chunk are two H2D copies.) Times, on one stream each direction, the H2D of
4 chunks x 2 arrays as 8 copies vs 4 cudaMemcpy2DAsync (height 2), with and without a concurrent D2H
of 4 x 1 MiB; also 4 contiguous 2 MiB copies for scale. CUDA events, best of --reps.

usage: python tools/copy_merge_probe.py [--piece-mib 1] [--reps 30]
"""
import argparse
import json

import torch
from cuda.bindings import runtime as rt


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--piece-mib", type=float, default=1.0)
    ap.add_argument("--chunks", type=int, default=4)
    ap.add_argument("--reps", type=int, default=30)
    a = ap.parse_args()
    piece = int(a.piece_mib * (1 << 20))
    n = a.chunks
    arr = n * piece                                  # one array's bytes
    host = torch.empty(3 * arr, dtype=torch.uint8, pin_memory=True)   # a | b | c
    dev = torch.empty(3 * arr, dtype=torch.uint8, device="cuda")
    hp, dp = host.data_ptr(), dev.data_ptr()
    s_in = torch.cuda.Stream()
    s_out = torch.cuda.Stream()
    H2D, D2H = rt.cudaMemcpyKind.cudaMemcpyHostToDevice, rt.cudaMemcpyKind.cudaMemcpyDeviceToHost

    def h2d_separate():
        for j in range(n):
            for k in range(2):
                rt.cudaMemcpyAsync(dp + k * arr + j * piece, hp + k * arr + j * piece, piece, H2D, s_in.cuda_stream)

    def h2d_2d():
        for j in range(n):
            rt.cudaMemcpy2DAsync(dp + j * piece, arr, hp + j * piece, arr, piece, 2, H2D, s_in.cuda_stream)

    def h2d_contig():
        for j in range(n):
            rt.cudaMemcpyAsync(dp + 2 * j * piece, hp + 2 * j * piece, 2 * piece, H2D, s_in.cuda_stream)

    def d2h():
        for j in range(n):
            rt.cudaMemcpyAsync(hp + 2 * arr + j * piece, dp + 2 * arr + j * piece, piece, D2H, s_out.cuda_stream)

    def timed(fn, with_d2h):
        best = 1e9
        for _ in range(a.reps):
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(s_in)
            s_out.wait_event(e0)
            fn()
            if with_d2h:
                d2h()
            s_in.wait_stream(s_out)
            e1.record(s_in)
            torch.cuda.synchronize()
            best = min(best, e0.elapsed_time(e1) * 1e3)
        return best

    for with_d2h in (False, True):
        rec = {"piece_bytes": piece, "chunks": n, "with_d2h": with_d2h}
        for name, fn in (("separate_8", h2d_separate), ("merged_2d_4", h2d_2d), ("contiguous_4", h2d_contig)):
            rec[name + "_us"] = timed(fn, with_d2h)
        print(json.dumps(rec), flush=True)


if __name__ == "__main__":
    main()
