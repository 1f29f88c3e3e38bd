#!/usr/bin/env python3
"""Host-link copy microbenchmark: where does the per-chunk cost of small pipelined copies come from?

For chunk sizes 2..32 MiB over a 1 GiB pinned host array and an 8-slot device ring:
  same     — one buffer copied repeatedly (what a naive link probe measures)
  stream   — streaming through the host array into ring slots (i % 8), one stream
  duplex   — `stream` H2D on one stream and streaming D2H on another, concurrently
  duplex_ev— as duplex, each copy preceded by cudaStreamWaitEvent on a cross-stream event
  rr3      — H2D round-robin over 3 streams (the paper's per-chunk streams) + D2H likewise
Prints one JSON line per (mode, size): GB/s per direction.
"""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    dev = torch.device("cuda:0")
    GB = 1 << 30
    H = torch.empty(GB, dtype=torch.uint8, pin_memory=True)
    H2 = torch.empty(GB, dtype=torch.uint8, pin_memory=True)
    H.fill_(1)
    H2.fill_(2)
    ring_in = torch.empty(8 * (32 << 20), dtype=torch.uint8, device=dev)
    ring_out = torch.empty(8 * (32 << 20), dtype=torch.uint8, device=dev)
    ring_out.fill_(3)
    s1, s2, s3 = torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream()
    ss = [torch.cuda.Stream() for _ in range(6)]

    def run(mode, sz):
        n = GB // sz
        torch.cuda.synchronize()
        e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        ev = torch.cuda.Event()
        ev.record(s3)
        e[0].record(s1)
        e[2].record(s2)
        for s in ss:
            s.wait_event(e[0])
        for i in range(n):
            slot = i % 8
            hin = H[i * sz:(i + 1) * sz]
            hout = H2[i * sz:(i + 1) * sz]
            din = ring_in[slot * sz:(slot + 1) * sz]
            dout = ring_out[slot * sz:(slot + 1) * sz]
            if mode == "same":
                with torch.cuda.stream(s1):
                    din.copy_(H[:sz], non_blocking=True)
            elif mode == "stream":
                with torch.cuda.stream(s1):
                    din.copy_(hin, non_blocking=True)
            elif mode in ("duplex", "duplex_ev"):
                if mode == "duplex_ev":
                    s1.wait_event(ev)
                    s2.wait_event(ev)
                with torch.cuda.stream(s1):
                    din.copy_(hin, non_blocking=True)
                with torch.cuda.stream(s2):
                    hout.copy_(dout, non_blocking=True)
            elif mode == "rr3":
                with torch.cuda.stream(ss[i % 3]):
                    din.copy_(hin, non_blocking=True)
                with torch.cuda.stream(ss[3 + i % 3]):
                    hout.copy_(dout, non_blocking=True)
        for s in ss:
            ev2 = torch.cuda.Event()
            ev2.record(s)
            s1.wait_event(ev2)
            s2.wait_event(ev2)
        e[1].record(s1)
        e[3].record(s2)
        torch.cuda.synchronize()
        t1 = e[0].elapsed_time(e[1]) * 1e-3
        t2 = e[2].elapsed_time(e[3]) * 1e-3
        return {"mode": mode, "MiB": sz >> 20, "h2d_gbs": GB / t1 / 1e9 if mode != "same" or True else None,
                "d2h_gbs": GB / t2 / 1e9 if mode in ("duplex", "duplex_ev", "rr3") else None,
                "per_copy_us": t1 / n * 1e6}

    for mode in ("same", "stream", "duplex", "duplex_ev", "rr3"):
        for mib in (2, 4, 8, 16, 32):
            run(mode, mib << 20)
            best = max((run(mode, mib << 20) for _ in range(3)), key=lambda r: r["h2d_gbs"])
            print(json.dumps(best), flush=True)


if __name__ == "__main__":
    main()
