#!/usr/bin/env python3
"""Cost of cross-stream signalling between pipelined 4 MiB copies (what the scheduler pays per chunk).

Modes (1 GiB streamed each way in `--mib` copies, 8-slot rings):
  free      — H2D stream and D2H stream independent (the duplex floor)
  rec       — free + cudaEventRecord after every copy (no one waits)
  chain     — D2H(j) waits an event recorded after H2D(j)
  chain_k   — H2D(j) -> event -> tiny kernel on a 3rd stream -> event -> D2H(j)
  chain_k3  — chain_k, and H2D(j) also waits the kernel of chunk j-3 (ring slot reuse, as pp does)
  fifo_k    — H2D(j) and kernel(j) FIFO on one stream, D2H(j) waits the kernel's event
Prints per-mode total ms and per-direction GB/s.
"""
import argparse
import json

import torch


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--mib", type=int, default=4)
    a = ap.parse_args()
    sz = a.mib << 20
    GB = 1 << 30
    n = GB // sz
    H = torch.empty(GB, dtype=torch.uint8, pin_memory=True)
    H2 = torch.empty(GB, dtype=torch.uint8, pin_memory=True)
    ring_in = torch.empty(8 * sz, dtype=torch.uint8, device="cuda")
    ring_out = torch.zeros(8 * sz, dtype=torch.uint8, device="cuda")
    tiny = torch.zeros(1024, device="cuda")
    sh, sk, sd = torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream()

    def run(mode):
        torch.cuda.synchronize()
        t0 = torch.cuda.Event(enable_timing=True)
        t1 = torch.cuda.Event(enable_timing=True)
        t0.record(sh)
        sk.wait_event(t0)
        sd.wait_event(t0)
        kev = []
        for j in range(n):
            s = j % 8
            hin, hout = H[j * sz:(j + 1) * sz], H2[j * sz:(j + 1) * sz]
            din, dout = ring_in[s * sz:(s + 1) * sz], ring_out[s * sz:(s + 1) * sz]
            if mode == "chain_k3" and j >= 3:
                sh.wait_event(kev[j - 3])
            with torch.cuda.stream(sh):
                din.copy_(hin, non_blocking=True)
                if mode == "fifo_k":
                    tiny.add_(1.0)
            e_h = torch.cuda.Event()
            if mode != "free":
                e_h.record(sh)
            if mode in ("chain_k", "chain_k3"):
                sk.wait_event(e_h)
                with torch.cuda.stream(sk):
                    tiny.add_(1.0)
                e_k = torch.cuda.Event()
                e_k.record(sk)
                kev.append(e_k)
                sd.wait_event(e_k)
            elif mode in ("chain", "fifo_k"):
                sd.wait_event(e_h)
            with torch.cuda.stream(sd):
                hout.copy_(dout, non_blocking=True)
            if mode == "rec":
                torch.cuda.Event().record(sd)
        e = torch.cuda.Event()
        e.record(sd)
        sh.wait_event(e)
        e2 = torch.cuda.Event()
        e2.record(sk)
        sh.wait_event(e2)
        t1.record(sh)
        torch.cuda.synchronize()
        return t0.elapsed_time(t1)

    for mode in ("free", "rec", "chain", "chain_k", "chain_k3", "fifo_k"):
        run(mode)
        ms = min(run(mode) for _ in range(3))
        print(json.dumps({"mode": mode, "MiB": a.mib, "ms": ms, "gbs_per_dir": GB / (ms * 1e-3) / 1e9,
                          "us_per_chunk": ms * 1e3 / n}), flush=True)


if __name__ == "__main__":
    main()
