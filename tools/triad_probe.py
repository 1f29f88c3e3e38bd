#!/usr/bin/env python3
"""Triad measurements (BASELINE.json configs[0]): c = a + s*b in fp32.

  resident   n = 2^28 arrays already in HBM, one launch (the kernel's HBM roofline: 12 B per element)
  configs[0] n = 2^20 pinned host arrays, c = 2^18 (4 chunks), 2 streams, through pp_launch
             (H2D 8 MiB, D2H 4 MiB per launch), vs the naive synchronous offload and the link roofline
  chunks     the same pipelined launch at larger n and several (c, S), to show where fill/drain stops
             dominating

Prints one JSON line per measurement. No oracle here: parity is tests/test_gpu_parity.py's job; this
tool checks that every pipelined output is bit-identical to the resident kernel's output.

usage: python tools/triad_probe.py [--reps 20]
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


def events_ms(fn, reps, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    out = []
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        out.append(e0.elapsed_time(e1))
    return out


def stats(xs):
    return {"mean_ms": statistics.mean(xs), "median_ms": statistics.median(xs), "min_ms": min(xs)}


def diag_configs0(dev, s, reps):
    """configs[0] variants: per-stage vs paper streams, CUDA-graph replay, chunk counts; op trace."""
    import time
    nn = 1 << 20
    ha = torch.empty(nn, dtype=torch.float32, pin_memory=True)
    hb = torch.empty(nn, dtype=torch.float32, pin_memory=True)
    hc = torch.empty(nn, dtype=torch.float32, pin_memory=True)
    synth.fill(ha, "random", seed=synth.SEED_A)
    synth.fill(hb, "random", seed=synth.SEED_B)
    for (c, S, pol, graph, smc) in [(1 << 18, 2, 1, 0, 0), (1 << 18, 2, 0, 0, 0), (1 << 18, 2, 1, 1, 0),
                                    (1 << 18, 2, 0, 1, 0), (1 << 18, 2, 3, 1, 0), (1 << 18, 4, 3, 1, 0),
                                    (1 << 17, 2, 1, 1, 0), (1 << 20, 1, 1, 1, 0), (1 << 18, 2, 0, 0, 1),
                                    (1 << 18, 2, 1, 0, 1), (1 << 18, 2, 4, 0, 1), (1 << 18, 2, 0, 1, 1)]:
        with pp.Region(dev) as r:
            r.map("to", ha)
            r.map("to", hb)
            r.map("from", hc)
            r.pipeline(c, S)
            r.set_option(pp.PP_OPT_STREAM_POLICY, pol)
            r.set_option(pp.PP_OPT_GRAPH, graph)
            r.set_option(pp.PP_OPT_SM_COPY, (4 << 20) if smc else 0)
            ev = events_ms(lambda: r.launch(0, nn, "triad", s=s), reps)
            lib = []
            wall = []
            for _ in range(reps):
                t = time.perf_counter()
                r.launch(0, nn, "triad", s=s)
                wall.append((time.perf_counter() - t) * 1e3)
                lib.append(r.query()["last_ms"])
            rec = {"case": "diag", "chunk": c, "streams": S, "policy": pol, "graph": graph, "sm_copy": smc,
                   "events_median_ms": statistics.median(ev), "lib_median_ms": statistics.median(lib),
                   "wall_median_ms": statistics.median(wall)}
            if not graph:
                r.set_option(pp.PP_OPT_TRACE, 1)
                r.launch(0, nn, "triad", s=s)
                rec["trace"] = [(t["kind"], t["chunk"], round(t["start_ms"] * 1e3, 1), round(t["end_ms"] * 1e3, 1))
                                for t in r.trace()]
            print(json.dumps(rec), flush=True)
    # naive for reference
    with pp.Region(dev) as rn:
        rn.map("to", ha)
        rn.map("to", hb)
        rn.map("from", hc)
        tn = events_ms(lambda: rn.naive(0, nn, "triad", s=s), reps)
        q = rn.query()
        print(json.dumps({"case": "diag-naive", "events_median_ms": statistics.median(tn),
                          "phase_ms": [q["naive_h2d_ms"], q["naive_kernel_ms"], q["naive_d2h_ms"]]}), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--diag", action="store_true", help="configs[0] schedule variants + op trace only")
    a = ap.parse_args()
    dev = 0
    torch.cuda.set_device(dev)
    s = 3.0
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {"hbm_gbs": 6650.0}
    link = pp.pp_probe_link(dev, 256 << 20, 5)

    # ---- resident n = 2^28 (1 GiB per array)
    n = 1 << 28
    da = torch.empty(n, dtype=torch.float32, device="cuda")
    db = torch.empty_like(da)
    dc = torch.empty_like(da)
    ha = torch.empty(n, dtype=torch.float32, pin_memory=True)
    synth.fill(ha, "random", seed=synth.SEED_A)
    da.copy_(ha)
    synth.fill(ha, "random", seed=synth.SEED_B)
    db.copy_(ha)
    del ha
    with pp.Region(dev) as r:
        r.map("to", da)
        r.map("to", db)
        r.map("from", dc)
        r.pipeline(n, 1)
        ts = []
        for i in range(a.reps + 3):
            r.launch(0, n, "triad", s=s)
            if i >= 3:
                ts.append(r.query()["last_ms"])       # the library's CUDA events on its own stream
    st = stats(ts)
    gbs = 12 * n / (st["median_ms"] * 1e-3) / 1e9
    print(json.dumps({"case": "resident", "n": n, **st, "gbs": gbs, "hbm_peak_gbs": peaks["hbm_gbs"],
                      "frac": gbs / peaks["hbm_gbs"], "bytes_per_launch": 12 * n}), flush=True)
    ref_full = dc  # the resident output, the consistency reference below

    if a.diag:
        diag_configs0(dev, s, a.reps)
        return
    # ---- pipelined from pinned host: configs[0] and larger n
    cases = [(1 << 20, 1 << 18, 2, "configs[0]"), (1 << 20, 1 << 16, 3, ""), (1 << 24, 1 << 20, 3, ""),
             (1 << 26, 1 << 22, 3, ""), (1 << 28, 1 << 22, 3, ""), (1 << 28, 1 << 24, 3, "")]
    host = {}
    for (nn, c, S, tag) in cases:
        if nn not in host:
            ha = torch.empty(nn, dtype=torch.float32, pin_memory=True)
            hb = torch.empty(nn, dtype=torch.float32, pin_memory=True)
            hc = torch.empty(nn, dtype=torch.float32, pin_memory=True)
            synth.fill(ha, "random", seed=synth.SEED_A)
            synth.fill(hb, "random", seed=synth.SEED_B)
            host[nn] = (ha, hb, hc)
        ha, hb, hc = host[nn]
        synth.fill_sentinel(hc)
        rec = {"case": tag or "pipelined", "n": nn, "chunk": c, "streams": S}
        with pp.Region(dev) as r:
            r.map("to", ha)
            r.map("to", hb)
            r.map("from", hc)
            r.pipeline(c, S)
            ts = events_ms(lambda: r.launch(0, nn, "triad", s=s), a.reps)
            info = r.query()
        st = stats(ts)
        bin_, bout = info["h2d_bytes"], info["d2h_bytes"]
        t_roof = max(bin_ / (link["h2d"] * 1e9), bout / (link["d2h"] * 1e9))
        t_roof_dx = max(bin_ / (link["duplex_h2d"] * 1e9), bout / (link["duplex_d2h"] * 1e9))
        rec.update(st)
        rec.update({"e2e_gbs": (bin_ + bout) / (st["median_ms"] * 1e-3) / 1e9, "h2d_bytes": bin_, "d2h_bytes": bout,
                    "ring_bytes": info["ring_bytes"], "t_roof_ms": t_roof * 1e3,
                    "frac_of_roofline": t_roof / (st["median_ms"] * 1e-3),
                    "frac_of_duplex": t_roof_dx / (st["median_ms"] * 1e-3), "nchunks": info["nchunks"],
                    "consistent_with_resident": bool(torch.equal(hc.view(torch.int32),
                                                                 ref_full[:nn].cpu().view(torch.int32)))})
        # fill/drain bound for few chunks: the first chunk's H2D and the last chunk's D2H cannot overlap
        nch = info["nchunks"]
        rec["fill_drain_bound_frac"] = nch / (nch + 1) if nch > 1 else 0.5
        # naive synchronous offload of the same launch
        with pp.Region(dev) as rn:
            rn.map("to", ha)
            rn.map("to", hb)
            rn.map("from", hc)
            tn = events_ms(lambda: rn.naive(0, nn, "triad", s=s), max(5, a.reps // 2))
            info_n = rn.query()
            rn.naive_release()
        rec["naive_median_ms"] = statistics.median(tn)
        rec["speedup_vs_naive"] = rec["naive_median_ms"] / st["median_ms"]
        rec["naive_device_bytes"] = info_n["naive_bytes"]
        rec["hbm_saved"] = 1.0 - info["ring_bytes"] / info_n["naive_bytes"]
        print(json.dumps(rec), flush=True)
    print(json.dumps({"case": "link", **link}), flush=True)


if __name__ == "__main__":
    main()
