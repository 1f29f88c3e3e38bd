#!/usr/bin/env python3
"""bench.py — pipelined chunked offload (Cui et al., IPDPS'17) on B200.

Metric (BASELINE.json): "pipelined end-to-end GB/s vs host-link roofline; speedup & HBM saved vs naive".
Workload (N=1, BASELINE.json configs[1]): 3-D 7-point stencil (Fig. 2) over 512^3 fp64,
+-1-plane halo, 8-plane input ring (chunk 2), 3 streams, one sweep k = 1..510.

One JSON line on rank 0:
  value  — GB/s of the step's algorithmic bytes (distinct input planes + output planes) with the
           arrays RESIDENT in HBM (pp_map of device tensors: the index handler is the identity,
           one chunk), device-timed with CUDA events on the launching stream.
  e2e    — the paper's metric: the same loop through the C ABI with PINNED HOST arrays, every
           step's H2D and D2H inside the timed region (pp_launch, chunk 2, 3 streams, 8+6 planes of
           ring), GB/s = (H2D + D2H bytes) / time, plus the host-link pipeline roofline fraction.
  naive  — the synchronous full-footprint offload on the same arrays: speedup and
           device memory saved.
  roofline — the dominant kernel (stencil7, resident launch) vs measured HBM copy peak.
  cpu_baseline — the CPU oracle on the box's cores, bounded sample, same metric.
N>1 (torchrun): every rank pipelines its own 510-plane slab of one global array (weak scaling,
halo planes re-read from host, no data-path collective); value = all ranks' bytes / max-over-ranks
time. `--impl reference` times the CPU oracle (rank 0 only) on the same config.
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "pipelined end-to-end GB/s vs host-link roofline; speedup & HBM saved vs naive"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--n", type=int, default=512, help="grid edge (nz = n per rank)")
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    ap.add_argument("--chunk", type=int, default=2)
    ap.add_argument("--streams", type=int, default=3)
    ap.add_argument("--policy", type=int, default=1)
    ap.add_argument("--graph", type=int, default=0)
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-naive", action="store_true")
    ap.add_argument("--no-schedules", action="store_true", help="skip the alternative-schedule table")
    ap.add_argument("--no-autotune", action="store_true", help="headline with the literal chunk/streams")
    ap.add_argument("--verify", type=int, default=1, help="bit-exact consistency check of the pipelined output vs the resident output")
    return ap.parse_args()


class Clocks:
    """nvidia-smi sampler running during the timed regions (B200_PROFILING.md clocks line)."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap,utilization.gpu")

    def __init__(self, dev):
        self.dev = dev
        self.p = None

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                       "-lms", "100", "-i", str(self.dev)], stdout=subprocess.PIPE,
                                      stderr=subprocess.DEVNULL, text=True)
        except Exception:  # noqa: BLE001
            self.p = None
        time.sleep(0.3)
        return self

    def __exit__(self, *a):
        self.rows = []
        if self.p is None:
            return
        time.sleep(0.25)
        self.p.terminate()
        try:
            out, _ = self.p.communicate(timeout=5)
        except Exception:  # noqa: BLE001
            self.p.kill()
            out = ""
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) >= 8:
                self.rows.append(f)

    def summary(self):
        if not getattr(self, "rows", None):
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        load = [float(r[0]) for r in self.rows if r[7].isdigit() and int(r[7]) > 0] or sm
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in self.rows:
            for n, v in zip(names, r[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": statistics.median(load) if load else None,
                "sm_max_mhz": float(self.rows[0][1]) if self.rows else None,
                "reasons": sorted(reasons), "samples": len(self.rows)}


def dist_init():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def reference_arm(args, ws, rank):
    """--impl reference: the CPU oracle as it stands on the box's host cores (rank 0 only)."""
    if rank != 0:
        return
    import oracle
    import synth
    n = args.n
    dt = np.float64 if args.dtype == "f64" else np.float32
    esz = np.dtype(dt).itemsize
    # each step is the whole configs[1] sweep (planes [1, n-1) of the n^3 array: ~30 ms on a
    # 16-thread host), so the arm times the oracle on exactly the workload the GPU arm runs
    m = n - 2
    A0 = np.empty((m + 2, n, n), dtype=dt)
    synth.fill(A0, "random", seed=synth.SEED_A, nx=n, ny=n)
    out = np.empty_like(A0)
    c0 = dt(1) / dt(6)
    c1 = c0 / dt(6)
    for _ in range(args.warmup):
        oracle.stencil7(A0, out, 1, m + 1, c0, c1)
    t = time.perf_counter()
    for _ in range(args.steps):
        oracle.stencil7(A0, out, 1, m + 1, c0, c1)
    el = time.perf_counter() - t
    plane = n * n * esz
    bytes_step = (m + 2) * plane + m * plane
    v = bytes_step * args.steps / el / 1e9
    sample = f"the whole sweep, planes [1,{m + 1}) of the {n}^3 {args.dtype} stencil, per step (oracle, all host threads)"
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": v, "unit": "GB/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": el / args.steps * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": args.dtype,
        "data": "synthetic", "config": workload_config(args, ws),
        "cpu_baseline": {"value": v, "unit": "GB/s", "cores": oracle.threads(), "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": v, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}))


def ncu_traffic(path, min_grid=200):
    """DRAM bytes (read + write) per launch of the resident stencil launch in a committed
    `ncu --set full` capture (raw CSV export); None if unavailable."""
    import csv
    try:
        rows = list(csv.reader(open(path)))
    except OSError:
        return None
    if len(rows) < 3:
        return None
    hdr, units = rows[0], rows[1]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    for r in rows[2:]:
        d, u = dict(zip(hdr, r)), dict(zip(hdr, units))
        try:
            if int(d.get("launch__grid_size", "0")) < min_grid:
                continue
            return (float(d["dram__bytes_read.sum"]) * scale.get(u["dram__bytes_read.sum"], 1)
                    + float(d["dram__bytes_write.sum"]) * scale.get(u["dram__bytes_write.sum"], 1))
        except (KeyError, ValueError):
            continue
    return None


def workload_config(args, ws):
    return {"workload": f"BASELINE.json configs[1]: 3D 7-point stencil {args.n}^3 {args.dtype}, +-1-plane halo, "
                        f"{args.streams * args.chunk + 2}-plane input ring (+{args.streams * args.chunk} output), "
                        f"3 streams; chunk size picked by the runtime within that device budget (pp_autotune)",
            "nz_per_rank": args.n, "ny": args.n, "nx": args.n, "chunk": args.chunk, "streams": args.streams,
            "stream_policy": ["per-chunk", "per-stage", "two-stream", "copies round-robin per direction + kernel stream",
                              "per-chunk H2D+kernel, separate D2H streams"][args.policy], "cuda_graph": bool(args.graph),
            "parallelism": (f"slab x{ws}" if ws > 1 else "single GPU") + (
                " (ranks share cuda:0: functional test, not scaling)" if os.environ.get("PP_BENCH_SHARE_GPU") == "1" else ""),
            "l2": "inputs larger than L2 (value: 1 GiB in + 1 GiB out resident per step); e2e streams from host",
            "value_mode": "arrays resident in HBM, identity index map, one kernel launch per step",
            "e2e_mode": "pinned host arrays through pp_launch (C ABI), H2D/D2H inside the timed region"}


def main():
    args = parse()
    ws, rank, local = dist_init()
    if args.impl == "reference":
        reference_arm(args, ws, rank)
        return
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_cuissf17_b200 as pp
    import synth

    # PP_BENCH_SHARE_GPU=1: functional test of the N>1 path on one GPU (all ranks on cuda:0, gloo for
    # the timing reductions). Not a scaling measurement: the ranks share one host link.
    share = os.environ.get("PP_BENCH_SHARE_GPU") == "1"
    dev = 0 if share else local
    torch.cuda.set_device(dev)
    # one process per GPU: run on (and first-touch the host slab from) the GPU's local NUMA node
    from paper_conf_ipps_cuissf17_b200 import hostmem
    bound_cpus = hostmem.bind_local_cpus(dev) if ws > 1 and not share else None
    if ws > 1:
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    def barrier():
        if ws > 1:
            dist.barrier()

    def max_over_ranks(x):
        if ws == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cpu" if share else "cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    n = args.n
    tdt = torch.float64 if args.dtype == "f64" else torch.float32
    esz = 8 if args.dtype == "f64" else 4
    plane = n * n * esz
    # global array of ws*(n-2)+2 planes; this rank's loop slab [lo_g, hi_g) and its host planes
    nz_g = ws * (n - 2) + 2
    lo_g, hi_g = pp.pp_partition(1, nz_g - 1, ws, rank)
    p0 = lo_g - 1                      # first plane this rank's host slab holds
    nzl = hi_g - lo_g + 2
    A0 = torch.empty((nzl, n, n), dtype=tdt, pin_memory=True)
    An = torch.empty((nzl, n, n), dtype=tdt, pin_memory=True)
    synth.fill(A0, "random", seed=synth.SEED_A, g0=p0 * n * n, nx=n, ny=n)
    synth.fill_sentinel(An)
    c0 = (np.float64(1) / 6) if tdt == torch.float64 else float(np.float32(1) / np.float32(6))
    c1 = (np.float64(c0) / 6) if tdt == torch.float64 else float(np.float32(c0) / np.float32(6))
    c0, c1 = float(c0), float(c1)
    lo, hi = 1, nzl - 1                # local loop range (global [lo_g, hi_g))
    iters = hi - lo
    B_in = nzl * plane                 # distinct input planes (halo reuse: each copied once)
    B_out = iters * plane
    stream = torch.cuda.Stream()

    def timed(fn, steps, warmup):
        for _ in range(warmup):
            fn()
        barrier()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(steps):
            fn()
        e1.record(stream)
        torch.cuda.synchronize()
        barrier()
        return e0.elapsed_time(e1) / steps     # ms per step on this rank

    clk = Clocks(dev)
    with clk:
        # ---------------- value: resident in HBM --------------------------------------------
        dA = A0.to(f"cuda:{dev}")
        dN = torch.empty_like(dA)
        rv = pp.Region(dev)
        rv.map("to", dA, -1, 3)
        rv.map("from", dN)
        rv.pipeline(0, 1)              # auto chunk: one chunk for resident arrays
        rv.use_streams([stream.cuda_stream])
        ms_v = timed(lambda: rv.launch_async(lo, hi, "stencil7", c0=c0, c1=c1), args.steps, args.warmup)
        rv.wait()
        info_v = rv.query()
        ms_v_max = max_over_ranks(ms_v)
        value = ws * (B_in + B_out) / (ms_v_max * 1e-3) / 1e9
        kernel_path = info_v["kernel_path"]
        # ---------------- e2e: pinned host arrays through the C ABI ---------------------------
        # configs[1]'s device budget: the ring of `chunk` planes x `streams` in flight (8 + 6 planes
        # = 28 MiB for c=2, S=3); within it the runtime picks the chunk size with
        # pp_autotune unless --no-autotune (then the literal c, S)
        ring_budget = ((args.streams * args.chunk + 2) + args.streams * args.chunk) * plane
        re = pp.Region(dev)
        re.map("to", A0, -1, 3)
        re.map("from", An)
        re.pipeline(args.chunk, args.streams)
        re.set_option(pp.PP_OPT_STREAM_POLICY, args.policy)
        re.set_option(pp.PP_OPT_GRAPH, args.graph)
        re.mem_limit(ring_budget)
        tune = None
        if not args.no_autotune:
            tune = re.autotune(lo, hi, "stencil7", trials=6, c0=c0, c1=c1)
        ms_e = timed(lambda: re.launch(lo, hi, "stencil7", c0=c0, c1=c1), args.steps, args.warmup)
        info_e = re.query()
        ms_e_max = max_over_ranks(ms_e)
        e2e = ws * (info_e["h2d_bytes"] + info_e["d2h_bytes"]) / (ms_e_max * 1e-3) / 1e9
        # ---------------- the same loop under other schedules (context for the headline) -------
        schedules = []
        if not args.no_schedules:
            for name, c, S, pol, gr, mir in (
                    ("literal c=2, 3 chunks in flight, per-stage streams (policy 1)", 2, 3, 1, 0, 1),
                    ("literal c=2 S=3, the paper's per-chunk streams (policy 0)", 2, 3, 0, 0, 1),
                    ("literal c=2 S=3, copies round-robin per direction (policy 3)", 2, 3, 3, 0, 1),
                    ("literal c=2 S=3, per-chunk H2D+kernel streams, CUDA graph (policy 4)", 2, 3, 4, 1, 1),
                    ("c=6, 1 chunk in flight, mirrored rings OFF (wrapping copies split in two)", 6, 1, 1, 0, 0),
                    ("auto chunk, S=3, budget = free HBM", 0, 3, 1, 0, 1),
                    ("c=16 S=6 (388 MiB ring)", 16, 6, 1, 0, 1)):
                rs = pp.Region(dev)
                rs.set_option(pp.PP_OPT_MIRROR, mir)
                rs.map("to", A0, -1, 3)
                rs.map("from", An)
                rs.pipeline(c, S)
                rs.set_option(pp.PP_OPT_STREAM_POLICY, pol)
                rs.set_option(pp.PP_OPT_GRAPH, gr)
                ms_s = timed(lambda: rs.launch(lo, hi, "stencil7", c0=c0, c1=c1), max(3, args.steps // 2), 1)
                qs = rs.query()
                ms_s = max_over_ranks(ms_s)
                schedules.append({"schedule": name, "chunk": qs["chunk_size"], "streams": qs["num_streams"],
                                  "ring_bytes": qs["ring_bytes"], "copies": qs["n_h2d"] + qs["n_d2h"], "ms": ms_s,
                                  "gbs": ws * (qs["h2d_bytes"] + qs["d2h_bytes"]) / (ms_s * 1e-3) / 1e9})
                rs.close()
        # ---------------- naive synchronous offload -----------------------------------------
        naive = None
        if not args.no_naive:
            rn = pp.Region(dev)
            rn.map("to", A0, -1, 3)
            rn.map("from", An)
            ms_n = timed(lambda: rn.naive(lo, hi, "stencil7", c0=c0, c1=c1), max(3, args.steps // 2), 1)
            info_n = rn.query()
            ms_n_max = max_over_ranks(ms_n)
            naive = {"ms_per_step": ms_n_max,
                     "gbs": ws * (info_n["h2d_bytes"] + info_n["d2h_bytes"]) / (ms_n_max * 1e-3) / 1e9,
                     "phase_ms": {"h2d": info_n["naive_h2d_ms"], "kernel": info_n["naive_kernel_ms"],
                                  "d2h": info_n["naive_d2h_ms"]},
                     "device_bytes": info_n["naive_bytes"],
                     "speedup_pipelined_vs_naive": ms_n_max / ms_e_max,
                     "hbm_saved": 1.0 - info_e["ring_bytes"] / info_n["naive_bytes"]}
            rn.close()
    clocks = clk.summary()

    # ---------------- consistency of the timed outputs (no oracle here: full-size parity against the
    # oracle is tests/test_gpu_parity.py's job). The pipelined host output (last written by the
    # naive / schedule legs, which all map the same An) must be bit-identical to the resident
    # value-leg output on every computed plane, and the planes outside [lo, hi) must keep the sentinel.
    verified = None
    if args.verify:
        hN = dN.cpu()
        iv = torch.int64 if esz == 8 else torch.int32
        diff = int((An[lo:hi].view(iv) != hN[lo:hi].view(iv)).sum())
        sent = torch.empty_like(An[:1])
        synth.fill_sentinel(sent)
        untouched = all(torch.equal(An[k:k + 1].view(iv), sent.view(iv)) for k in range(nzl) if k < lo or k >= hi)
        verified = {"check": "pipelined host output == resident output (bit-exact), sentinel outside [lo,hi)",
                    "planes_checked": hi - lo, "mismatches": diff, "sentinel_intact": bool(untouched)}

    # ---------------- link roofline ------------------------------------------------------------
    barrier()                          # N > 1: every rank probes its link at the same time
    link = pp.pp_probe_link(dev, 256 << 20, 5)
    import json as _j
    peaks = _j.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {"hbm_gbs": 6650.0}
    hbm_peak = peaks["hbm_gbs"]
    hbm_src = "measured" if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else "fallback"
    t_roof = max(info_e["h2d_bytes"] / (link["h2d"] * 1e9), info_e["d2h_bytes"] / (link["d2h"] * 1e9),
                 (B_in + B_out) / (hbm_peak * 1e9))
    t_roof_duplex = max(info_e["h2d_bytes"] / (link["duplex_h2d"] * 1e9),
                        info_e["d2h_bytes"] / (link["duplex_d2h"] * 1e9))
    # N > 1: each rank streams its own slab through its own link concurrently, so the job's roofline
    # is the slowest rank's (max over ranks), compared with the max-over-ranks e2e time
    t_roof = max_over_ranks(t_roof)
    t_roof_duplex = max_over_ranks(t_roof_duplex)
    link_roof = {"bw_h2d_gbs": link["h2d"], "bw_d2h_gbs": link["d2h"], "duplex_h2d_gbs": link["duplex_h2d"],
                 "duplex_d2h_gbs": link["duplex_d2h"], "t_roof_ms": t_roof * 1e3,
                 "frac": t_roof / (ms_e_max * 1e-3), "t_roof_duplex_ms": t_roof_duplex * 1e3,
                 "frac_of_duplex": t_roof_duplex / (ms_e_max * 1e-3),
                 "probe": "pinned cudaMemcpyAsync 256 MiB, best of 5, each direction alone and concurrently"
                          + (f"; all {ws} ranks probing at once, roofline = the slowest rank's" if ws > 1 else "")}

    # ---------------- cpu baseline (rank 0, N=1 only) --------------------------------------------
    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu:
        import oracle
        # all host threads over the whole workload (every plane of the same 512^3 array, so nothing
        # is cache-resident between reps), ~10 s; plus one thread on an 8-plane slice, ~3 s
        full = np.empty_like(A0.numpy())
        oracle.stencil7(A0.numpy(), full, lo, hi, c0, c1)       # warm (first touch of `full`)
        reps, t = 0, time.perf_counter()
        while True:
            oracle.stencil7(A0.numpy(), full, lo, hi, c0, c1)
            reps += 1
            if time.perf_counter() - t > 10.0:
                break
        el = (time.perf_counter() - t) / reps
        cores = oracle.threads()
        m = 8
        oracle.set_threads(1)
        try:
            reps1, t1 = 0, time.perf_counter()
            while True:
                oracle.stencil7(A0.numpy(), full, 1, m + 1, c0, c1)
                reps1 += 1
                if time.perf_counter() - t1 > 3.0:
                    break
            el1 = (time.perf_counter() - t1) / reps1
        finally:
            oracle.set_threads(cores)
        del full
        cpu = {"value": (B_in + B_out) / el / 1e9, "unit": "GB/s", "cores": cores, "kind": "oracle",
               "sample": f"the whole configs[1] sweep (planes [{lo},{hi}) of the same {n}^3 {args.dtype} array), "
                         f"{reps} reps in ~10 s, all {cores} host threads",
               "single_thread": {"value": ((m + 2) * plane + m * plane) / el1 / 1e9, "unit": "GB/s", "cores": 1,
                                 "sample": f"planes [1,{m + 1}), {reps1} reps in ~3 s"}}

    if rank == 0:
        kernel_bytes = B_in + B_out
        rec = {
            "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_v_max, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": args.dtype, "data": "synthetic (counter-based U[0,1), seed 2017)",
            "config": dict(workload_config(args, ws), numa_bound_cpus=len(bound_cpus) if bound_cpus else None),
            "roofline": {"bound": "hbm", "achieved": kernel_bytes / (ms_v * 1e-3) / 1e9, "peak": hbm_peak,
                         "unit": "GB/s", "frac": kernel_bytes / (ms_v * 1e-3) / 1e9 / hbm_peak,
                         "traffic": ncu_traffic(os.path.join(ROOT, "profiles", "r1s3_ncu_stencil7_tma_raw.csv")),
                         "traffic_source": "profiles/r1s3_ncu_stencil7_tma_raw.csv (ncu --set full, same resident launch)",
                         "kernel": "stencil7 " + {1: "generic", 2: "tma"}.get(kernel_path, "?"),
                         "peak_source": f"{hbm_src} (MEASURED_PEAKS.json hbm_gbs)",
                         "algorithmic_bytes_per_launch": kernel_bytes},
            "e2e": {"value": e2e, "unit": "GB/s", "h2d_bytes_per_step": info_e["h2d_bytes"],
                    "d2h_bytes_per_step": info_e["d2h_bytes"], "ms_per_step": ms_e_max,
                    "chunk": info_e["chunk_size"], "chunks_in_flight": info_e["num_streams"],
                    "device_budget_bytes": ring_budget, "autotune": tune,
                    "graph_replayed": bool(info_e["graph_replayed"]),
                    "chunks": info_e["nchunks"], "ring_planes": info_e["ring_planes"],
                    "ring_bytes": info_e["ring_bytes"], "library_ms": info_e["last_ms"],
                    "link_roofline": link_roof, "schedules": schedules},
            "naive": naive,
            "cpu_baseline": cpu,
            "verify": verified,
            "clocks": clocks,
            "gpu_launches": args.steps * (info_v["n_kernels"] + info_e["n_kernels"]),
            "gpu_launches_detail": {"value_per_step": info_v["n_kernels"], "e2e_per_step": info_e["n_kernels"]},
        }
        print(json.dumps(rec))
    rv.close()
    re.close()
    if ws > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
