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
           step's H2D and D2H inside the timed region (pp_launch within the 8+6-plane ring budget,
           3 streams), GB/s = (H2D + D2H bytes) / time, plus the host-link pipeline roofline fraction.
  ooc    — BASELINE.json configs[2], the north_star target: fp32 stencil over a host array LARGER
           THAN THE GPU's HBM (sized from MemAvailable, 2 MiB pages, in place: reading S24), 4e9 B
           device budget, c = 8, S = 3. Every timed sweep starts from the seeded field and is
           verified bit-for-bit on every plane by the CPU oracle (outside the timed region).
           N > 1: the same array slab-partitioned over the ranks (BASELINE.json configs[3]).
  triad  — BASELINE.json configs[0]: c = a + s*b, n = 2^20 fp32, 4 chunks, 2 streams.
  naive  — the synchronous full-footprint offload on the same arrays: speedup and
           device memory saved (library-accounted and cudaMemGetInfo deltas, reading S22).
  roofline — the dominant kernel (stencil7, resident launch) vs measured HBM copy peak.
  cpu_baseline — the CPU oracle on the box's cores, bounded sample, same metric.
Host-link rooflines take, per direction, the best rate demonstrated by the probe (each direction
alone or both at once, at the start and the end of the run). Timings give mean / median / min over
the timed steps (reading S21). N>1 (torchrun): every rank pipelines its own 510-plane slab of one
global array (weak scaling, halo planes re-read from host, no data-path collective); value = all
ranks' bytes / max-over-ranks time. `--impl reference` times the CPU oracle (rank 0 only) on the
same config.
"""
import argparse
import json
import math
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
    ap.add_argument("--no-triad", action="store_true", help="skip the configs[0] triad record")
    ap.add_argument("--no-temporal", action="store_true", help="skip the NEXT-1 multi-sweep record")
    ap.add_argument("--verify", type=int, default=1, help="bit-exact consistency check of the pipelined output vs the resident output")
    ap.add_argument("--ooc", default="auto",
                    help="configs[2] out-of-core record: 'auto' (host array just larger than HBM, capped by "
                         "MemAvailable), a size in GB, or 'off'")
    ap.add_argument("--ooc-steps", type=int, default=3)
    ap.add_argument("--ooc-warmup", type=int, default=1)
    ap.add_argument("--ooc-verify", default="all", choices=["all", "last", "none"],
                    help="oracle verification of every timed out-of-core sweep, the last one, or none")
    ap.add_argument("--ooc-headroom-gb", type=float, default=12.0)
    ap.add_argument("--ooc-sweeps", type=int, default=8,
                    help="one extra in-place pass of this many fused Jacobi sweeps over the > HBM array (NEXT-1); "
                         "at N > 1 each rank also holds this many halo planes per side")
    ap.add_argument("--ooc-peer-halo", type=int, default=1,
                    help="N > 1: one extra out-of-core sweep with NVLink peer halos (pp_halo_*) instead of re-reads")
    ap.add_argument("--ooc-interior-ab", type=int, default=1,
                    help="one extra out-of-core sweep with interior-only copy-back (PP_OPT_D2H_INTERIOR)")
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


def meminfo(key):
    for line in open("/proc/meminfo"):
        if line.startswith(key + ":"):
            return int(line.split()[1]) * 1024
    return 0


def stats(xs):
    """mean / median / min of per-step times (reading S21: the paper averages 6 runs)."""
    return {"mean_ms": statistics.mean(xs), "median_ms": statistics.median(xs), "min_ms": min(xs),
            "steps_ms": [round(x, 4) for x in xs] if len(xs) <= 12 else None}


def link_capacity(probes):
    """Per-direction host-link capacity: the best rate any probe demonstrated, alone or duplex."""
    h2d = max(max(p["h2d"], p["duplex_h2d"]) for p in probes)
    d2h = max(max(p["d2h"], p["duplex_d2h"]) for p in probes)
    return h2d, d2h


def link_roofline(probes, b_in, b_out, t_meas_s, b_hbm=0, hbm_peak=None, t_roof_reduce=lambda x: x):
    """T_roof = max(B_in / BW_h2d, B_out / BW_d2h, B_hbm / BW_hbm) with BW per direction = best
    demonstrated rate (alone or duplex); also the fractions against the alone-only and duplex-only
    bounds, for context. t_roof_reduce: max over ranks when every rank streams its own slab."""
    h2d, d2h = link_capacity(probes)
    alone_h2d = max(p["h2d"] for p in probes)
    alone_d2h = max(p["d2h"] for p in probes)
    dx_h2d = max(p["duplex_h2d"] for p in probes)
    dx_d2h = max(p["duplex_d2h"] for p in probes)
    hbm_t = b_hbm / (hbm_peak * 1e9) if hbm_peak else 0.0
    t_roof = t_roof_reduce(max(b_in / (h2d * 1e9), b_out / (d2h * 1e9), hbm_t))
    t_alone = t_roof_reduce(max(b_in / (alone_h2d * 1e9), b_out / (alone_d2h * 1e9), hbm_t))
    t_dx = t_roof_reduce(max(b_in / (dx_h2d * 1e9), b_out / (dx_d2h * 1e9), hbm_t))
    return {"bw_h2d_gbs": h2d, "bw_d2h_gbs": d2h, "t_roof_ms": t_roof * 1e3, "frac": t_roof / t_meas_s,
            "alone_h2d_gbs": alone_h2d, "alone_d2h_gbs": alone_d2h, "duplex_h2d_gbs": dx_h2d,
            "duplex_d2h_gbs": dx_d2h, "frac_of_alone": t_alone / t_meas_s, "frac_of_duplex": t_dx / t_meas_s,
            "bound": "per direction max(alone, duplex) over every probe of the run (the best rate the link "
                     "demonstrated); duplex timed over both copies' common window"}


def reference_arm(args, ws, rank):
    """--impl reference: the CPU oracle as it stands on the box's host cores (rank 0 only)."""
    if rank != 0:
        return
    import oracle
    import synth
    # all of the host's cores (torchrun exports OMP_NUM_THREADS=1 to every rank; only rank 0 runs here)
    oracle.set_threads(os.cpu_count() or 1)
    synth.set_threads(os.cpu_count() or 1)
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
                              "per-chunk H2D+kernel, separate D2H streams", "per-array copy streams"][args.policy],
            "cuda_graph": bool(args.graph),
            "parallelism": (f"slab x{ws}" if ws > 1 else "single GPU") + (
                " (ranks share cuda:0: functional test, not scaling)" if os.environ.get("PP_BENCH_SHARE_GPU") == "1" else ""),
            "l2": "inputs larger than L2 (value: 1 GiB in + 1 GiB out resident per step); e2e and ooc stream from host",
            "value_mode": "arrays resident in HBM, identity index map, one kernel launch per step",
            "e2e_mode": "pinned host arrays through pp_launch (C ABI), H2D/D2H inside the timed region"}


class Ctx:
    """Per-run plumbing shared by the legs: device, ranks, the timing stream and reductions."""

    def __init__(self, torch, dist, ws, rank, dev, share):
        self.torch, self.dist, self.ws, self.rank, self.dev, self.share = torch, dist, ws, rank, dev, share
        self._stream = None

    @property
    def stream(self):
        if self._stream is None:
            self._stream = self.torch.cuda.Stream()
        return self._stream

    def barrier(self):
        if self.ws > 1:
            self.dist.barrier()

    def reduce(self, xs, op="max"):
        """Element-wise reduction of a list of floats over ranks (identity at N = 1)."""
        single = not isinstance(xs, (list, tuple))
        xs = [xs] if single else list(xs)
        if self.ws > 1:
            t = self.torch.tensor(xs, dtype=self.torch.float64, device="cpu" if self.share else "cuda")
            self.dist.all_reduce(t, op={"max": self.dist.ReduceOp.MAX, "sum": self.dist.ReduceOp.SUM,
                                        "min": self.dist.ReduceOp.MIN}[op])
            xs = t.cpu().tolist()
        return xs[0] if single else xs

    def timed(self, fn, steps, warmup):
        """Per-step device times (ms, CUDA events on the timing stream), max over ranks per step."""
        torch = self.torch
        for _ in range(warmup):
            fn()
        self.barrier()
        torch.cuda.synchronize()
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(steps + 1)]
        ev[0].record(self.stream)
        for i in range(steps):
            fn()
            ev[i + 1].record(self.stream)
        torch.cuda.synchronize()
        self.barrier()
        return self.reduce([ev[i].elapsed_time(ev[i + 1]) for i in range(steps)], "max")

    def timed_lib(self, r, launch, steps, warmup):
        """timed() over `launch` (an async pp launch on region r) plus each launch's device duration as
        the library measures it: CUDA events it records on the launch stream right before and after its
        ops (pp_query last_ms), collected between launches (the wait each launch performs anyway is made
        explicit). Returns (per-step ms, per-launch device ms), max over ranks per step."""
        ks = []

        def step():
            r.wait()
            ks.append(r.query()["last_ms"])
            launch()
        per = self.timed(step, steps, warmup)
        r.wait()
        ks.append(r.query()["last_ms"])
        return per, self.reduce(ks[-steps:], "max")

    def settle_link(self, pp, max_s=8.0, nbytes=256 << 20):
        """Untimed: repeat a short duplex link probe until two consecutive results agree within 1.5%
        and sit within 3% of the best seen (or max_s passes). Some boxes start a run with the host link
        ~10% slower for a few seconds (first probe 44.6-45.4 GB/s duplex, 49.5 later in the same run);
        this keeps that phase out of the timed legs and records it."""
        hist, t0, best = [], time.time(), 0.0
        while True:
            # one collective per round: every rank sees the same probe value and the same stop decision
            d = float(self.reduce(pp.pp_probe_link(self.dev, nbytes, 2)["duplex_h2d"], "min"))
            late = float(self.reduce(float(time.time() - t0 >= max_s), "max"))
            hist.append(round(d, 2))
            best = max(best, d)
            if late or (len(hist) >= 2 and abs(hist[-1] - hist[-2]) <= 0.015 * best and d >= 0.97 * best):
                break
        return {"duplex_gbs": hist, "seconds": round(time.time() - t0, 2)}

    def probe(self, pp, nbytes=512 << 20, reps=8):
        self.barrier()                 # N > 1: every rank probes its link at the same time
        return pp.pp_probe_link(self.dev, nbytes, reps)


def ooc_verify(A, p0, c0, c1, oracle, synth, B=14):
    """Verify-in-place of an in-place sweep over local planes [1, nz-1) of A (global plane index of
    local plane 0 = p0): regenerate the original input planes block by block from the counter-based
    generator and let the oracle recompute and compare every element's bits; planes 0 and nz-1 must
    still hold the input. Returns (planes_checked, mismatches)."""
    nz, ny, nx = A.shape
    buf = np.empty((B + 2, ny, nx), dtype=A.dtype)
    bad = checked = 0
    for k0 in range(1, nz - 1, B):
        k1 = min(k0 + B, nz - 1)
        m = k1 - k0
        src = buf[: m + 2]
        synth.fill(src, "random", seed=synth.SEED_A, g0=(p0 + k0 - 1) * ny * nx, nx=nx, ny=ny)
        bad += oracle.stencil7_verify(src, A[k0 - 1:k1 + 1], 1, m + 1, c0, c1)
        checked += m
    iv = np.uint32 if A.dtype == np.float32 else np.uint64
    for k in (0, nz - 1):
        synth.fill(buf[:1], "random", seed=synth.SEED_A, g0=(p0 + k) * ny * nx, nx=nx, ny=ny)
        bad += int(np.count_nonzero(buf[0].view(iv) != A[k].view(iv)))
    return checked, bad


def lightcone_verify(A, p0, T, c0, c1, oracle, synth, blocks=12, w=64, seed=5, kvalid=None, real_lo=True,
                     real_hi=True):
    """Verification of a T-sweep in-place pass over local planes [1, nz-1) of A (planes 0 and nz-1 and
    every plane's edge ring fixed at the input; global plane of local plane 0 = p0). Output point (k,j,i)
    depends only on inputs within distance T in each dimension, so a sub-block regenerated from the
    counter-based generator and swept T times by the oracle with its faces held fixed reproduces A^T
    exactly on the points farther than T from its faces (or on the array's real faces). `blocks`
    sub-blocks with a w x w core, some on the y = 0 / x = nx-1 edges. Returns (points, mismatches).
    A slab of a larger array (N > 1): only local planes kvalid = [klo, khi) are checked, and its end
    planes count as real faces only where they are the global array's (real_lo / real_hi)."""
    nz, ny, nx = A.shape
    klo, khi = kvalid if kvalid else (1, nz - 1)
    iv = np.uint32 if A.dtype == np.float32 else np.uint64
    rng = np.random.default_rng(seed)
    bad = checked = 0
    for b in range(blocks):
        kc = int(rng.integers(max(1, klo), min(nz - 1, khi)))
        jc = int(rng.integers(0, max(1, ny - w))) if b % 2 else 0
        ic = int(rng.integers(0, max(1, nx - w))) if b % 3 else max(0, nx - w)
        k0, k1 = max(0, kc - T - 1), min(nz, kc + T + 2)
        j0, j1 = max(0, jc - T - 1), min(ny, jc + w + T + 1)
        i0, i1 = max(0, ic - T - 1), min(nx, ic + w + T + 1)
        blk = np.empty((k1 - k0, j1 - j0, i1 - i0), dtype=A.dtype)
        for k in range(k0, k1):
            for j in range(j0, j1):
                synth.fill(blk[k - k0, j - j0], "random", seed=synth.SEED_A,
                           g0=((p0 + k) * ny + j) * nx + i0, nx=nx, ny=ny)
        ref = blk.copy()
        oracle.stencil7_sweeps(blk, ref, 1, k1 - k0 - 1, c0, c1, T)
        kk = [k for k in range(k0, k1) if (k - k0 > T or (k0 == 0 and real_lo))
              and (k1 - 1 - k > T or (k1 == nz and real_hi)) and max(1, klo) <= k < min(nz - 1, khi)]
        jj = [j for j in range(j0, j1) if (j - j0 > T or j0 == 0) and (j1 - 1 - j > T or j1 == ny)]
        ii = [i for i in range(i0, i1) if (i - i0 > T or i0 == 0) and (i1 - 1 - i > T or i1 == nx)]
        if not (kk and jj and ii):
            continue
        want = ref[kk[0] - k0:kk[-1] - k0 + 1, jj[0] - j0:jj[-1] - j0 + 1, ii[0] - i0:ii[-1] - i0 + 1]
        got = np.ascontiguousarray(A[kk[0]:kk[-1] + 1, jj[0]:jj[-1] + 1, ii[0]:ii[-1] + 1])
        bad += int(np.count_nonzero(want.view(iv) != got.view(iv)))
        checked += want.size
    return checked, bad


def ooc_temporal(args, cx, pp, synth, oracle, Abuf, pb0, kvalid, real_lo, real_hi, ny, nx, c0, c1, probes,
                 ms_single):
    """NEXT-1 over the > HBM array: one in-place pass of T Jacobi sweeps (fused level pairs) through the
    host link, 32e9 B device budget (the level rings of the light cone need more than a single sweep's
    4e9 B), verified on light-cone sub-blocks. N > 1 (configs[3]): each rank's buffer holds its slab
    plus T halo planes on each interior side (re-read from host memory); its pass runs over the whole
    buffer and its own planes kvalid are exact, because an error from a held-fixed buffer end moves one
    plane per sweep and stops T planes in."""
    torch = cx.torch
    T = args.ooc_sweeps
    nb = Abuf.shape[0]
    synth.fill(Abuf, "random", seed=synth.SEED_A, g0=pb0 * ny * nx, nx=nx, ny=ny)
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    with pp.Region(cx.dev) as rt:
        rt.set_option(pp.PP_OPT_INPLACE, 1)
        rt.map("to", Abuf, -1, 3)          # already page-locked for the leg
        rt.map("from", Abuf)
        rt.pipeline(0, 3)
        # ranks sharing one GPU (PP_BENCH_SHARE_GPU functional runs) split its memory
        share = int(os.environ.get("LOCAL_WORLD_SIZE", cx.ws)) if cx.share else 1
        rt.mem_limit(int(min(32e9, 0.6 * torch.cuda.mem_get_info(cx.dev)[1] / share)))
        rt.set_option(pp.PP_OPT_SWEEPS, T)
        rt.set_option(pp.PP_OPT_FUSE, 2)
        cx.barrier()
        torch.cuda.synchronize()
        ev0.record(cx.stream)
        rt.launch(1, nb - 1, "stencil7", c0=c0, c1=c1)
        ev1.record(cx.stream)
        torch.cuda.synchronize()
        cx.barrier()
        q = rt.query()
    ms = cx.reduce(ev0.elapsed_time(ev1), "max")
    t = time.time()
    ck, bad = lightcone_verify(Abuf, pb0, T, c0, c1, oracle, synth, kvalid=kvalid, real_lo=real_lo, real_hi=real_hi)
    link = cx.reduce(float(q["h2d_bytes"] + q["d2h_bytes"]), "sum")
    return {"sweeps_per_pass": T, "fuse": 2, "ms_per_pass": ms, "jacobi_sweeps_per_s": T / (ms * 1e-3),
            "effective_gbs": T * link / (ms * 1e-3) / 1e9, "speedup_vs_T_single_sweep_passes": T * ms_single / ms,
            "link_frac": link_roofline(probes, q["h2d_bytes"], q["d2h_bytes"], ms * 1e-3,
                                       t_roof_reduce=lambda x: cx.reduce(x, "max"))["frac"],
            "chunk": q["chunk_size"], "ring_bytes": q["ring_bytes"], "launches_per_pass": q["n_kernels"],
            "halo_planes_per_side": T if cx.ws > 1 else 1,
            "verify": {"points_checked": int(cx.reduce(float(ck), "sum")), "mismatches": int(cx.reduce(float(bad), "sum")),
                       "seconds": time.time() - t,
                       "mode": "light-cone sub-blocks x12 per rank (64 x 64 core, T-wide halo) regenerated and swept "
                               "T times by the oracle"}}


def ooc_global_planes(spec, hbm, plane, avail, headroom_gb, ws, halo=1):
    """(planes wanted, planes host RAM allows) for the out-of-core array: 'auto' = just over the GPU's
    HBM (+0.5%, + the two boundary planes); else spec GB. The limit keeps headroom_gb of MemAvailable
    free and leaves room for the 2 x halo duplicated planes of each of the ws-1 interior slab boundaries."""
    if spec == "auto":
        want = math.ceil(hbm * 1.005 / plane) + 2
    else:
        want = int(float(spec) * 1e9 // plane)
    limit = int((avail - headroom_gb * 1e9) // plane) - 2 * halo * (ws - 1)
    return want, limit


def ooc_leg(args, cx, pp, synth, probes):
    """BASELINE.json configs[2] (N = 1) / configs[3] (N > 1): in-place fp32 7-point stencil over a host
    array larger than one GPU's HBM, 4e9 B device budget, c = 8, S = 3, every timed sweep verified."""
    import oracle                      # verification only, outside every timed region
    from paper_conf_ipps_cuissf17_b200 import hostmem
    torch = cx.torch
    nx = ny = 4096
    plane = nx * ny * 4
    hbm = torch.cuda.mem_get_info(cx.dev)[1]
    # every rank reads MemAvailable before anyone allocates; all take the smallest size (MIN)
    avail = meminfo("MemAvailable")
    H = args.ooc_sweeps if (cx.ws > 1 and args.ooc_sweeps > 1) else 1
    want, limit = ooc_global_planes(args.ooc, hbm, plane, avail, args.ooc_headroom_gb, cx.ws, H)
    nz_global = int(cx.reduce(float(min(want, limit)), "min"))
    if nz_global < 3 * cx.ws + 2:
        return {"skipped": f"host RAM too small (MemAvailable {avail / 1e9:.1f} GB)"}
    lo_g, hi_g = pp.pp_partition(1, nz_global - 1, cx.ws, cx.rank)
    # this rank's host buffer: global planes [pb0, pb1) — its slab with one halo plane per side for
    # the single sweeps, H = T per side when a T-sweep pass follows at N > 1 (configs[3] + NEXT-1)
    pb0, pb1 = max(0, lo_g - H), min(nz_global, hi_g + H)
    p0 = lo_g - 1                      # the single sweeps map the view of global [lo_g - 1, hi_g + 1)
    nz = hi_g - lo_g + 2
    rec = {"workload": f"BASELINE.json configs[{2 if cx.ws == 1 else 3}]: in-place fp32 7-point stencil "
                       f"[{nz_global}][{ny}][{nx}] ({nz_global * plane / 1e9:.1f} GB host array, 2 MiB pages)"
                       + (f", slab-partitioned over {cx.ws} GPUs (halo planes re-read from host)" if cx.ws > 1 else "")
                       + ", 4e9 B device budget per GPU, c = 8, S = 3",
           "host_array_bytes": nz_global * plane, "hbm_total_bytes": hbm,
           "exceeds_hbm": nz_global * plane > hbm, "host_mem_available": avail,
           "size_capped_by_host_ram": want > limit}
    t = time.time()
    Abuf = hostmem.alloc_host((pb1 - pb0, ny, nx), np.float32)
    synth.fill(Abuf, "random", seed=synth.SEED_A, g0=pb0 * ny * nx, nx=nx, ny=ny)
    A = Abuf[p0 - pb0:p0 - pb0 + nz]
    rec["generate_s"] = time.time() - t
    c0 = float(np.float32(1) / np.float32(6))
    c1 = float(np.float32(c0) / np.float32(6))
    t = time.time()
    rpin = pp.Region(cx.dev)           # page-locks the whole buffer once (cudaHostRegister)
    rpin.map("to", Abuf)
    r = pp.Region(cx.dev)
    r.set_option(pp.PP_OPT_INPLACE, 1)
    r.map("to", A, -1, 3)
    r.map("from", A)
    rec["pin_s"] = time.time() - t
    r.pipeline(8, 3)
    r.mem_limit(int(4e9))
    steps = []
    verify = {"planes_checked": 0, "mismatches": 0, "sweeps_verified": 0, "seconds": 0.0}
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    total = args.ooc_warmup + args.ooc_steps
    for it in range(total):
        if it > 0:                     # every sweep starts from the seeded field (not timed)
            synth.fill(A, "random", seed=synth.SEED_A, g0=p0 * ny * nx, nx=nx, ny=ny)
        cx.barrier()
        torch.cuda.synchronize()
        ev0.record(cx.stream)
        r.launch(1, nz - 1, "stencil7", c0=c0, c1=c1)   # blocking: host planes final on return
        ev1.record(cx.stream)
        torch.cuda.synchronize()
        cx.barrier()
        ms = ev0.elapsed_time(ev1)
        if it < args.ooc_warmup:
            continue
        steps.append(ms)
        if args.ooc_verify == "all" or (args.ooc_verify == "last" and it == total - 1):
            t = time.time()
            ck, bad = ooc_verify(A, p0, c0, c1, oracle, synth)
            verify["planes_checked"] += ck
            verify["mismatches"] += bad
            verify["sweeps_verified"] += 1
            verify["seconds"] += time.time() - t
    q = r.query()
    probes.append(cx.probe(pp))                    # the link again, right after the timed sweeps
    # A/B: the same in-place sweep copying back plane interiors only (reading S5b, NEXT-3): in place
    # the host array is identical (edges keep A0), so it is verified the same way
    interior = None
    if args.ooc_interior_ab:
        synth.fill(A, "random", seed=synth.SEED_A, g0=p0 * ny * nx, nx=nx, ny=ny)
        r.set_option(pp.PP_OPT_D2H_INTERIOR, 1)
        cx.barrier()
        torch.cuda.synchronize()
        ev0.record(cx.stream)
        r.launch(1, nz - 1, "stencil7", c0=c0, c1=c1)
        ev1.record(cx.stream)
        torch.cuda.synchronize()
        cx.barrier()
        ms_i = cx.reduce(ev0.elapsed_time(ev1), "max")
        qi = r.query()
        ck, bad = ooc_verify(A, p0, c0, c1, oracle, synth) if args.ooc_verify != "none" else (0, 0)
        interior = {"ms": ms_i, "d2h_bytes": qi["d2h_bytes"], "vs_whole_planes": ms_i / statistics.mean(steps),
                    "gbs": (qi["h2d_bytes"] + qi["d2h_bytes"]) / (ms_i * 1e-3) / 1e9,
                    "planes_checked": int(cx.reduce(float(ck), "sum")),
                    "mismatches": int(cx.reduce(float(bad), "sum")),
                    "copy": "one cudaMemcpy3DAsync per chunk (rows 1..ny-2, columns 1..nx-2)"}
    peer = peer_halo_ab(args, cx, pp, synth, oracle, r, A, p0, nz, ny, nx, c0, c1, steps) if cx.ws > 1 else None
    temporal = None
    if args.ooc_sweeps > 1:
        temporal = ooc_temporal(args, cx, pp, synth, oracle, Abuf, pb0, (lo_g - pb0, hi_g - pb0), pb0 == 0,
                                pb1 == nz_global, ny, nx, c0, c1, probes, statistics.mean(steps))
    r.close()
    rpin.close()                       # unregisters the host buffer
    del A, Abuf
    steps = cx.reduce(steps, "max")
    st = stats(steps)
    b_in, b_out = q["h2d_bytes"], q["d2h_bytes"]
    roof = link_roofline(probes, b_in, b_out, st["mean_ms"] * 1e-3,
                         t_roof_reduce=lambda x: cx.reduce(x, "max"))
    tot_in, tot_out = cx.reduce(float(b_in), "sum"), cx.reduce(float(b_out), "sum")
    verify["planes_checked"] = int(cx.reduce(float(verify["planes_checked"]), "sum"))
    verify["seconds"] = cx.reduce(verify["seconds"], "max")
    verify["mismatches"] = int(cx.reduce(float(verify["mismatches"]), "sum"))
    verify["check"] = ("every timed sweep's host output, every element of every computed plane, vs the CPU "
                       "oracle's verify-in-place (inputs regenerated from the counter-based generator); "
                       "the two boundary planes still hold the input")
    rec.update({"e2e_gbs": (tot_in + tot_out) / (st["mean_ms"] * 1e-3) / 1e9, **st,
                "h2d_bytes_per_sweep": tot_in, "d2h_bytes_per_sweep": tot_out, "warmup": args.ooc_warmup,
                "steps": args.ooc_steps, "chunk": q["chunk_size"], "chunks_in_flight": q["num_streams"],
                "nchunks": q["nchunks"], "ring_planes": q["ring_planes"], "ring_bytes": q["ring_bytes"],
                "device_fraction_of_array": q["ring_bytes"] / (nz_global * plane / cx.ws),
                "kernel_path": q["kernel_path"], "gpu_launches_per_sweep": q["n_kernels"],
                "link_roofline": roof, "verify": verify, "interior_d2h_ab": interior, "peer_halo_ab": peer,
                "temporal": temporal,
                "cpu_baseline": ({"value": (tot_in + tot_out) * verify["sweeps_verified"] / verify["seconds"] / 1e9
                                  if verify["seconds"] > 0 else None, "unit": "GB/s",
                                  "cores": oracle.threads(), "kind": "oracle (verify-in-place)",
                                  "sample": f"the oracle recomputing every plane of {verify['sweeps_verified']} sweeps of "
                                            "this array in place (input regenerated from the counter-based generator, "
                                            "each element compared with the GPU's bits), all host threads"
                                            + (f" of each of the {cx.ws} ranks" if cx.ws > 1 else "")}
                                 if verify["sweeps_verified"] else None),
                "timing": "CUDA events around the blocking pp_launch on the timing stream, max over ranks; the "
                          "untimed refill of the seeded field precedes each sweep"})
    return rec


def peer_halo_ab(args, cx, pp, synth, oracle, r, A, p0, nz, ny, nx, c0, c1, steps):
    """N > 1 A/B: the same out-of-core sweep with each rank's upper halo plane taken
    over NVLink from the next rank's side slot (pp_halo_export / pp_halo_import over CUDA IPC) instead
    of re-read from host memory. One sweep, verified like the others; every rank takes part in every
    collective even when P2P is unavailable or a launch fails (then the record says why)."""
    if not args.ooc_peer_halo:
        return None
    torch = cx.torch
    import torch.distributed as dist
    from torch.multiprocessing.reductions import reduce_tensor
    side = torch.empty((ny, nx), dtype=torch.float32, device=f"cuda:{cx.dev}")
    flag = torch.zeros(1, dtype=torch.int32, device=f"cuda:{cx.dev}")
    mine = (reduce_tensor(side), reduce_tensor(flag))
    every = [None] * cx.ws
    dist.all_gather_object(every, mine)
    why = ""
    peer_side = peer_flag = None
    if cx.rank + 1 < cx.ws:
        try:
            (fs, a_s), (ff, a_f) = every[cx.rank + 1]
            peer_side, peer_flag = fs(*a_s), ff(*a_f)
            pdev = peer_side.device.index
            if pdev != cx.dev:
                from cuda.bindings import runtime as cudart
                ok = cudart.cudaDeviceCanAccessPeer(cx.dev, pdev)
                if ok[0] != cudart.cudaError_t.cudaSuccess or not ok[1]:
                    why = f"cuda:{cx.dev} cannot access cuda:{pdev} peer-to-peer"
                else:
                    cudart.cudaSetDevice(cx.dev)
                    cudart.cudaDeviceEnablePeerAccess(pdev, 0)   # (already enabled is fine)
        except Exception as e:  # noqa: BLE001
            why = f"opening the next rank's side slot failed: {e!r}"[:300]
    ok_all = cx.reduce(0.0 if why else 1.0, "min") > 0
    if not ok_all:
        return {"skipped": why or "another rank could not open its peer's side slot"}
    synth.fill(A, "random", seed=synth.SEED_A, g0=p0 * ny * nx, nx=nx, ny=ny)
    if cx.rank > 0:
        r.halo_export(0, 1, side.data_ptr(), flag.data_ptr(), 1)             # global plane lo_g
    if peer_side is not None:
        r.halo_import(0, nz - 1, peer_side.data_ptr(), peer_side.device.index, peer_flag.data_ptr(), 1)
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    err = ""
    cx.barrier()
    torch.cuda.synchronize()
    ev0.record(cx.stream)
    try:
        r.launch(1, nz - 1, "stencil7", c0=c0, c1=c1)
    except Exception as e:  # noqa: BLE001
        err = repr(e)[:300]
    ev1.record(cx.stream)
    torch.cuda.synchronize()
    cx.barrier()
    r.halo_clear()
    q = r.query()
    ms = cx.reduce(ev0.elapsed_time(ev1), "max")
    del peer_side, peer_flag                   # release the IPC mappings before the exporters free them
    torch.cuda.synchronize()
    cx.barrier()
    failed = cx.reduce(1.0 if err else 0.0, "max") > 0
    ck, bad = (0, 0) if (err or args.ooc_verify == "none") else ooc_verify(A, p0, c0, c1, oracle, synth)
    rec = {"ms": ms, "vs_host_reread": ms / statistics.mean(steps),
           "peer_bytes": cx.reduce(float(q["peer_bytes"]), "sum"),
           "h2d_bytes": cx.reduce(float(q["h2d_bytes"]), "sum"),
           "planes_checked": int(cx.reduce(float(ck), "sum")), "mismatches": int(cx.reduce(float(bad), "sum")),
           "how": "rank g keeps global plane lo_g in a side slot after its H2D; rank g-1 waits on the slot's "
                  "flag and copies it with cudaMemcpyPeerAsync instead of re-reading it from host memory"}
    if failed:
        rec["error"] = err or "a launch failed on another rank"
    return rec


def kernels_leg(args, cx, pp, synth, hbm_peak, dA64, dN64):
    """Driver-visible per-kernel roofline records (resident arrays in HBM, one launch per step, CUDA
    events on the launching stream): the Fig. 2 stencil in both dtypes, the Polybench 3-D convolution
    (NEXT-2) in both dtypes and the configs[0] triad body at a size that fills HBM bandwidth."""
    torch = cx.torch
    n = 512
    out = []
    dA32 = dA64[:n].float() if dA64.shape[0] >= n else None
    if dA32 is None:
        return out
    dN32 = torch.empty_like(dA32)
    plane = n * n
    for kernel, dt, dA, dN in (("stencil7", "f32", dA32, dN32), ("conv3d", "f64", dA64[:n], dN64[:n]),
                               ("conv3d", "f32", dA32, dN32)):
        esz = 8 if dt == "f64" else 4
        with pp.Region(cx.dev) as r:
            r.map("to", dA, -1, 3)
            r.map("from", dN)
            r.pipeline(0, 1)
            r.use_streams([cx.stream.cuda_stream])
            kw = {"c0": 1.0 / 6.0, "c1": 1.0 / 36.0} if kernel == "stencil7" else {}
            per = cx.timed(lambda: r.launch_async(1, n - 1, kernel, **kw), max(5, args.steps), 3)
            _, kern = cx.timed_lib(r, lambda: r.launch_async(1, n - 1, kernel, **kw), max(5, args.steps), 1)
            path = r.query()["kernel_path"]
        byts = (n + (n - 2)) * plane * esz
        st, sk = stats(per), stats(kern)
        gbs = byts / (sk["mean_ms"] * 1e-3) / 1e9
        out.append({"kernel": f"{kernel} ({'tma' if path == 2 else 'generic'})", "dtype": dt, "shape": [n, n, n],
                    "algorithmic_bytes": byts, "ms": sk["mean_ms"], "min_ms": sk["min_ms"], "gbs": gbs,
                    "frac_of_hbm_peak": gbs / hbm_peak, "step_ms": st["mean_ms"],
                    "frac_of_step": byts / (st["mean_ms"] * 1e-3) / 1e9 / hbm_peak})
    nt = 1 << 28
    ta, tb, tc = (torch.empty(nt, dtype=torch.float32, device=f"cuda:{cx.dev}") for _ in range(3))
    ta.fill_(1.0)
    tb.fill_(2.0)
    with pp.Region(cx.dev) as r:
        r.map("to", ta)
        r.map("to", tb)
        r.map("from", tc)
        r.pipeline(0, 1)
        r.use_streams([cx.stream.cuda_stream])
        per = cx.timed(lambda: r.launch_async(0, nt, "triad", s=3.0), max(5, args.steps), 3)
        _, kern = cx.timed_lib(r, lambda: r.launch_async(0, nt, "triad", s=3.0), max(5, args.steps), 1)
    st, sk = stats(per), stats(kern)
    gbs = 12 * nt / (sk["mean_ms"] * 1e-3) / 1e9
    out.append({"kernel": "triad", "dtype": "f32", "shape": [nt], "algorithmic_bytes": 12 * nt, "ms": sk["mean_ms"],
                "min_ms": sk["min_ms"], "gbs": gbs, "frac_of_hbm_peak": gbs / hbm_peak, "step_ms": st["mean_ms"],
                "frac_of_step": 12 * nt / (st["mean_ms"] * 1e-3) / 1e9 / hbm_peak})
    del ta, tb, tc, dA32, dN32
    return out


def temporal_leg(args, cx, pp, A0, An, lo, hi, c0, c1, ms_single, probes):
    """NEXT-1: T Jacobi sweeps of the configs[1] array per pass over the host link
    (PP_OPT_SWEEPS, pairs of levels fused on chip: PP_OPT_FUSE = 2), device budget = free HBM, the chunk
    size and chunks in flight picked by pp_autotune. Each pass's host output is checked bit for bit
    against the naive full-footprint T-sweep run."""
    torch = cx.torch
    iv = torch.int64 if A0.element_size() == 8 else torch.int32
    out = []
    ref = torch.empty_like(An).pin_memory()
    for T in (16, 64):
        with pp.Region(cx.dev) as rn:                # reference: full device arrays, T sweeps
            rn.map("to", A0, -1, 3)
            rn.map("from", ref)
            rn.set_option(pp.PP_OPT_SWEEPS, T)
            rn.set_option(pp.PP_OPT_FUSE, 2)
            rn.naive(lo, hi, "stencil7", c0=c0, c1=c1)
        with pp.Region(cx.dev) as r:
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.pipeline(0, 3)
            r.set_option(pp.PP_OPT_SWEEPS, T)
            r.set_option(pp.PP_OPT_FUSE, 2)
            tune = r.autotune(lo, hi, "stencil7", trials=4, c0=c0, c1=c1)   # the runtime picks c, S
            st = stats(cx.timed(lambda: r.launch(lo, hi, "stencil7", c0=c0, c1=c1), max(3, args.steps // 2), 2))
            q = r.query()
        same = bool(torch.equal(An[lo:hi].view(iv), ref[lo:hi].view(iv)))
        link = q["h2d_bytes"] + q["d2h_bytes"]
        out.append({"sweeps_per_pass": T, "fuse": 2, "ms_per_pass": st["mean_ms"], "min_ms": st["min_ms"],
                    "jacobi_sweeps_per_s": T / (st["mean_ms"] * 1e-3),
                    "effective_gbs": T * link / (st["mean_ms"] * 1e-3) / 1e9,
                    "speedup_vs_T_single_sweep_passes": T * ms_single / st["mean_ms"],
                    "link_frac": link_roofline(probes, q["h2d_bytes"], q["d2h_bytes"], st["mean_ms"] * 1e-3)["frac"],
                    "chunk": q["chunk_size"], "chunks_in_flight": q["num_streams"], "graph": bool(tune["graph"]),
                    "ring_bytes": q["ring_bytes"], "launches_per_pass": q["n_kernels"],
                    "bit_identical_to_naive_T_sweeps": same})
    return out


def triad_leg(args, cx, pp, synth, probes):
    """BASELINE.json configs[0]: c = a + s*b over 2^20 fp32 from pinned host arrays, 4 chunks,
    2 streams (literal, eager and CUDA-graph replay), vs naive and the link roofline."""
    torch = cx.torch
    n = 1 << 20
    hab = torch.empty(2 * n, dtype=torch.float32, pin_memory=True)     # a | b: equally spaced pieces
    ha, hb = hab[:n], hab[n:]
    hc = torch.empty(n, dtype=torch.float32, pin_memory=True)
    synth.fill(ha, "random", seed=synth.SEED_A)
    synth.fill(hb, "random", seed=synth.SEED_B)
    da, db, dc = ha.cuda(), hb.cuda(), torch.empty(n, dtype=torch.float32, device="cuda")
    with pp.Region(cx.dev) as rr:          # resident reference output (consistency check)
        rr.map("to", da)
        rr.map("to", db)
        rr.map("from", dc)
        rr.launch(0, n, "triad", s=3.0)
    ref = dc.cpu()
    steps = max(50, args.steps * 10)
    out = {"workload": "BASELINE.json configs[0]: c[i] = a[i] + s*b[i], n = 2^20 fp32, 4 chunks (c = 2^18), "
                       "2 streams, pinned host arrays (a and b the two halves of one buffer)", "schedules": []}
    best = None
    M = ", a and b pieces merged into one 2-D H2D copy per chunk (PP_OPT_MERGE_COPIES)"
    for name, pol, graph, smc, merge in (
            ("literal c=2^18 S=2, per-stage streams", 1, 0, 0, 0),
            ("literal c=2^18 S=2, per-chunk streams (paper), CUDA graph", 0, 1, 0, 0),
            ("literal c=2^18 S=2, per-stage streams, CUDA graph", 1, 1, 0, 0),
            ("literal c=2^18 S=2, copies round-robin per direction, CUDA graph", 3, 1, 0, 0),
            ("literal c=2^18 S=2, per-chunk streams, SM-driven copies (PP_OPT_SM_COPY)", 0, 1, 1, 0),
            ("literal c=2^18 S=2, per-stage streams, SM-driven copies (PP_OPT_SM_COPY)", 1, 1, 1, 0),
            ("literal c=2^18 S=2, per-array copy streams (a, b on two copy engines)", 5, 0, 0, 0),
            ("literal c=2^18 S=2, per-array copy streams, CUDA graph", 5, 1, 0, 0),
            ("literal c=2^18 S=2, per-stage streams" + M, 1, 0, 0, 1),
            ("literal c=2^18 S=2, per-stage streams, CUDA graph" + M, 1, 1, 0, 1),
            ("literal c=2^18 S=2, per-chunk streams (paper), CUDA graph" + M, 0, 1, 0, 1)):
        with pp.Region(cx.dev) as r:
            r.map("to", ha)
            r.map("to", hb)
            r.map("from", hc)
            r.pipeline(1 << 18, 2)
            r.set_option(pp.PP_OPT_STREAM_POLICY, pol)
            r.set_option(pp.PP_OPT_GRAPH, graph)
            r.set_option(pp.PP_OPT_SM_COPY, (4 << 20) if smc else 0)
            r.set_option(pp.PP_OPT_MERGE_COPIES, merge)
            synth.fill_sentinel(hc)
            per = cx.timed(lambda: r.launch(0, n, "triad", s=3.0), steps, 5)
            q = r.query()
        st = stats(per)
        roof = link_roofline(probes, q["h2d_bytes"], q["d2h_bytes"], st["mean_ms"] * 1e-3)
        rec = {"schedule": name, "gbs": (q["h2d_bytes"] + q["d2h_bytes"]) / (st["mean_ms"] * 1e-3) / 1e9,
               **{k: v for k, v in st.items() if k != "steps_ms"}, "frac": roof["frac"],
               "nchunks": q["nchunks"], "ring_bytes": q["ring_bytes"], "graph_replayed": bool(q["graph_replayed"]),
               "copy_jobs": q["n_h2d"] + q["n_d2h"] - q["merged_copies"],
               "bit_identical_to_resident": bool(torch.equal(hc.view(torch.int32), ref.view(torch.int32)))}
        out["schedules"].append(rec)
        if best is None or rec["mean_ms"] < best[0]["mean_ms"]:
            best = (rec, q, roof)
    rec, q, roof = best
    with pp.Region(cx.dev) as rn:
        rn.map("to", ha)
        rn.map("to", hb)
        rn.map("from", hc)
        pn = cx.timed(lambda: rn.naive(0, n, "triad", s=3.0), steps, 5)
        qn = rn.query()
    out.update({"e2e_gbs": rec["gbs"], "ms_per_step": rec["mean_ms"], "schedule": rec["schedule"],
                "h2d_bytes_per_step": q["h2d_bytes"], "d2h_bytes_per_step": q["d2h_bytes"],
                "link_roofline": roof, "fill_drain_cap": 4 / 5,
                "naive_ms": statistics.mean(pn), "speedup_vs_naive": statistics.mean(pn) / rec["mean_ms"],
                "hbm_saved": 1.0 - q["ring_bytes"] / qn["naive_bytes"],
                "gpu_launches_per_step": q["n_kernels"],
                "gpu_launches": (len(out["schedules"]) + 1) * steps * q["n_kernels"]})
    return out


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
    cx = Ctx(torch, dist, ws, rank, dev, share)
    if ws > 1:
        # torchrun exports OMP_NUM_THREADS=1: give the host-side fills and the oracle's verification
        # this rank's share of the cores (its NUMA-local CPUs when bound)
        local_ws = int(os.environ.get("LOCAL_WORLD_SIZE", ws))
        nthr = max(1, (os.cpu_count() or 1) // local_ws)
        if bound_cpus:
            nthr = min(nthr, len(bound_cpus))
        synth.set_threads(nthr)
        import oracle
        oracle.set_threads(nthr)
    launches = 0

    n = args.n
    tdt = torch.float64 if args.dtype == "f64" else torch.float32
    esz = 8 if args.dtype == "f64" else 4
    plane = n * n * esz
    c0 = (np.float64(1) / 6) if tdt == torch.float64 else float(np.float32(1) / np.float32(6))
    c1 = (np.float64(c0) / 6) if tdt == torch.float64 else float(np.float32(c0) / np.float32(6))
    c0, c1 = float(c0), float(c1)

    clk = Clocks(dev)
    with clk:
        settle = [cx.settle_link(pp)]
        probes = [cx.probe(pp)]
        # ---------------- configs[2]/[3]: host array larger than HBM (first: the largest host
        # allocation is made while host memory is unfragmented, and released before the rest) ------
        ooc = None
        if args.ooc != "off":
            ooc = ooc_leg(args, cx, pp, synth, probes)
            launches += ooc.get("gpu_launches_per_sweep", 0) * ooc.get("steps", 0)

        # ---------------- configs[1] arrays: global array of ws*(n-2)+2 planes; this rank's loop
        # slab [lo_g, hi_g) and its host planes
        nz_g = ws * (n - 2) + 2
        lo_g, hi_g = pp.pp_partition(1, nz_g - 1, ws, rank)
        p0 = lo_g - 1                  # first plane this rank's host slab holds
        nzl = hi_g - lo_g + 2
        A0 = torch.empty((nzl, n, n), dtype=tdt, pin_memory=True)
        An = torch.empty((nzl, n, n), dtype=tdt, pin_memory=True)
        synth.fill(A0, "random", seed=synth.SEED_A, g0=p0 * n * n, nx=n, ny=n)
        synth.fill_sentinel(An)
        lo, hi = 1, nzl - 1            # local loop range (global [lo_g, hi_g))
        iters = hi - lo
        B_in = nzl * plane             # distinct input planes (halo reuse: each copied once)
        B_out = iters * plane
        iv = torch.int64 if esz == 8 else torch.int32

        def check_host_output(label):
            """Bit-identity of the pipelined host output with the resident output on every computed
            plane; the sentinel must survive outside [lo, hi)."""
            diff = int((An[lo:hi].view(iv) != hN[lo:hi].view(iv)).sum())
            sent = torch.empty_like(An[:1])
            synth.fill_sentinel(sent)
            untouched = all(torch.equal(An[k:k + 1].view(iv), sent.view(iv)) for k in range(nzl) if k < lo or k >= hi)
            synth.fill_sentinel(An)    # the next leg starts from the sentinel again
            return {"leg": label, "planes_checked": hi - lo, "mismatches": diff, "sentinel_intact": bool(untouched)}

        # ---------------- value: resident in HBM --------------------------------------------
        dA = A0.to(f"cuda:{dev}")
        dN = torch.empty_like(dA)
        rv = pp.Region(dev)
        rv.map("to", dA, -1, 3)
        rv.map("from", dN)
        rv.pipeline(0, 1)              # auto chunk: one chunk for resident arrays
        rv.use_streams([cx.stream.cuda_stream])
        per_v = cx.timed(lambda: rv.launch_async(lo, hi, "stencil7", c0=c0, c1=c1), args.steps, args.warmup)
        rv.wait()
        # the kernel's own duration for the roofline: the same launches again, each one's CUDA events
        _, kern_v = cx.timed_lib(rv, lambda: rv.launch_async(lo, hi, "stencil7", c0=c0, c1=c1), args.steps, 1)
        info_v = rv.query()
        st_v = stats(per_v)
        ms_v = st_v["mean_ms"]
        value = ws * (B_in + B_out) / (ms_v * 1e-3) / 1e9
        kernel_path = info_v["kernel_path"]
        launches += 2 * args.steps * info_v["n_kernels"]   # the value loop and the kernel-timing loop
        hN = dN.cpu()
        kernels = None
        if ws == 1 and args.dtype == "f64":
            kernels = kernels_leg(args, cx, pp, synth, json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
                                  if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0, dA, dN)
            launches += sum(2 * max(5, args.steps) for _ in kernels)
        # ---------------- e2e: pinned host arrays through the C ABI ---------------------------
        # configs[1]'s device budget: the ring of `chunk` planes x `streams` in flight (8 + 6 planes
        # = 28 MiB for c=2, S=3); within it the runtime picks the chunk size with
        # pp_autotune unless --no-autotune (then the literal c, S)
        ring_budget = ((args.streams * args.chunk + 2) + args.streams * args.chunk) * plane
        torch.cuda.synchronize()
        free0 = torch.cuda.mem_get_info(dev)[0]
        re = pp.Region(dev)
        re.map("to", A0, -1, 3)
        re.map("from", An)
        re.pipeline(args.chunk, args.streams)
        re.set_option(pp.PP_OPT_STREAM_POLICY, args.policy)
        re.set_option(pp.PP_OPT_GRAPH, args.graph)
        re.mem_limit(ring_budget)
        tune = None
        if not args.no_autotune:
            tune = re.autotune(lo, hi, "stencil7", trials=8, c0=c0, c1=c1)
        synth.fill_sentinel(An)
        settle.append(cx.settle_link(pp))   # the > HBM leg just released ~190 GB of host memory
        per_e = cx.timed(lambda: re.launch(lo, hi, "stencil7", c0=c0, c1=c1), args.steps, args.warmup)
        info_e = re.query()
        used_e = free0 - torch.cuda.mem_get_info(dev)[0]
        st_e = stats(per_e)
        ms_e = st_e["mean_ms"]
        e2e = ws * (info_e["h2d_bytes"] + info_e["d2h_bytes"]) / (ms_e * 1e-3) / 1e9
        launches += args.steps * info_e["n_kernels"]
        verified = [check_host_output("e2e headline (the timed schedule)")] if args.verify else []
        copy_bytes = info_e["chunk_size"] * plane
        copy_probe = cx.probe(pp, copy_bytes, 16)
        # ---------------- the same loop under other schedules (context for the headline) -------
        schedules = []
        if not args.no_schedules:
            for name, c, S, pol, gr, mir, intr in (
                    ("literal c=2, 3 chunks in flight, per-stage streams (policy 1)", 2, 3, 1, 0, 1, 0),
                    ("literal c=2 S=3, the paper's per-chunk streams (policy 0)", 2, 3, 0, 0, 1, 0),
                    ("literal c=2 S=3, copies round-robin per direction (policy 3)", 2, 3, 3, 0, 1, 0),
                    ("literal c=2 S=3, per-chunk H2D+kernel streams, CUDA graph (policy 4)", 2, 3, 4, 1, 1, 0),
                    ("c=6, 1 chunk in flight, mirrored rings OFF (wrapping copies split in two)", 6, 1, 1, 0, 0, 0),
                    ("c=6, 1 chunk in flight, whole-plane copy-back (S5)", 6, 1, 1, 0, 1, 0),
                    ("c=6, 1 chunk in flight, interior-only copy-back (S5b, cudaMemcpy3DAsync)", 6, 1, 1, 0, 1, 1),
                    ("c=6, 1 chunk in flight, SM-driven copies (PP_OPT_SM_COPY)", 6, 1, 1, 0, 1, 2),
                    ("c=6, 1 chunk in flight, persistent kernel + flag gates (PP_OPT_PERSISTENT)", 6, 1, 1, 0, 1, 3),
                    ("literal c=2 S=3, persistent kernel + flag gates (PP_OPT_PERSISTENT)", 2, 3, 1, 0, 1, 3),
                    ("auto chunk, S=3, budget = free HBM", 0, 3, 1, 0, 1, 0),
                    ("c=16 S=6 (388 MiB ring)", 16, 6, 1, 0, 1, 0)):
                rs = pp.Region(dev)
                rs.set_option(pp.PP_OPT_MIRROR, mir)
                rs.set_option(pp.PP_OPT_D2H_INTERIOR, 1 if intr == 1 else 0)
                rs.set_option(pp.PP_OPT_SM_COPY, (64 << 20) if intr == 2 else 0)
                rs.set_option(pp.PP_OPT_PERSISTENT, 1 if intr == 3 else 0)
                rs.map("to", A0, -1, 3)
                rs.map("from", An)
                rs.pipeline(c, S)
                rs.set_option(pp.PP_OPT_STREAM_POLICY, pol)
                rs.set_option(pp.PP_OPT_GRAPH, gr)
                ps = stats(cx.timed(lambda: rs.launch(lo, hi, "stencil7", c0=c0, c1=c1), max(3, args.steps // 2), 1))
                qs = rs.query()
                schedules.append({"schedule": name, "chunk": qs["chunk_size"], "streams": qs["num_streams"],
                                  "ring_bytes": qs["ring_bytes"], "copies": qs["n_h2d"] + qs["n_d2h"],
                                  "ms": ps["mean_ms"], "median_ms": ps["median_ms"], "min_ms": ps["min_ms"],
                                  "gbs": ws * (qs["h2d_bytes"] + qs["d2h_bytes"]) / (ps["mean_ms"] * 1e-3) / 1e9})
                rs.close()
            if args.verify:
                verified.append(check_host_output("last alternative schedule (whole planes)"))
        # ---------------- naive synchronous offload -----------------------------------------
        naive = None
        if not args.no_naive:
            torch.cuda.synchronize()
            free_n0 = torch.cuda.mem_get_info(dev)[0]
            rn = pp.Region(dev)
            rn.map("to", A0, -1, 3)
            rn.map("from", An)
            pn = stats(cx.timed(lambda: rn.naive(lo, hi, "stencil7", c0=c0, c1=c1), max(3, args.steps // 2), 1))
            info_n = rn.query()
            used_n = free_n0 - torch.cuda.mem_get_info(dev)[0]
            ms_n = pn["mean_ms"]
            naive = {"ms_per_step": ms_n, "median_ms": pn["median_ms"], "min_ms": pn["min_ms"],
                     "gbs": ws * (info_n["h2d_bytes"] + info_n["d2h_bytes"]) / (ms_n * 1e-3) / 1e9,
                     "phase_ms": {"h2d": info_n["naive_h2d_ms"], "kernel": info_n["naive_kernel_ms"],
                                  "d2h": info_n["naive_d2h_ms"]},
                     "device_bytes": info_n["naive_bytes"],
                     "speedup_pipelined_vs_naive": ms_n / ms_e,
                     "hbm_saved": 1.0 - info_e["ring_bytes"] / info_n["naive_bytes"],
                     "cudaMemGetInfo_used_delta": {"pipelined": used_e, "naive": used_n,
                                                   "hbm_saved": 1.0 - used_e / used_n if used_n > 0 else None}}
            rn.close()
            if args.verify:
                verified.append(check_host_output("naive"))
        # ---------------- NEXT-1: T sweeps per pass over the link ---------------------------------
        temporal = None
        if ws == 1 and not args.no_temporal:
            temporal = temporal_leg(args, cx, pp, A0, An, lo, hi, c0, c1, ms_e, probes)
            launches += sum(t["launches_per_pass"] * max(3, args.steps // 2) for t in temporal)
            synth.fill_sentinel(An)
        # ---------------- configs[0] triad ------------------------------------------------------
        triad = None
        if not args.no_triad and ws == 1:
            triad = triad_leg(args, cx, pp, synth, probes)
            launches += triad["gpu_launches"]
        probes.append(cx.probe(pp))
    clocks = clk.summary()

    # ---------------- link roofline (configs[1] e2e) --------------------------------------------
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {"hbm_gbs": 6650.0}
    hbm_peak = peaks["hbm_gbs"]
    hbm_src = "measured" if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else "fallback"
    # N > 1: each rank streams its own slab through its own link concurrently, so the job's roofline
    # is the slowest rank's (max over ranks), compared with the max-over-ranks e2e time
    link_roof = link_roofline(probes, info_e["h2d_bytes"], info_e["d2h_bytes"], ms_e * 1e-3,
                              b_hbm=B_in + B_out, hbm_peak=hbm_peak, t_roof_reduce=lambda x: cx.reduce(x, "max"))
    # the same bound at the schedule's own copy size: one chunk's copy (c planes) alone and duplex, best
    # of 16 — what the copy engines deliver per copy of that size, per-copy setup included
    if copy_probe is not None:
        cb_h2d = max(copy_probe["h2d"], copy_probe["duplex_h2d"])
        cb_d2h = max(copy_probe["d2h"], copy_probe["duplex_d2h"])
        t_cs = cx.reduce(max(info_e["h2d_bytes"] / (cb_h2d * 1e9), info_e["d2h_bytes"] / (cb_d2h * 1e9)), "max")
        t_csd = cx.reduce(max(info_e["h2d_bytes"] / (copy_probe["duplex_h2d"] * 1e9),
                              info_e["d2h_bytes"] / (copy_probe["duplex_d2h"] * 1e9)), "max")
        link_roof["at_copy_size"] = {"copy_bytes": copy_bytes, "h2d_gbs": cb_h2d, "d2h_gbs": cb_d2h,
                                     "t_ms": t_cs * 1e3, "frac": t_cs / (ms_e * 1e-3),
                                     "t_duplex_ms": t_csd * 1e3, "frac_of_duplex": t_csd / (ms_e * 1e-3),
                                     "probe": copy_probe,
                                     "note": "one copy of the schedule's size (c planes), alone and both directions "
                                             "at once, best of 16: the steady state moves both at once"}
    link_roof["probe"] = ("pinned cudaMemcpyAsync 512 MiB, best of 8, each direction alone and both at once, "
                          "at the start and the end of the run"
                          + (f"; all {ws} ranks probing at once, roofline = the slowest rank's" if ws > 1 else ""))
    link_roof["probes"] = probes

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
        ms_k = stats(kern_v)["mean_ms"]
        rec = {
            "metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_v, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": args.dtype, "data": "synthetic (counter-based U[0,1), seed 2017)",
            "config": dict(workload_config(args, ws), numa_bound_cpus=len(bound_cpus) if bound_cpus else None),
            "value_stats": st_v,
            "roofline": {"bound": "hbm", "achieved": kernel_bytes / (ms_k * 1e-3) / 1e9, "peak": hbm_peak,
                         "unit": "GB/s", "frac": kernel_bytes / (ms_k * 1e-3) / 1e9 / hbm_peak,
                         "kernel_ms": ms_k, "kernel_ms_stats": stats(kern_v),
                         "kernel_timing": "the launch's own CUDA events on its stream (library t0/t1 around the "
                                          "single kernel of a resident launch), over a second timed loop of the "
                                          "same launches; value / ms_per_step include the host's per-launch "
                                          "wait and enqueue",
                         "frac_of_step": kernel_bytes / (ms_v * 1e-3) / 1e9 / hbm_peak,
                         "traffic": ncu_traffic(os.path.join(ROOT, "profiles", "r2_ncu_stencil7_tma_raw.csv")),
                         "traffic_source": "profiles/r2_ncu_stencil7_tma_raw.csv (ncu --set full, same resident launch)",
                         "kernel": "stencil7 " + {1: "generic", 2: "tma"}.get(kernel_path, "?"),
                         "peak_source": f"{hbm_src} (MEASURED_PEAKS.json hbm_gbs)",
                         "algorithmic_bytes_per_launch": kernel_bytes},
            "e2e": {"value": e2e, "unit": "GB/s", "h2d_bytes_per_step": info_e["h2d_bytes"],
                    "d2h_bytes_per_step": info_e["d2h_bytes"], "ms_per_step": ms_e,
                    "median_ms": st_e["median_ms"], "min_ms": st_e["min_ms"],
                    "chunk": info_e["chunk_size"], "chunks_in_flight": info_e["num_streams"],
                    "device_budget_bytes": ring_budget, "autotune": tune,
                    "graph_replayed": bool(info_e["graph_replayed"]),
                    "chunks": info_e["nchunks"], "ring_planes": info_e["ring_planes"],
                    "ring_bytes": info_e["ring_bytes"], "cudaMemGetInfo_used_delta": used_e,
                    "library_ms": info_e["last_ms"], "link_roofline": link_roof, "schedules": schedules},
            "ooc": ooc,
            "triad": triad,
            "kernels": kernels,
            "temporal": temporal,
            "naive": naive,
            "cpu_baseline": cpu,
            "verify": verified,
            "clocks": clocks,
            "link_settle": settle,
            "gpu_launches": launches,
            "gpu_launches_detail": {"value_per_step": info_v["n_kernels"], "e2e_per_step": info_e["n_kernels"],
                                    "ooc_per_sweep": (ooc or {}).get("gpu_launches_per_sweep")},
        }
        print(json.dumps(rec))
    rv.close()
    re.close()
    if ws > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
