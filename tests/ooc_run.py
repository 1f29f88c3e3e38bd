#!/usr/bin/env python3
"""Out-of-core sweep (BASELINE.json configs[2]): 3-D fp32 7-point stencil over a host array LARGER
THAN THE GPU's HBM, 4 GB device budget, 3 streams, one GPU.

The box has ~196 GiB of host RAM against ~179 GiB of HBM, so input + output cannot both be held:
the sweep runs in the library's in-place mode (PP_OPT_INPLACE, reading S24) — outputs overwrite
the input planes on the host after they have been copied in. Inputs are the counter-based field
(synth/), so verification regenerates the original planes block by block and checks EVERY output
plane bit-for-bit with the oracle's verify-in-place (no third array).

Test infrastructure (it lives under tests/ because it runs the CPU oracle to verify the GPU output;
the product path never imports oracle/). tests/test_gpu_parity.py runs it at 16 GB; the full-size
runs behind profiles/r1_ooc_*.json use --gb auto.

usage: python tests/ooc_run.py [--gb auto|N] [--nx 4096 --ny 4096] [--budget 4e9] [--chunk 8] [--streams 3]

BASELINE.json configs[3] (the same sweep slab-partitioned over G GPUs): launch it with torchrun, one
rank per GPU. Rank g pipelines the contiguous slab [lo_g, hi_g) of the global loop (pp_partition)
through its own link, from its own host buffer of global planes [lo_g - 1, hi_g + 1) generated at
their global indices — the two halo planes are re-read copies, no data moves between GPUs
(SURVEY.md §8(e)). Each rank verifies its own planes; rank 0 prints one line with the aggregate
bytes over the max-over-ranks time. PP_BENCH_SHARE_GPU=1 puts every rank on cuda:0 (functional
test on a one-GPU box, not a scaling measurement). Single sweeps only (T = 1): a multi-sweep slab
would need T-plane halos.
"""
import argparse
import ctypes
import json
import math
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_ipps_cuissf17_b200 as pp  # noqa: E402
import synth  # noqa: E402


def hbm_total_bytes():
    # from nvidia-smi, so no CUDA context (and its host allocations) exists before the big array
    import subprocess
    out = subprocess.run(["nvidia-smi", "--query-gpu=memory.total", "--format=csv,noheader,nounits", "-i", "0"],
                         capture_output=True, text=True).stdout.strip()
    return int(float(out.splitlines()[0])) * (1 << 20)


def meminfo(key):
    for line in open("/proc/meminfo"):
        if line.startswith(key + ":"):
            return int(line.split()[1]) * 1024
    return 0


def alloc_huge(nbytes):
    """Anonymous mapping advised for transparent huge pages, so the pinned host array is made of
    2 MiB pages: with 4 KiB pages the copy engines' host-address translation collapses (measured
    11-21 GB/s instead of ~50 GB/s per direction on a 192 GB array)."""
    import mmap
    m = mmap.mmap(-1, nbytes, flags=mmap.MAP_PRIVATE | mmap.MAP_ANONYMOUS)
    try:
        m.madvise(mmap.MADV_HUGEPAGE)
    except (AttributeError, OSError):
        pass
    return m


def dist_setup():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    dev = 0 if os.environ.get("PP_BENCH_SHARE_GPU") == "1" else local
    if ws > 1:
        import torch.distributed as dist
        dist.init_process_group("gloo")          # only timing scalars and counts cross ranks
    return ws, rank, dev


def reduce(x, op):
    import torch
    import torch.distributed as dist
    t = torch.tensor([float(x)], dtype=torch.float64)
    dist.all_reduce(t, op={"max": dist.ReduceOp.MAX, "sum": dist.ReduceOp.SUM, "min": dist.ReduceOp.MIN}[op])
    return float(t.item())


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gb", default="auto")
    ap.add_argument("--nx", type=int, default=4096)
    ap.add_argument("--ny", type=int, default=4096)
    ap.add_argument("--budget", type=float, default=4e9)
    ap.add_argument("--chunk", type=int, default=8)
    ap.add_argument("--streams", type=int, default=3)
    ap.add_argument("--policy", type=int, default=1)
    ap.add_argument("--verify", default="all", choices=["all", "sample", "none"])
    ap.add_argument("--headroom-gb", type=float, default=10.0)
    ap.add_argument("--sweeps", type=int, default=1, help="timed sweeps (verification needs exactly 1)")
    ap.add_argument("--trace", action="store_true", help="per-chunk copy bandwidth profile of the last sweep")
    ap.add_argument("--alloc", default="mmap-huge", choices=["mmap-huge", "numpy"])
    ap.add_argument("--T", type=int, default=1, help="Jacobi sweeps per pass (PP_OPT_SWEEPS, temporal blocking)")
    ap.add_argument("--fuse", type=int, default=1, help="levels per fused kernel pass (PP_OPT_FUSE)")
    ap.add_argument("--verify-blocks", type=int, default=12, help="light-cone blocks verified when T > 1")
    a = ap.parse_args()
    import oracle
    ws, rank, dev = dist_setup()
    if ws > 1 and a.T > 1:
        raise SystemExit("multi-rank runs are single sweeps (a T-sweep slab needs T-plane halos)")
    nx, ny = a.nx, a.ny
    plane = nx * ny * 4
    hbm = hbm_total_bytes()
    avail = meminfo("MemAvailable")
    if a.gb == "auto":
        nz = math.ceil(hbm * 1.005 / plane) + 2
    else:
        nz = int(float(a.gb) * 1e9 // plane)
    # every rank on this host holds its slab plus two halo planes
    limit = int((avail - a.headroom_gb * 1e9) // plane) - 2 * (ws - 1)
    capped = nz > limit
    nz_global = min(nz, limit)
    if ws > 1:
        # every rank must partition the same global array: ranks read MemAvailable at slightly
        # different moments, so agree on the smallest size before anyone allocates
        nz_global = int(reduce(nz_global, "min"))
    lo_g, hi_g = pp.pp_partition(1, nz_global - 1, ws, rank)
    p0 = lo_g - 1                              # global index of local plane 0
    nz = hi_g - lo_g + 2                       # local planes [0, nz): global [lo_g - 1, hi_g + 1)
    total = nz * plane
    rec = {"workload": f"BASELINE.json configs[{2 if ws == 1 else 3}]: in-place fp32 7-point stencil "
                       f"[{nz_global}][{ny}][{nx}] ({nz_global * plane / 1e9:.1f} GB host array)"
                       + (f", slab-partitioned over {ws} ranks" if ws > 1 else "")
                       + f", {a.budget / 1e9:.0f} GB device budget per GPU",
           "host_array_bytes": nz_global * plane, "hbm_total_bytes": hbm, "exceeds_hbm": nz_global * plane > hbm,
           "host_mem_available": avail, "size_capped_by_host_ram": capped, "ranks": ws}
    if ws > 1:
        rec["rank0_slab"] = [lo_g, hi_g]
    t = time.time()
    huge0 = meminfo("AnonHugePages")
    if a.alloc == "mmap-huge":
        buf = alloc_huge(total)
        A = np.frombuffer(buf, dtype=np.float32).reshape(nz, ny, nx)
    else:
        A = np.empty((nz, ny, nx), dtype=np.float32)
    synth.fill(A, "random", seed=synth.SEED_A, g0=p0 * ny * nx, nx=nx, ny=ny)
    rec["generate_s"] = time.time() - t
    rec["anon_hugepages_bytes"] = meminfo("AnonHugePages") - huge0
    rec["alloc"] = a.alloc
    try:
        rec["thp"] = open("/sys/kernel/mm/transparent_hugepage/enabled").read().strip()
    except OSError:
        pass
    c0 = float(np.float32(1) / np.float32(6))
    c1 = float(np.float32(c0) / np.float32(6))

    # warm-up on a small separate array (kernel path, TMA descriptors, streams)
    W = np.empty((24, ny, nx), dtype=np.float32)
    synth.fill(W, "random", seed=7, nx=nx, ny=ny)
    with pp.Region(dev) as rw:
        rw.set_option(pp.PP_OPT_INPLACE, 1)
        rw.map("to", W, -1, 3)
        rw.map("from", W)
        rw.pipeline(a.chunk, a.streams)
        rw.mem_limit(int(a.budget))
        rw.set_option(pp.PP_OPT_SWEEPS, a.T)
        rw.set_option(pp.PP_OPT_FUSE, min(a.fuse, a.T))
        rw.launch(1, 23, "stencil7", c0=c0, c1=c1)
    del W

    r = pp.Region(dev)
    r.set_option(pp.PP_OPT_INPLACE, 1)
    r.set_option(pp.PP_OPT_STREAM_POLICY, a.policy)
    r.set_option(pp.PP_OPT_SWEEPS, a.T)
    r.set_option(pp.PP_OPT_FUSE, min(a.fuse, a.T))
    t = time.time()
    r.map("to", A, -1, 3)                     # page-locks the array (cudaHostRegister)
    r.map("from", A)
    rec["pin_s"] = time.time() - t
    r.pipeline(a.chunk, a.streams)
    r.mem_limit(int(a.budget))
    sweeps_ms = []
    for it in range(a.sweeps):
        if a.trace and it == a.sweeps - 1:
            r.set_option(pp.PP_OPT_TRACE, 1)
        if ws > 1:
            reduce(0, "max")                   # barrier: all ranks start together
        t = time.time()
        r.launch(1, nz - 1, "stencil7", c0=c0, c1=c1)
        wall = time.time() - t
        sweeps_ms.append(r.query()["last_ms"] if ws == 1 else reduce(r.query()["last_ms"], "max"))
    q = r.query()
    if a.trace:
        tr = r.trace()
        # bandwidth of each copy while it ran, by position in the array (deciles)
        prof = {}
        for kind in ("H2D", "D2H"):
            ops = [t for t in tr if t["kind"] == kind]
            dec = []
            for d in range(10):
                part = ops[d * len(ops) // 10:(d + 1) * len(ops) // 10]
                if part:
                    dec.append(round(sum(t["bytes"] for t in part) / (sum(t["end_ms"] - t["start_ms"] for t in part) * 1e-3) / 1e9, 1))
            prof[kind + "_gbs_by_decile"] = dec
        prof["launch_ms_by_decile"] = [round(t["end_ms"], 1) for t in tr if t["kind"] == "KER"][:: max(1, q["nchunks"] // 10)]
        rec["trace_profile"] = prof
    r.close()                                  # unregisters the host array
    ms = sweeps_ms[-1]                         # max over ranks when ws > 1
    rec["sweeps_ms"] = sweeps_ms
    if ws > 1:
        reduce(0, "max")                       # all ranks probe their links at once
    link = pp.pp_probe_link(dev, 256 << 20, 5)
    B_in, B_out = q["h2d_bytes"], q["d2h_bytes"]
    t_roof = max(B_in / (link["h2d"] * 1e9), B_out / (link["d2h"] * 1e9))
    t_roof_dx = max(B_in / (link["duplex_h2d"] * 1e9), B_out / (link["duplex_d2h"] * 1e9))
    if ws > 1:                                 # the job: every rank's bytes, the slowest rank's roofline
        t_roof, t_roof_dx = reduce(t_roof, "max"), reduce(t_roof_dx, "max")
        B_in, B_out = reduce(B_in, "sum"), reduce(B_out, "sum")
    rec.update({"sweep_ms": ms, "sweep_wall_s": wall, "e2e_gbs": (B_in + B_out) / (ms * 1e-3) / 1e9,
                "h2d_bytes": B_in, "d2h_bytes": B_out, "chunk": q["chunk_size"], "streams": q["num_streams"],
                "nchunks": q["nchunks"], "ring_planes": q["ring_planes"], "ring_bytes": q["ring_bytes"],
                "device_fraction_of_array": q["ring_bytes"] / total, "link": link,
                "t_roof_ms": t_roof * 1e3, "frac_of_roofline": t_roof / (ms * 1e-3),
                "frac_of_duplex_roofline": t_roof_dx / (ms * 1e-3), "kernel_path": q["kernel_path"]})

    rec["sweeps_per_pass"] = a.T
    rec["fuse"] = min(a.fuse, a.T)
    rec["jacobi_sweeps_per_s"] = a.T / (ms * 1e-3)
    rec["effective_gbs"] = a.T * (B_in + B_out) / (ms * 1e-3) / 1e9
    # T > 1: verify sampled blocks by the light cone — output plane k depends only on input planes
    # [k-T, k+T], so sweeping a regenerated block [b0, b1) with its end planes held fixed reproduces
    # the true A^T exactly on planes at distance > T from both block ends (or at the real boundary)
    if a.verify != "none" and a.sweeps == 1 and a.T > 1:
        # windowed light cone: an output point depends only on inputs within distance T in every
        # dimension, so a small (x, y, z) sub-block regenerated from the counter-based generator and
        # swept T times with its faces held fixed reproduces the true A^T on points farther than T
        # from the sub-block's faces (or at the array's real boundaries, which match exactly)
        t = time.time()
        T = a.T
        w = 64
        bad = checked = 0
        rng = np.random.default_rng(5)
        for blkno in range(a.verify_blocks):
            kc = int(rng.integers(1, nz - 1))
            jc = int(rng.integers(0, ny - w)) if blkno % 2 else 0          # every other block on the y=0 edge
            ic = int(rng.integers(0, nx - w)) if blkno % 3 else nx - w      # some on the x = nx-1 edge
            k0, k1 = max(0, kc - T - 1), min(nz, kc + T + 2)
            j0, j1 = max(0, jc - T - 1), min(ny, jc + w + T + 1)
            i0, i1 = max(0, ic - T - 1), min(nx, ic + w + T + 1)
            blk = np.empty((k1 - k0, j1 - j0, i1 - i0), dtype=np.float32)
            for k in range(k0, k1):
                for j in range(j0, j1):
                    synth.fill(blk[k - k0, j - j0], "random", seed=synth.SEED_A, g0=(k * ny + j) * nx + i0,
                               nx=nx, ny=ny)
            ref = blk.copy()
            # sweep the block's interior planes; planes 0 and nz-1 of the array stay fixed as in the run
            oracle.stencil7_sweeps(blk, ref, 1, k1 - k0 - 1, c0, c1, T)
            # exact where the light cone stays inside the block or hits the array's real faces
            kk = [k for k in range(k0, k1) if (k - k0 > T or k0 == 0) and (k1 - 1 - k > T or k1 == nz) and 1 <= k < nz - 1]
            jj = [j for j in range(j0, j1) if (j - j0 > T or j0 == 0) and (j1 - 1 - j > T or j1 == ny)]
            ii = [i for i in range(i0, i1) if (i - i0 > T or i0 == 0) and (i1 - 1 - i > T or i1 == nx)]
            if not (kk and jj and ii):
                continue
            sub_ref = ref[kk[0] - k0:kk[-1] - k0 + 1, jj[0] - j0:jj[-1] - j0 + 1, ii[0] - i0:ii[-1] - i0 + 1]
            sub_got = A[kk[0]:kk[-1] + 1, jj[0]:jj[-1] + 1, ii[0]:ii[-1] + 1]
            bad += int(np.count_nonzero(sub_ref.view(np.uint32) != np.ascontiguousarray(sub_got).view(np.uint32)))
            checked += sub_ref.size
        rec["verify"] = {"points_checked": checked, "mismatches": bad,
                         "mode": f"windowed light-cone sub-blocks x{a.verify_blocks} (64x64 core, T-wide halo)",
                         "seconds": time.time() - t}
    # verification: regenerate original inputs block by block, compare every output plane's bits
    if a.verify != "none" and a.sweeps == 1 and a.T == 1:
        t = time.time()
        B = 14
        bad = 0
        checked = 0
        ks = list(range(1, nz - 1, B))
        if a.verify == "sample":
            ks = ks[:2] + ks[len(ks) // 2:len(ks) // 2 + 1] + ks[-2:]
        buf = np.empty((B + 2, ny, nx), dtype=np.float32)
        for k0 in ks:
            k1 = min(k0 + B, nz - 1)
            m = k1 - k0
            src = buf[: m + 2]
            synth.fill(src, "random", seed=synth.SEED_A, g0=(p0 + k0 - 1) * ny * nx, nx=nx, ny=ny)
            got = A[k0 - 1:k1 + 1]
            bad += oracle.stencil7_verify(src, got, 1, m + 1, c0, c1)
            checked += m
        edge = np.empty((1, ny, nx), dtype=np.float32)
        for k in (0, nz - 1):                  # planes outside [1, nz-1) must still hold the input
            synth.fill(edge, "random", seed=synth.SEED_A, g0=(p0 + k) * ny * nx, nx=nx, ny=ny)
            bad += int(np.count_nonzero(edge[0].view(np.uint32) != A[k].view(np.uint32)))
        if ws > 1:
            checked, bad = int(reduce(checked, "sum")), int(reduce(bad, "sum"))
        rec["verify"] = {"planes_checked": checked, "mismatches": int(bad), "mode": a.verify,
                         "seconds": time.time() - t}
    if rank == 0:
        print(json.dumps(rec, default=lambda o: o.item() if hasattr(o, "item") else str(o)), flush=True)


if __name__ == "__main__":
    main()
