#!/usr/bin/env python3
"""Tiny launches over every kernel path, run under compute-sanitizer (memcheck / racecheck /
synccheck) by tools/gpu_round.sh `sanitize`. Exits non-zero on a parity mismatch."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ipps_cuissf17_b200 as pp  # noqa: E402
import synth  # noqa: E402


def main():
    bad = 0
    for dt, path in ((torch.float64, pp.KPATH_TMA), (torch.float32, pp.KPATH_TMA), (torch.float64, pp.KPATH_GENERIC),
                     (torch.int64, pp.KPATH_GENERIC)):
        A0 = torch.empty((9, 20, 24), dtype=dt, pin_memory=True)
        synth.fill(A0, "random", seed=5, nx=24, ny=20)
        An = torch.zeros_like(A0).pin_memory()
        c0, c1 = (3.0, 5.0) if dt == torch.int64 else (1 / 6, 1 / 36)
        if dt == torch.float32:
            c0, c1 = float(np.float32(1) / np.float32(6)), float(np.float32(1) / np.float32(36))
        with pp.Region(0) as r:
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.pipeline(2, 3)
            r.set_option(pp.PP_OPT_KERNEL_PATH, path)
            r.launch(1, 8, "stencil7", c0=c0, c1=c1)
        ref = np.zeros(tuple(A0.shape), dtype=A0.numpy().dtype)
        oracle.stencil7(A0.numpy(), ref, 1, 8, int(c0) if dt == torch.int64 else c0, int(c1) if dt == torch.int64 else c1)
        bad += int(not np.array_equal(An.numpy()[1:8], ref[1:8]))
    n = 1000
    ab = torch.rand(2 * n, dtype=torch.float32).pin_memory()   # a | b in one buffer: merged 2-D copies
    a, b = ab[:n], ab[n:]
    for merge in (0, 1):
        c = torch.zeros(n, dtype=torch.float32).pin_memory()
        with pp.Region(0) as r:
            r.map("to", a)
            r.map("to", b)
            r.map("from", c)
            r.pipeline(256, 2)
            r.set_option(pp.PP_OPT_MERGE_COPIES, merge)
            r.set_option(pp.PP_OPT_MIRROR, 0)
            r.launch(0, n, "triad", s=3.0)
            bad += int(r.query()["merged_copies"] != (4 if merge else 0))
        ref = np.zeros(n, np.float32)
        oracle.triad(a.numpy(), b.numpy(), np.float32(3), ref)
        bad += int(not np.array_equal(c.numpy(), ref))
    P = torch.empty((12, 5), dtype=torch.int64, pin_memory=True)
    synth.fill(P, "plane", nx=5, ny=1)
    O = torch.zeros_like(P).pin_memory()
    with pp.Region(0) as r:
        r.map("to", P, -1, 3)
        r.map("from", O)
        r.pipeline(3, 2)
        r.launch(1, 11, "probe")
    bad += int(not torch.all(O[1:11] == 13 * torch.arange(1, 11).view(-1, 1) + 8))
    for dt in (torch.float32, torch.float64):
        A = torch.empty((9, 12, 16), dtype=dt, pin_memory=True)
        synth.fill(A, "random", seed=3, nx=16, ny=12)
        B = torch.zeros_like(A).pin_memory()
        with pp.Region(0) as r:
            r.map("to", A, -1, 3)
            r.map("from", B)
            r.pipeline(2, 2)
            r.launch(1, 8, "conv3d")
        ref = np.zeros(tuple(A.shape), dtype=A.numpy().dtype)
        oracle.conv3d(A.numpy(), ref, 1, 8)
        bad += int(not np.array_equal(B.numpy()[1:8], ref[1:8]))
    A0 = torch.empty((14, 10, 16), dtype=torch.float64, pin_memory=True)
    synth.fill(A0, "random", seed=4, nx=16, ny=10)
    An = torch.zeros_like(A0).pin_memory()
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(2, 2)
        r.set_option(pp.PP_OPT_SWEEPS, 3)
        r.launch(1, 13, "stencil7", c0=1 / 6, c1=1 / 36)
    ref = np.zeros(tuple(A0.shape))
    oracle.stencil7_sweeps(A0.numpy(), ref, 1, 13, 1 / 6, 1 / 36, 3)
    bad += int(not np.array_equal(An.numpy()[1:13], ref[1:13]))
    # fused multi-level chains (PP_OPT_FUSE): several tiles and z-segments, both dtypes
    for dt, L in ((torch.float64, 2), (torch.float32, 4), (torch.float64, 3)):
        A0 = torch.empty((16, 40, 136), dtype=dt, pin_memory=True)
        synth.fill(A0, "random", seed=6, nx=136, ny=40)
        An = torch.zeros_like(A0).pin_memory()
        c0, c1 = (1 / 6, 1 / 36) if dt == torch.float64 else (float(np.float32(1) / np.float32(6)),
                                                             float(np.float32(1) / np.float32(36)))
        with pp.Region(0) as r:
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.pipeline(3, 2)
            r.set_option(pp.PP_OPT_SWEEPS, 5)
            r.set_option(pp.PP_OPT_FUSE, L)
            r.launch(1, 15, "stencil7", c0=c0, c1=c1)
        ref = np.zeros(tuple(A0.shape), dtype=A0.numpy().dtype)
        oracle.stencil7_sweeps(A0.numpy(), ref, 1, 15, c0, c1, 5)
        bad += int(not np.array_equal(An.numpy()[1:15], ref[1:15]))
    # mirrored rings (PP_OPT_MIRROR): 2 MiB planes, so each ring is whole VMM granules and the chunks
    # that wrap are copied in one piece through the second mapping
    A0 = torch.empty((12, 512, 512), dtype=torch.float64, pin_memory=True)
    synth.fill(A0, "random", seed=7, nx=512, ny=512)
    An = torch.zeros_like(A0).pin_memory()
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(3, 1)
        r.launch(1, 11, "stencil7", c0=1 / 6, c1=1 / 36)
        q = r.query()
    ref = np.zeros(tuple(A0.shape))
    oracle.stencil7(A0.numpy(), ref, 1, 11, 1 / 6, 1 / 36)
    bad += int(not np.array_equal(An.numpy()[1:11], ref[1:11])) + int(q["n_h2d"] != q["nchunks"])
    # round 2 paths: conv3d on the TMA path with ragged tiles (FMA-folded terms, paired row chains),
    # interior-only copy-back, SM-driven copies, the pageable bounce ring, slot-tag checks, a peer halo
    for dt in (torch.float32, torch.float64):
        A = torch.empty((10, 40, 136), dtype=dt, pin_memory=True)
        synth.fill(A, "random", seed=8, nx=136, ny=40)
        B = torch.zeros_like(A).pin_memory()
        with pp.Region(0) as r:
            r.map("to", A, -1, 3)
            r.map("from", B)
            r.pipeline(3, 2)
            r.set_option(pp.PP_OPT_KERNEL_PATH, pp.KPATH_TMA)
            r.set_option(pp.PP_OPT_DEBUG_TAGS, 1)
            r.launch(1, 9, "conv3d")
            bad += int(r.query()["debug_violations"] != 0)
        ref = np.zeros(tuple(A.shape), dtype=A.numpy().dtype)
        oracle.conv3d(A.numpy(), ref, 1, 9)
        bad += int(not np.array_equal(B.numpy()[1:9], ref[1:9]))
    A0 = torch.empty((9, 20, 24), dtype=torch.float64, pin_memory=True)
    synth.fill(A0, "random", seed=9, nx=24, ny=20)
    for opt, val in ((pp.PP_OPT_D2H_INTERIOR, 1), (pp.PP_OPT_SM_COPY, 1 << 20)):
        An = torch.zeros_like(A0).pin_memory()
        with pp.Region(0) as r:
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.pipeline(2, 3)
            r.set_option(opt, val)
            r.launch(1, 8, "stencil7", c0=1 / 6, c1=1 / 36)
        ref = np.zeros(tuple(A0.shape))
        if opt == pp.PP_OPT_D2H_INTERIOR:
            oracle.stencil7_fig2(A0.numpy(), ref, 1, 8, 1 / 6, 1 / 36)
        else:
            oracle.stencil7(A0.numpy(), ref, 1, 8, 1 / 6, 1 / 36)
        bad += int(not np.array_equal(An.numpy()[1:8], ref[1:8]))
    Ap = A0.numpy().copy()                         # pageable, through the bounce ring
    Bp = np.zeros_like(Ap)
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_AUTO_PIN, 0)
        r.map("to", Ap, -1, 3)
        r.map("from", Bp)
        r.pipeline(2, 2)
        r.launch(1, 8, "stencil7", c0=1 / 6, c1=1 / 36)
    ref = np.zeros(tuple(A0.shape))
    oracle.stencil7(A0.numpy(), ref, 1, 8, 1 / 6, 1 / 36)
    bad += int(not np.array_equal(Bp[1:8], ref[1:8]))
    side = torch.zeros((20, 24), dtype=torch.float64, device="cuda")
    flag = torch.zeros(1, dtype=torch.int32, device="cuda")
    lo_b, up_b = A0[0:6].clone().pin_memory(), A0[4:9].clone().pin_memory()   # slabs [1,5) and [5,8)
    lo_o, up_o = torch.zeros_like(lo_b).pin_memory(), torch.zeros_like(up_b).pin_memory()
    lo_b[-1].fill_(7.0)                            # the upper halo must come from the peer's side slot
    with pp.Region(0) as rl, pp.Region(0) as ru:
        for r, hb, ob in ((rl, lo_b, lo_o), (ru, up_b, up_o)):
            r.map("to", hb, -1, 3)
            r.map("from", ob)
            r.pipeline(2, 2)
        ru.halo_export(0, 1, side.data_ptr(), flag.data_ptr(), 1)
        rl.halo_import(0, 5, side.data_ptr(), 0, flag.data_ptr(), 1)
        ru.launch_async(1, 4, "stencil7", c0=1 / 6, c1=1 / 36)
        rl.launch_async(1, 5, "stencil7", c0=1 / 6, c1=1 / 36)
        ru.wait()
        rl.wait()
    bad += int(not np.array_equal(lo_o.numpy()[1:5], ref[1:5])) + int(not np.array_equal(up_o.numpy()[1:4], ref[5:8]))
    print("sanitize cases mismatches:", bad)
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()
