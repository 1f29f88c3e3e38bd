"""Host-side logic of bench.py (CPU only): the link roofline from several probes, per-step statistics,
and the out-of-core verification (`ooc_verify`) that the driver-visible configs[2] record relies on."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
import oracle  # noqa: E402
import synth  # noqa: E402


def test_link_roofline_takes_the_best_rate_per_direction():
    probes = [{"h2d": 55.0, "d2h": 46.0, "duplex_h2d": 50.0, "duplex_d2h": 50.0},
              {"h2d": 54.0, "d2h": 47.0, "duplex_h2d": 49.0, "duplex_d2h": 51.0}]
    assert bench.link_capacity(probes) == (55.0, 51.0)
    b_in, b_out = 1.1e9, 1.0e9
    roof = bench.link_roofline(probes, b_in, b_out, 0.025)
    t = max(b_in / 55e9, b_out / 51e9)
    assert abs(roof["t_roof_ms"] - t * 1e3) < 1e-9 and abs(roof["frac"] - t / 0.025) < 1e-12
    # each alone-only / duplex-only bound is never tighter than the combined one
    assert roof["frac_of_alone"] >= roof["frac"] - 1e-12 and roof["frac_of_duplex"] >= roof["frac"] - 1e-12
    # the HBM term binds when it is the slowest stage
    assert bench.link_roofline(probes, 1.0, 1.0, 1.0, b_hbm=6.5e12, hbm_peak=6500.0)["t_roof_ms"] == 1000.0


def test_stats():
    st = bench.stats([3.0, 1.0, 2.0])
    assert st == {"mean_ms": 2.0, "median_ms": 2.0, "min_ms": 1.0, "steps_ms": [3.0, 1.0, 2.0]}
    assert bench.stats(list(range(1, 20)))["steps_ms"] is None


def test_ooc_verify_counts_every_wrong_element():
    """ooc_verify regenerates the seeded input block by block and lets the oracle compare every computed
    plane of an in-place result; boundary planes must still hold the input."""
    nz, ny, nx = 37, 9, 12
    p0 = 5                                            # global index of local plane 0 (a slab)
    A = np.empty((nz, ny, nx), np.float32)
    synth.fill(A, "random", seed=synth.SEED_A, g0=p0 * ny * nx, nx=nx, ny=ny)
    c0 = float(np.float32(1) / np.float32(6))
    c1 = float(np.float32(c0) / np.float32(6))
    out = A.copy()
    oracle.stencil7(A, out, 1, nz - 1, c0, c1)        # what an in-place sweep leaves on the host
    assert bench.ooc_verify(out, p0, c0, c1, oracle, synth) == (nz - 2, 0)
    bad = out.copy()
    bad.view(np.uint32)[17, 4, 5] ^= 1                # one flipped bit in a computed plane
    bad.view(np.uint32)[0, 0, 0] ^= 1                 # and one in the boundary plane
    assert bench.ooc_verify(bad, p0, c0, c1, oracle, synth) == (nz - 2, 2)
    wrong_p0 = bench.ooc_verify(out, p0 + 1, c0, c1, oracle, synth)   # another slab's input
    assert wrong_p0[1] > 0


def test_lightcone_verify_checks_a_T_sweep_in_place_pass():
    nz, ny, nx, T = 30, 40, 44, 3
    p0 = 2
    A = np.empty((nz, ny, nx), np.float64)
    synth.fill(A, "random", seed=synth.SEED_A, g0=p0 * ny * nx, nx=nx, ny=ny)
    out = A.copy()
    oracle.stencil7_sweeps(A, out, 1, nz - 1, 1 / 6, 1 / 36, T)
    ck, bad = bench.lightcone_verify(out, p0, T, 1 / 6, 1 / 36, oracle, synth, blocks=8, w=16)
    assert ck > 0 and bad == 0
    # a single-sweep result is not a 3-sweep result: the check must see it
    one = A.copy()
    oracle.stencil7(A, one, 1, nz - 1, 1 / 6, 1 / 36)
    assert bench.lightcone_verify(one, p0, T, 1 / 6, 1 / 36, oracle, synth, blocks=8, w=16)[1] > 0


def test_slab_T_sweep_pass_with_T_halo_planes_matches_the_global_pass():
    """bench.py's configs[3] T-sweep pass: a rank that holds its slab [lo, hi) plus T halo planes per
    interior side and sweeps the whole buffer T times (buffer ends held fixed) gets exactly the global
    pass's values on [lo, hi); with T - 1 halo planes the edge plane is wrong. lightcone_verify with
    kvalid / real faces accepts the slab."""
    nzg, ny, nx, T = 40, 24, 28, 3
    G = np.empty((nzg, ny, nx), np.float64)
    synth.fill(G, "random", seed=synth.SEED_A, g0=0, nx=nx, ny=ny)
    truth = G.copy()
    oracle.stencil7_sweeps(G, truth, 1, nzg - 1, 1 / 6, 1 / 36, T)
    for lo, hi in ((1, 20), (20, 39)):
        for H in (T, T - 1):
            pb0, pb1 = max(0, lo - H), min(nzg, hi + H)
            buf = G[pb0:pb1].copy()
            out = buf.copy()
            oracle.stencil7_sweeps(buf, out, 1, pb1 - pb0 - 1, 1 / 6, 1 / 36, T)
            same = np.array_equal(out[lo - pb0:hi - pb0], truth[lo:hi])
            assert same == (H == T or (pb0 == 0 and pb1 == nzg)), (lo, H)
            if H == T:
                ck, bad = bench.lightcone_verify(out, pb0, T, 1 / 6, 1 / 36, oracle, synth, blocks=8, w=12,
                                                 kvalid=(lo - pb0, hi - pb0), real_lo=pb0 == 0,
                                                 real_hi=pb1 == nzg)
                assert ck > 0 and bad == 0
