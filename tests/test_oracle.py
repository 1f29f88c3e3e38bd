"""Pins for the CPU oracle (oracle/), independent of the oracle's own code (ROUND-1 parity gate ③).

Each test checks the oracle against something the paper or mathematics fixes, never against a
retyped copy of its formula:
  * closed forms of the Fig. 2 stencil that hold exactly in any summation
    order (constant / linear fields -> 0, quadratic -> 6, checkerboard -> 6-12x, with c0=6, c1=1);
  * the library special case: with (c0,c1) = (6,1) the stencil is the discrete Laplacian, so on
    integer data it must equal scipy.ndimage.laplace; general dyadic coefficients must equal
    scipy.ndimage.correlate with the 7-point kernel (all exact on small integers);
  * hand-worked rounding examples W1-W4 (tests/golden/) that pin the evaluation
    order, plus the exact rational value within the IEEE error bound;
  * invariants: edge pass-through, planes outside [lo,hi) untouched, axis-permutation symmetry,
    serial == threaded bits, the probe's closed form 13k+8.
Plausible mistakes these catch: a dropped neighbour (closed forms, Laplacian), a wrong sign (quad -> 6),
a swapped stride / transposed operand (non-cubic shapes vs scipy), a wrong plane (probe, linear-in-k),
FMA contraction or another order (W2/W3/W4 bits).
"""
import os
import struct
from fractions import Fraction

import numpy as np
import pytest
import scipy.ndimage as ndi

import oracle
import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def bits(x):
    x = np.asarray(x)
    if x.dtype == np.float64:
        return struct.unpack("<Q", struct.pack("<d", float(x)))[0]
    return struct.unpack("<I", struct.pack("<f", float(x)))[0]


def field(shape, kind, dtype, seed=0):
    nz, ny, nx = shape
    a = np.empty(shape, dtype=dtype)
    synth.fill(a, kind, seed=seed, nx=nx, ny=ny)
    return a


def run(A0, lo=None, hi=None, c0=6, c1=1):
    nz = A0.shape[0]
    lo = 1 if lo is None else lo
    hi = nz - 1 if hi is None else hi
    out = np.empty_like(A0)
    synth.fill_sentinel(out)
    oracle.stencil7(A0, out, lo, hi, c0, c1)
    return out


def interior(x):
    return x[1:-1, 1:-1, 1:-1]


# ------------------------------------------------------------------ generator sanity (shared module)
def test_synth_matches_numpy_transcription():
    for dt in (np.float64, np.float32):
        a = np.empty(1000, dtype=dt)
        synth.fill(a, "random", seed=2017, g0=12345)
        ref = synth.random_np(dt, 2017, 12345, 1000)
        assert np.array_equal(a.view(np.uint8), ref.view(np.uint8))
        assert 0.0 <= a.min() and a.max() < 1.0


# ------------------------------------------------------------------ stencil closed forms
@pytest.mark.parametrize("dtype", [np.float64, np.float32, np.int64])
@pytest.mark.parametrize("shape", [(5, 6, 7), (9, 4, 11), (3, 3, 3)])
def test_stencil_closed_forms(dtype, shape):
    # constant and linear fields: Laplacian 0; quadratic i^2+j^2+k^2: 6; checkerboard: 6 - 12x
    for kind, expect in (("const", lambda a: 0), ("linear", lambda a: 0), ("quad", lambda a: 6),
                         ("checker", lambda a: 6 - 12 * a)):
        A0 = field(shape, kind, dtype, seed=7)
        out = run(A0)
        got = interior(out).astype(np.float64)
        want = np.broadcast_to(np.asarray(expect(interior(A0).astype(np.float64)), np.float64), got.shape)
        assert np.array_equal(got, want), kind


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_stencil_edges_pass_through_and_untouched_planes(dtype):
    A0 = field((8, 5, 6), "random", dtype, seed=2017)
    out = run(A0, lo=2, hi=6, c0=dtype(1) / dtype(6), c1=dtype(1) / dtype(36))
    sent = synth.sentinel(str(np.dtype(dtype)))
    u = out.view(np.uint64 if dtype == np.float64 else np.uint32)
    # planes outside [lo,hi) untouched
    assert np.all(u[:2] == sent) and np.all(u[6:] == sent)
    # edge ring of computed planes equals the input (reading S5)
    for k in range(2, 6):
        for sl in (np.s_[k, 0, :], np.s_[k, -1, :], np.s_[k, :, 0], np.s_[k, :, -1]):
            assert np.array_equal(out[sl].view(u.dtype), A0[sl].view(u.dtype))
    assert not np.any(u[2:6, 1:-1, 1:-1] == sent)


@pytest.mark.parametrize("shape", [(5, 6, 7), (7, 9, 4), (12, 5, 13)])
def test_stencil_equals_scipy_laplace(shape):
    # (c0,c1) = (6,1): out = sum(6 face neighbours) - 6*ctr = discrete Laplacian (exact on integers)
    A0 = field(shape, "randint", np.float64, seed=99)
    out = run(A0, c0=6.0, c1=1.0)
    lap = ndi.laplace(A0, mode="constant")
    assert np.array_equal(interior(out), interior(lap))


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_stencil_equals_scipy_correlate_dyadic(dtype):
    # general dyadic coefficients are exact on small integers, so any correct order must agree
    c0, c1 = 0.5, 0.125
    A0 = field((6, 7, 9), "randint", dtype, seed=5)
    out = run(A0, c0=c0, c1=c1)
    w = np.zeros((3, 3, 3))
    for d in ((0, 1, 1), (2, 1, 1), (1, 0, 1), (1, 2, 1), (1, 1, 0), (1, 1, 2)):
        w[d] = c1
    w[1, 1, 1] = -c0
    ref = ndi.correlate(A0.astype(np.float64), w, mode="constant")
    assert np.array_equal(interior(out).astype(np.float64), interior(ref))


def test_stencil_axis_permutation_symmetry():
    # On fully-interior points the 7-point stencil commutes with swapping the in-plane axes i,j.
    A0 = field((6, 7, 8), "randint", np.float64, seed=3)
    out = run(A0, c0=6.0, c1=1.0)
    At = np.ascontiguousarray(A0.transpose(0, 2, 1))
    outt = run(At, c0=6.0, c1=1.0)
    assert np.array_equal(interior(out), interior(outt.transpose(0, 2, 1)))


def test_stencil_int64_wraps_like_twos_complement():
    A0 = field((5, 5, 5), "random", np.int64, seed=11)      # full-range int64: sums overflow
    out = run(A0, c0=3, c1=5)
    U = A0.view(np.uint64)
    k, j, i = 2, 2, 2
    with np.errstate(over="ignore"):
        s = (U[k + 1, j, i] + U[k - 1, j, i] + U[k, j + 1, i] + U[k, j - 1, i] + U[k, j, i + 1] + U[k, j, i - 1])
        want = (s * np.uint64(5) - U[k, j, i] * np.uint64(3))
    assert out.view(np.uint64)[k, j, i] == want


# ------------------------------------------------------------------ worked rounding examples (golden)
def _golden(name):
    rows = []
    for line in open(os.path.join(GOLDEN, name)):
        if line.strip() and not line.startswith("#"):
            rows.append(line.split())
    return rows


def _grid_for(expr):
    kk, jj, ii = np.meshgrid(np.arange(3), np.arange(3), np.arange(3), indexing="ij")
    return {"i+3j+9k": ii + 3 * jj + 9 * kk,
            "i^2+j^2+k^2": ii ** 2 + jj ** 2 + kk ** 2,
            "1+i+2j^2+3k^3": 1 + ii + 2 * jj ** 2 + 3 * kk ** 3}[expr]


@pytest.mark.parametrize("row", _golden("stencil7_worked_examples.txt"), ids=lambda r: r[0])
def test_stencil_worked_examples(row):
    name, expr = row[0], row[1]
    nb = [int(v) for v in row[2:8]]
    ctr = int(row[8])
    want64, want32 = int(row[9], 16), int(row[10], 16)
    g = _grid_for(expr)
    # the fixture's neighbour listing must describe the field (guards the fixture itself)
    assert [g[2, 1, 1], g[0, 1, 1], g[1, 2, 1], g[1, 0, 1], g[1, 1, 2], g[1, 1, 0]] == nb and g[1, 1, 1] == ctr
    for dt, want in ((np.float64, want64), (np.float32, want32)):
        c0 = dt(1) / dt(6)
        c1 = c0 / dt(6)
        out = run(g.astype(dt), c0=c0, c1=c1)
        r = out[1, 1, 1]
        assert bits(r) == want, (name, dt, hex(bits(r)))
        # and it lies within the IEEE error bound of the exact real value of the expression
        exact = Fraction(sum(nb)) * Fraction(float(c1)) - Fraction(ctr) * Fraction(float(c0))
        eps = Fraction(1, 2 ** (53 if dt == np.float64 else 24))
        scale = Fraction(sum(abs(v) for v in nb)) * Fraction(float(c1)) + Fraction(ctr) * Fraction(float(c0))
        assert abs(Fraction(float(r)) - exact) <= 8 * eps * scale


# ------------------------------------------------------------------ Fig. 2 as printed (reading S5b)
def test_fig2_literal_writes_interior_only():
    """stencil7_fig2 (Fig. 2's own loops i, j in [1, n-1)): the quadratic field gives 6 and a linear
    field 0 at every written point (closed forms with (c0,c1) = (6,1)); the edge ring of computed
    planes and every plane outside [lo,hi) keep the caller's values; the worked examples W1-W3 give
    the golden bits; and on integer data it is scipy's Laplacian on the interior."""
    nz, ny, nx = 9, 10, 11
    for dt in (np.float64, np.float32):
        for kind, want in (("quad", 6.0), ("linear", 0.0)):
            A = field((nz, ny, nx), kind, dt)
            out = np.empty_like(A)
            synth.fill_sentinel(out)
            oracle.stencil7_fig2(A, out, 2, 7, dt(6), dt(1))
            assert np.all(out[2:7, 1:-1, 1:-1] == want)
            assert synth.count_sentinel(out) == out.size - 5 * (ny - 2) * (nx - 2)
            assert synth.count_sentinel(np.ascontiguousarray(out[2:7, 1:-1, 1:-1])) == 0
    A = field((nz, ny, nx), "randint", np.float64, seed=4)
    out = np.zeros_like(A)
    oracle.stencil7_fig2(A, out, 1, nz - 1, 6.0, 1.0)
    assert np.array_equal(out[1:-1, 1:-1, 1:-1], ndi.laplace(A)[1:-1, 1:-1, 1:-1])
    for row in _golden("stencil7_worked_examples.txt"):
        g = _grid_for(row[1])
        for dt, want in ((np.float64, int(row[9], 16)), (np.float32, int(row[10], 16))):
            c0 = dt(1) / dt(6)
            o = np.zeros((3, 3, 3), dt)
            oracle.stencil7_fig2(g.astype(dt), o, 1, 2, c0, c0 / dt(6))
            assert bits(o[1, 1, 1]) == want, (row[0], dt)


@pytest.mark.parametrize("row", _golden("triad_worked_examples.txt"), ids=lambda r: r[0])
def test_triad_worked_examples(row):
    a, b, s = float(row[1]), float(row[2]), float(row[3])
    for dt, want in ((np.float64, int(row[4], 16)), (np.float32, int(row[5], 16))):
        A = np.full(4, a, dt)
        B = np.full(4, b, dt)
        C = np.zeros(4, dt)
        oracle.triad(A, B, dt(s), C)
        assert all(bits(x) == want for x in C), (dt, hex(bits(C[0])))


# ------------------------------------------------------------------ triad closed form / range
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_triad_closed_form(dtype):
    n = 1 << 20
    a = np.arange(n, dtype=dtype)
    b = (2 * np.arange(n)).astype(dtype)
    c = np.empty(n, dtype)
    synth.fill_sentinel(c)
    oracle.triad(a, b, dtype(3), c, 100, n - 7)
    assert np.array_equal(c[100:n - 7], (7 * np.arange(100, n - 7)).astype(dtype))   # 7*2^20 < 2^24
    assert synth.count_sentinel(c) == 100 + 7


# ------------------------------------------------------------------ probe closed form
def test_probe_plane_index_closed_form():
    nz, ny, nx = 20, 3, 5
    A = field((nz, ny, nx), "plane", np.int64)
    out = np.zeros_like(A)
    oracle.probe(A, out, 1, nz - 1)
    for k in range(1, nz - 1):
        assert np.all(out[k] == 13 * k + 8)
    assert np.all(out[0] == 0) and np.all(out[nz - 1] == 0)


def test_probe_brute_force_random():
    A = field((9, 2, 3), "random", np.int64, seed=4)
    out = np.zeros_like(A)
    oracle.probe(A, out, 1, 8)
    U = A.view(np.uint64).reshape(9, -1)
    for k in range(1, 8):
        for e in range(6):
            with np.errstate(over="ignore"):
                want = U[k - 1, e] + np.uint64(3) * U[k, e] + np.uint64(9) * U[k + 1, e]
            assert out.view(np.uint64).reshape(9, -1)[k, e] == want


# ------------------------------------------------------------------ verify-in-place, threads, ranges
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_verify_in_place(dtype):
    A0 = field((10, 9, 8), "random", dtype, seed=2017)
    c0 = dtype(1) / dtype(6)
    c1 = c0 / dtype(6)
    out = run(A0, c0=c0, c1=c1)
    assert oracle.stencil7_verify(A0, out, 1, 9, c0, c1) == 0
    u = out.view(np.uint64 if dtype == np.float64 else np.uint32)
    u[4, 3, 2] ^= 1
    u[5, 0, 0] ^= 1 << 3            # an edge point
    assert oracle.stencil7_verify(A0, out, 1, 9, c0, c1) == 2
    assert oracle.stencil7_verify(A0, out, 6, 9, c0, c1) == 0


def test_threads_bit_identical():
    A0 = field((33, 17, 19), "random", np.float64, seed=2017)
    n = oracle.threads()
    try:
        oracle.set_threads(1)
        a = run(A0, c0=1 / 6, c1=1 / 36)
        oracle.set_threads(max(2, n))
        b = run(A0, c0=1 / 6, c1=1 / 36)
    finally:
        oracle.set_threads(n)
    assert np.array_equal(a.view(np.uint64), b.view(np.uint64))


def test_ranges():
    A0 = field((6, 4, 4), "const", np.float64, seed=1)
    out = np.zeros_like(A0)
    with pytest.raises(ValueError):
        oracle.stencil7(A0, out, 0, 3, 6.0, 1.0)        # window k-1 = -1
    with pytest.raises(ValueError):
        oracle.stencil7(A0, out, 1, 6, 6.0, 1.0)        # window k+1 = 6 = nz
    oracle.stencil7(A0, out, 3, 3, 6.0, 1.0)            # empty range is legal
    assert np.all(out == 0)


# ------------------------------------------------------------------ T sweeps (NEXT-1 multi-sweep chains)
def run_sweeps(A0, T, lo=None, hi=None, c0=6, c1=1):
    nz = A0.shape[0]
    lo = 1 if lo is None else lo
    hi = nz - 1 if hi is None else hi
    out = np.empty_like(A0)
    synth.fill_sentinel(out)
    oracle.stencil7_sweeps(A0, out, lo, hi, c0, c1, T)
    return out


@pytest.mark.parametrize("dtype", [np.float64, np.float32, np.int64])
def test_sweeps_T1_equals_single_sweep(dtype):
    A0 = field((9, 7, 8), "random" if dtype != np.int64 else "randint", dtype, seed=2)
    c0, c1 = (dtype(1) / dtype(6), dtype(1) / dtype(36)) if dtype != np.int64 else (3, 5)
    a = run(A0, c0=c0, c1=c1)
    b = run_sweeps(A0, 1, c0=c0, c1=c1)
    assert np.array_equal(a.view(np.uint8), b.view(np.uint8))


@pytest.mark.parametrize("T", [1, 2, 3, 7])
def test_sweeps_doubling_closed_form(T):
    # (c0, c1) = (-2, 0): every interior point doubles each sweep, edges and outside planes stay A0
    A0 = field((10, 6, 7), "randint", np.float64, seed=8)
    out = run_sweeps(A0, T, lo=2, hi=8, c0=-2.0, c1=0.0)
    assert np.array_equal(out[2:8, 1:-1, 1:-1], (2.0 ** T) * A0[2:8, 1:-1, 1:-1])
    assert np.array_equal(out[2:8, 0, :], A0[2:8, 0, :]) and np.array_equal(out[2:8, :, -1], A0[2:8, :, -1])


@pytest.mark.parametrize("T", [1, 2, 3, 4])
def test_sweeps_checkerboard_far_field_closed_form(T):
    # L(x) = 6 - 12x for the checkerboard x, L(const) = 0  =>  L^T(x) = (-12)^(T-1) (6 - 12x) at every
    # point whose distance to all fixed boundaries (x/y edges, planes lo-1 and hi) is >= T
    nz, ny, nx = 14, 13, 12
    A0 = field((nz, ny, nx), "checker", np.float64)
    out = run_sweeps(A0, T)
    k0, k1 = (1 - 1) + T, (nz - 1) - T
    sl = np.s_[k0:k1 + 1, T:ny - T, T:nx - T]
    x = A0[sl]
    assert x.size > 0
    assert np.array_equal(out[sl], (-12.0) ** (T - 1) * (6.0 - 12.0 * x))


# ------------------------------------------------------------------ 3-D convolution (NEXT-2, reading C1)
def test_conv3d_closed_forms():
    # pins from tests/golden/conv3d_closed_forms.txt: constant -> 34a, i -> 34i, j -> 34j - 30, k -> 34k + 44
    nz, ny, nx = 7, 8, 9
    kk, jj, ii = np.meshgrid(np.arange(nz), np.arange(ny), np.arange(nx), indexing="ij")
    cases = [(np.full((nz, ny, nx), 3.0), lambda: np.full((nz, ny, nx), 102.0)),
             (ii.astype(np.float64), lambda: 34.0 * ii),
             (jj.astype(np.float64), lambda: 34.0 * jj - 30.0),
             (kk.astype(np.float64), lambda: 34.0 * kk + 44.0)]
    for A, want in cases:
        for dt in (np.float64, np.float32):
            Ad = np.ascontiguousarray(A.astype(dt))
            B = np.zeros_like(Ad)
            oracle.conv3d(Ad, B, 1, nz - 1)
            assert np.array_equal(interior(B).astype(np.float64), interior(want())), dt
            assert np.array_equal(B[1:nz - 1, 0, :], Ad[1:nz - 1, 0, :])       # edges pass through


def conv3d_worked_examples():
    """Examples of tests/golden/conv3d_worked_examples.txt: {(dtype, seed): (3x3x3 inputs, result bits,
    {wrong reading: its bits})} (derived in exact rationals by tests/golden/derive_conv3d_worked.py)."""
    ex = {}
    for line in open(os.path.join(GOLDEN, "conv3d_worked_examples.txt")):
        f = line.split()
        if not f or f[0].startswith("#"):
            continue
        if f[0] in ("input", "result", "alt"):
            dt = np.float64 if f[1] == "f64" else np.float32
            key = (f[1], int(f[2]))
            e = ex.setdefault(key, [np.zeros((3, 3, 3), dt), None, {}])
            if f[0] == "input":
                dk, dj, di = int(f[3]), int(f[4]), int(f[5])
                u = np.array([int(f[6], 16)], np.uint64 if dt == np.float64 else np.uint32)
                e[0][dk + 1, dj + 1, di + 1] = u.view(dt)[0]
            elif f[0] == "result":
                e[1] = int(f[3], 16)
            else:
                e[2][f[3]] = int(f[4], 16)
    return ex


def test_conv3d_worked_rounding_examples():
    """The oracle reproduces, bit for bit, the exact-rational hand derivation of reading C1 (Polybench's
    left-to-right order, every product and sum rounded, no FMA) on non-integer operands; every wrong
    reading the derivation tried (other orders, FMA contraction, merged coefficients, grouping,
    transposed operands) gives different bits in at least one example, so none of them passes."""
    ex = conv3d_worked_examples()
    assert {k[0] for k in ex} == {"f64", "f32"}
    for (fmt, seed), (A, want, alts) in ex.items():
        B = np.zeros_like(A)
        oracle.conv3d(A, B, 1, 2)
        assert bits(B[1, 1, 1]) == want, (fmt, seed, hex(bits(B[1, 1, 1])))
        assert all(v != want for v in alts.values())
    for fmt in ("f64", "f32"):
        caught = set().union(*(alts for (f, _), (_, _, alts) in ex.items() if f == fmt))
        assert {"reversed_order", "fma_contracted", "merged_coefficients", "per_plane_groups", "pairwise_tree",
                "dk_di_transposed"} | {f"swap_terms_{i}_{i + 1}" for i in range(1, 14)} <= caught, fmt


def test_conv3d_is_a_fixed_linear_27_point_correlation():
    # invariants that hold for ANY fixed 3x3x3 correlation: linearity and translation invariance
    A = field((8, 9, 10), "randint", np.float64, seed=12)
    Bm = field((8, 9, 10), "randint", np.float64, seed=13)
    oa, ob, oab = np.zeros_like(A), np.zeros_like(A), np.zeros_like(A)
    oracle.conv3d(A, oa, 1, 7)
    oracle.conv3d(Bm, ob, 1, 7)
    oracle.conv3d(np.ascontiguousarray(2 * A - 3 * Bm), oab, 1, 7)
    assert np.array_equal(interior(oab), interior(2 * oa - 3 * ob))
    sh = np.ascontiguousarray(np.roll(A, 1, axis=2))
    osh = np.zeros_like(A)
    oracle.conv3d(sh, osh, 1, 7)
    assert np.array_equal(osh[1:7, 1:-1, 2:-1], oa[1:7, 1:-1, 1:-2])
