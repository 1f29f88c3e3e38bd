"""CPU oracle — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl reference``
legs may import this package. The product package (``paper_conf_ipps_cuissf17_b200``) never imports it
and shares no code with it. See ``oracle.c`` for the definitions and their PAPER.md citations:

* ``stencil7``  — PAPER.md Fig. 2, plain unpartitioned loop, Fig. 2 evaluation order,
  edge pass-through (reading S5).
* ``stencil7_fig2`` — Fig. 2 exactly as printed: interior points only, edges untouched (reading S5b).
* ``triad``     — BASELINE.json configs[0] (not in the paper), ``c = a + (s*b)``.
* ``conv3d``    — Polybench 3DCONV body (§V.B; formula from PolyBench/GPU, reading C1).
* ``stencil7_sweeps`` — T Jacobi sweeps (composition of the single sweep; NEXT-1 multi-sweep chains).
* ``probe``     — int64 index-handler probe ``out[k] = in[k-1] + 3 in[k] + 9 in[k+1]``.
* ``stencil7_verify`` — verify-in-place: recompute and compare bits, no third array.

Every function is pinned by tests/test_oracle.py against closed forms, a library special case
(scipy.ndimage), hand-worked examples (tests/golden/) and brute-force invariants.
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liboracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make -C {os.path.dirname(_HERE)} oracle`")
        L = ctypes.CDLL(path)
        i64, vp, d, f = ctypes.c_int64, ctypes.c_void_p, ctypes.c_double, ctypes.c_float
        L.oracle_stencil7_f64.argtypes = [i64, i64, i64, vp, vp, i64, i64, d, d]
        L.oracle_stencil7_f32.argtypes = [i64, i64, i64, vp, vp, i64, i64, f, f]
        L.oracle_stencil7_i64.argtypes = [i64, i64, i64, vp, vp, i64, i64, i64, i64]
        L.oracle_stencil7_fig2_f64.argtypes = [i64, i64, i64, vp, vp, i64, i64, d, d]
        L.oracle_stencil7_fig2_f32.argtypes = [i64, i64, i64, vp, vp, i64, i64, f, f]
        L.oracle_stencil7_fig2_f64.restype = ctypes.c_int
        L.oracle_stencil7_fig2_f32.restype = ctypes.c_int
        L.oracle_conv3d_f64.argtypes = [i64, i64, i64, vp, vp, i64, i64]
        L.oracle_conv3d_f32.argtypes = [i64, i64, i64, vp, vp, i64, i64]
        L.oracle_conv3d_f64.restype = ctypes.c_int
        L.oracle_conv3d_f32.restype = ctypes.c_int
        L.oracle_stencil7_sweeps_f64.argtypes = [i64, i64, i64, vp, vp, i64, i64, d, d, i64]
        L.oracle_stencil7_sweeps_f32.argtypes = [i64, i64, i64, vp, vp, i64, i64, f, f, i64]
        L.oracle_stencil7_sweeps_i64.argtypes = [i64, i64, i64, vp, vp, i64, i64, i64, i64, i64]
        for n in ("oracle_stencil7_sweeps_f64", "oracle_stencil7_sweeps_f32", "oracle_stencil7_sweeps_i64"):
            getattr(L, n).restype = ctypes.c_int
        L.oracle_stencil7_verify_f64.argtypes = [i64, i64, i64, vp, vp, i64, i64, d, d]
        L.oracle_stencil7_verify_f32.argtypes = [i64, i64, i64, vp, vp, i64, i64, f, f]
        L.oracle_stencil7_verify_f64.restype = i64
        L.oracle_stencil7_verify_f32.restype = i64
        L.oracle_triad_f64.argtypes = [i64, vp, vp, d, vp, i64, i64]
        L.oracle_triad_f32.argtypes = [i64, vp, vp, f, vp, i64, i64]
        L.oracle_probe_i64.argtypes = [i64, i64, vp, vp, i64, i64]
        for n in ("oracle_stencil7_f64", "oracle_stencil7_f32", "oracle_stencil7_i64",
                  "oracle_triad_f64", "oracle_triad_f32", "oracle_probe_i64"):
            getattr(L, n).restype = ctypes.c_int
        L.oracle_threads.restype = ctypes.c_int
        L.oracle_set_threads.argtypes = [ctypes.c_int]
        _LIB = L
    return _LIB


def _p(x):
    if isinstance(x, np.ndarray):
        assert x.flags.c_contiguous
        return x.ctypes.data
    assert x.is_contiguous() and x.device.type == "cpu"
    return x.data_ptr()


def _dt(x):
    return str(x.dtype).replace("torch.", "")


def _check(rc, what):
    if rc != 0:
        raise ValueError(f"oracle {what}: bad range (rc={rc})")


def stencil7(A0, Anext, lo, hi, c0, c1):
    """Anext[lo:hi] = Fig. 2 stencil of A0 (3-D arrays [nz][ny][nx]); other planes untouched."""
    nz, ny, nx = A0.shape
    assert tuple(Anext.shape) == (nz, ny, nx) and _dt(A0) == _dt(Anext)
    fn = {"float64": lib().oracle_stencil7_f64, "float32": lib().oracle_stencil7_f32,
          "int64": lib().oracle_stencil7_i64}[_dt(A0)]
    _check(fn(nz, ny, nx, _p(A0), _p(Anext), lo, hi, c0, c1), "stencil7")
    return Anext


def stencil7_fig2(A0, Anext, lo, hi, c0, c1):
    """Fig. 2 exactly as printed: only interior points of planes [lo,hi) written (reading S5b)."""
    nz, ny, nx = A0.shape
    assert tuple(Anext.shape) == (nz, ny, nx) and _dt(A0) == _dt(Anext)
    fn = {"float64": lib().oracle_stencil7_fig2_f64, "float32": lib().oracle_stencil7_fig2_f32}[_dt(A0)]
    _check(fn(nz, ny, nx, _p(A0), _p(Anext), lo, hi, c0, c1), "stencil7_fig2")
    return Anext


def conv3d(A, B, lo, hi):
    """B[lo:hi] = Polybench 3DCONV body of A (reading C1); other planes untouched."""
    nz, ny, nx = A.shape
    fn = {"float64": lib().oracle_conv3d_f64, "float32": lib().oracle_conv3d_f32}[_dt(A)]
    _check(fn(nz, ny, nx, _p(A), _p(B), lo, hi), "conv3d")
    return B


def stencil7_sweeps(A0, Anext, lo, hi, c0, c1, sweeps):
    """Anext[lo:hi] = A^T after T Jacobi sweeps (planes outside [lo,hi) fixed at A0)."""
    nz, ny, nx = A0.shape
    fn = {"float64": lib().oracle_stencil7_sweeps_f64, "float32": lib().oracle_stencil7_sweeps_f32,
          "int64": lib().oracle_stencil7_sweeps_i64}[_dt(A0)]
    _check(fn(nz, ny, nx, _p(A0), _p(Anext), lo, hi, c0, c1, sweeps), "stencil7_sweeps")
    return Anext


def stencil7_verify(A0, got, klo, khi, c0, c1):
    """Number of elements of planes [klo,khi) of `got` whose bits differ from the oracle's."""
    nz, ny, nx = A0.shape
    fn = {"float64": lib().oracle_stencil7_verify_f64, "float32": lib().oracle_stencil7_verify_f32}[_dt(A0)]
    r = fn(nz, ny, nx, _p(A0), _p(got), klo, khi, c0, c1)
    if r < 0:
        raise ValueError("oracle stencil7_verify: bad range")
    return int(r)


def triad(a, b, s, c, lo=0, hi=None):
    n = a.shape[0]
    hi = n if hi is None else hi
    fn = {"float64": lib().oracle_triad_f64, "float32": lib().oracle_triad_f32}[_dt(a)]
    _check(fn(n, _p(a), _p(b), s, _p(c), lo, hi), "triad")
    return c


def probe(inp, out, lo, hi):
    nz = inp.shape[0]
    plane = int(np.prod(inp.shape[1:])) if len(inp.shape) > 1 else 1
    _check(lib().oracle_probe_i64(nz, plane, _p(inp), _p(out), lo, hi), "probe")
    return out


def threads():
    return int(lib().oracle_threads())


def set_threads(n):
    lib().oracle_set_threads(int(n))
