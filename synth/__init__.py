"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the oracle's tests.

Holds none of the method's arithmetic (SURVEY.md §8(d) "Inputs, exactly"): every value is a pure
function of (seed, global linear index g) via a counter-based splitmix64 hash, so slabs on different
ranks regenerate identical data. Implemented in C (``synth.c`` → ``libsynth.so``, OpenMP) because the
workloads reach 2^27+ elements; ``splitmix64_np`` is an independent numpy transcription used only to
check the C generator.
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

RANDOM, CONST, LINEAR, QUAD, CHECKER, PLANE, INDEX, CUBIC, RANDINT = range(9)
KINDS = {"random": RANDOM, "const": CONST, "linear": LINEAR, "quad": QUAD, "checker": CHECKER,
         "plane": PLANE, "index": INDEX, "cubic": CUBIC, "randint": RANDINT}

SENTINEL_F64 = 0x7FF8DEAD0000BEEF
SENTINEL_F32 = 0x7FC0BEEF
SENTINEL_I64 = 0x7FF8DEAD0000BEEF
SEED_A = 2017
SEED_B = 2018


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libsynth.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make -C {os.path.dirname(_HERE)} synth`")
        L = ctypes.CDLL(path)
        i64, u64, vp, ci = ctypes.c_int64, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_int
        for n in ("sy_fill_f64", "sy_fill_f32", "sy_fill_i64"):
            getattr(L, n).argtypes = [vp, i64, i64, ci, u64, i64, i64]
            getattr(L, n).restype = None
        L.sy_fill_pattern.argtypes = [vp, i64, ci, u64]
        L.sy_fill_pattern.restype = None
        L.sy_count_pattern.argtypes = [vp, i64, ci, u64]
        L.sy_count_pattern.restype = i64
        L.sy_set_threads.argtypes = [ci]
        L.sy_set_threads.restype = None
        L.sy_threads.restype = ci
        _LIB = L
    return _LIB


def _ptr_n_dt(x):
    """(address, element count, dtype-name) of a contiguous numpy array or CPU torch tensor."""
    if isinstance(x, np.ndarray):
        assert x.flags.c_contiguous
        return x.ctypes.data, x.size, str(x.dtype)
    # torch tensor (duck-typed so numpy users don't need torch)
    assert x.is_contiguous() and x.device.type == "cpu"
    return x.data_ptr(), x.numel(), str(x.dtype).replace("torch.", "")


def fill(x, kind="random", seed=SEED_A, g0=0, nx=1, ny=1):
    """Fill x (flat view) with field `kind` for global indices [g0, g0+x.size)."""
    p, n, dt = _ptr_n_dt(x)
    k = KINDS[kind] if isinstance(kind, str) else kind
    f = {"float64": lib().sy_fill_f64, "float32": lib().sy_fill_f32, "int64": lib().sy_fill_i64}[dt]
    f(p, g0, n, k, seed, nx, ny)
    return x


def sentinel(dt):
    return {"float64": SENTINEL_F64, "float32": SENTINEL_F32, "int64": SENTINEL_I64}[dt]


def fill_sentinel(x):
    p, n, dt = _ptr_n_dt(x)
    elem = 4 if dt == "float32" else 8
    lib().sy_fill_pattern(p, n, elem, sentinel(dt))
    return x


def count_sentinel(x):
    p, n, dt = _ptr_n_dt(x)
    elem = 4 if dt == "float32" else 8
    return int(lib().sy_count_pattern(p, n, elem, sentinel(dt)))


# ---- independent numpy transcription (tests of the generator itself) ----
def splitmix64_np(seed, g):
    g = np.asarray(g, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x = np.uint64(seed) ^ (g * np.uint64(0x9E3779B97F4A7C15))
        x = x + np.uint64(0x9E3779B97F4A7C15)
        x = (x ^ (x >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        x = (x ^ (x >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return x ^ (x >> np.uint64(31))


def random_np(dtype, seed, g0, n):
    h = splitmix64_np(seed, np.arange(g0, g0 + n, dtype=np.uint64))
    if dtype == np.float64:
        return (h >> np.uint64(11)).astype(np.float64) * 2.0 ** -53
    return ((h >> np.uint64(40)).astype(np.float64) * 2.0 ** -24).astype(np.float32)


def set_threads(n):
    """OpenMP worker threads of the fills (torchrun sets OMP_NUM_THREADS=1 per rank)."""
    lib().sy_set_threads(int(n))


def threads():
    return int(lib().sy_threads())
