"""ctypes declarations for libppipe.so (include/ppipe.h). Argument marshalling only.

The library is built in-tree (``make ppipe`` or ``__graft_entry__.build()``). There is no fallback:
if ``libppipe.so`` is missing or fails to load, importing the package raises.
"""
import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# PP_LIBPPIPE: another in-tree build of the same library (A/B experiments of tools/); default the package's own
LIB_PATH = os.environ.get("PP_LIBPPIPE") or os.path.join(_HERE, "libppipe.so")

PP_MAX_ARRAYS = 8

i32, i64, u64, vp, cp, sz, dbl = (ctypes.c_int, ctypes.c_int64, ctypes.c_uint64, ctypes.c_void_p,
                                  ctypes.c_char_p, ctypes.c_size_t, ctypes.c_double)


class pp_triad_args(ctypes.Structure):
    _fields_ = [("s", dbl)]


class pp_stencil_args(ctypes.Structure):
    _fields_ = [("c0", dbl), ("c1", dbl)]


class pp_view(ctypes.Structure):
    _fields_ = [("ring", vp), ("R", i64), ("base", i64), ("plane_elems", i64), ("plane_bytes", i64),
                ("outer", i64), ("outer_stride", i64)]


class pp_chunk(ctypes.Structure):
    _fields_ = [("index", i64), ("k0", i64), ("k1", i64), ("narrays", i32),
                ("view", pp_view * PP_MAX_ARRAYS)]


class pp_info(ctypes.Structure):
    _fields_ = [("chunk_size", i64), ("num_streams", ctypes.c_int32), ("narrays", ctypes.c_int32),
                ("nchunks", i64), ("ring_planes", i64 * PP_MAX_ARRAYS),
                ("resident", ctypes.c_int32 * PP_MAX_ARRAYS), ("pinned", ctypes.c_int32 * PP_MAX_ARRAYS),
                ("ring_bytes", u64), ("naive_bytes", u64), ("h2d_bytes", u64), ("d2h_bytes", u64),
                ("n_h2d", i64), ("n_d2h", i64), ("n_kernels", i64), ("n_waits", i64),
                ("last_ms", dbl), ("naive_h2d_ms", dbl), ("naive_kernel_ms", dbl), ("naive_d2h_ms", dbl),
                ("graph_replayed", ctypes.c_int32), ("kernel_path", ctypes.c_int32), ("peer_bytes", u64),
                ("debug_violations", i64), ("merged_copies", i64)]


class pp_trace_rec(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("stream", ctypes.c_int32), ("chunk", i64), ("array", ctypes.c_int32),
                ("pad", ctypes.c_int32), ("p0", i64), ("p1", i64), ("bytes", u64), ("start_ms", dbl),
                ("end_ms", dbl)]


class pp_tune_result(ctypes.Structure):
    _fields_ = [("chunk_size", i64), ("num_streams", ctypes.c_int32), ("policy", ctypes.c_int32),
                ("predicted_ms", dbl), ("measured_ms", dbl), ("candidates", ctypes.c_int32),
                ("trials", ctypes.c_int32), ("graph", ctypes.c_int32)]


PP_CHUNK_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.POINTER(pp_chunk), vp, vp)

# (name, restype, argtypes) for every symbol include/ppipe.h declares
SIGNATURES = [
    ("pp_region_create", i32, [ctypes.POINTER(vp), i32]),
    ("pp_region_destroy", None, [vp]),
    ("pp_map", i32, [vp, i32, vp, i32, i32, ctypes.POINTER(i64), i64, i64, ctypes.POINTER(i32)]),
    ("pp_map_ex", i32, [vp, i32, vp, i32, i32, ctypes.POINTER(i64), i32, i64, i64, ctypes.POINTER(i32)]),
    ("pp_pipeline", i32, [vp, i32, i64, i32]),
    ("pp_mem_limit", i32, [vp, sz]),
    ("pp_set_option", i32, [vp, i32, i64]),
    ("pp_launch", i32, [vp, i64, i64, i32, vp, sz]),
    ("pp_launch_async", i32, [vp, i64, i64, i32, vp, sz]),
    ("pp_wait", i32, [vp]),
    ("pp_launch_fn", i32, [vp, i64, i64, PP_CHUNK_FN, vp]),
    ("pp_naive", i32, [vp, i64, i64, i32, vp, sz]),
    ("pp_naive_release", i32, [vp]),
    ("pp_use_streams", i32, [vp, ctypes.POINTER(vp), i32]),
    ("pp_use_device_buffer", i32, [vp, vp, sz]),
    ("pp_query", i32, [vp, ctypes.POINTER(pp_info)]),
    ("pp_autotune", i32, [vp, i64, i64, i32, vp, sz, i32, ctypes.POINTER(pp_tune_result)]),
    ("pp_trace", i32, [vp, ctypes.POINTER(pp_trace_rec), i64, ctypes.POINTER(i64)]),
    ("pp_plan_dump", i32, [vp, i64, i64, ctypes.c_char_p, sz, ctypes.POINTER(sz)]),
    ("pp_plan_check", i32, [vp, i64, i64, i64, u64, ctypes.POINTER(i64)]),
    ("pp_partition", i32, [i64, i64, i32, i32, ctypes.POINTER(i64), ctypes.POINTER(i64)]),
    ("pp_probe_link", i32, [i32, sz, i32, ctypes.POINTER(dbl)]),
    ("pp_strerror", cp, [i32]),
    ("pp_last_error", cp, []),
    ("pp_version", i32, []),
    ("pp_build_flags", i32, []),
    ("pp_halo_export", i32, [vp, i32, i64, vp, vp, ctypes.c_uint32]),
    ("pp_halo_import", i32, [vp, i32, i64, vp, i32, vp, ctypes.c_uint32]),
    ("pp_halo_clear", i32, [vp]),
    ("pp_view_plane", i32, [ctypes.POINTER(pp_view), i64, i64, ctypes.POINTER(vp), ctypes.POINTER(i64)]),
]

_LIB = None


def lib():
    global _LIB
    if _LIB is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: build it with `make ppipe` (or "
                              f"__graft_entry__.build()); there is no fallback path")
        L = ctypes.CDLL(LIB_PATH)
        for name, res, args in SIGNATURES:
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _LIB = L
    return _LIB
