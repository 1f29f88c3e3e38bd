"""Host-side tests of the C ABI (no GPU): the library loads, exports every symbol include/ppipe.h
declares, validates arguments with the documented status codes, and its planner obeys the paper's
chunking/ring rules (readings S7-S13)."""
import ctypes
import re

import numpy as np
import pytest

import paper_conf_ipps_cuissf17_b200 as pp
from paper_conf_ipps_cuissf17_b200 import _ffi


def header_symbols():
    txt = open(_ffi.LIB_PATH.replace("paper_conf_ipps_cuissf17_b200/libppipe.so", "include/ppipe.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(pp_[a-z_]+)\s*\(", txt)) - {"pp_chunk_fn"})


def test_library_exports_every_declared_symbol():
    lib = ctypes.CDLL(_ffi.LIB_PATH)
    syms = header_symbols()
    assert len(syms) >= 20
    for s in syms:
        assert hasattr(lib, s), s
    # the Python binding declares exactly the header's functions
    assert sorted(n for n, _, _ in _ffi.SIGNATURES) == syms


def test_version_and_strerror():
    assert pp.pp_version() == (0, 1)
    assert pp.pp_strerror(pp.PP_EBUDGET).startswith("ring does not fit")
    assert pp.pp_strerror(99) == "unknown status"


def region(nz=40, ny=6, nx=5, dtype=np.float64):
    r = pp.Region(-1)
    A0 = np.zeros((nz, ny, nx), dtype)
    An = np.zeros_like(A0)
    r.map("to", A0, -1, 3)
    r.map("from", An)
    return r, A0, An


def parse_plan(txt):
    lines = txt.strip().splitlines()
    hdr = dict(kv.split("=") for kv in lines[0].split()[1:])
    ops = []
    for ln in lines[1:]:
        f = ln.split()
        d = dict(kv.split("=", 1) for kv in f[1:])
        p0, p1 = map(int, d["p"].split(":"))
        ops.append({"kind": f[0], "j": int(d["j"]), "a": int(d["a"]), "p0": p0, "p1": p1, "s": int(d["s"]),
                    "st": int(d["st"]), "deps": [int(x) for x in d["deps"].split(",") if x]})
    return hdr, ops


# ------------------------------------------------------------------ argument validation
def test_argument_errors():
    r = pp.Region(-1)
    A = np.zeros((10, 4, 4))
    with pytest.raises(pp.PPError) as e:
        r.map("from", A, -1, 3)                       # halo on an output (reading S12)
    assert e.value.status == pp.PP_EUNSUPPORTED
    with pytest.raises(pp.PPError) as e:
        r.map("to", A, 0, 0)
    assert e.value.status == pp.PP_EINVAL
    with pytest.raises(pp.PPError) as e:
        r.pipeline(2, 3, kind=pp.PP_ADAPTIVE)         # adaptive is future work
    assert e.value.status == pp.PP_EUNSUPPORTED
    with pytest.raises(pp.PPError) as e:
        r.pipeline(2, 0)
    assert e.value.status == pp.PP_EINVAL
    with pytest.raises(pp.PPError) as e:
        r.set_option(pp.PP_OPT_STREAM_POLICY, 7)
    assert e.value.status == pp.PP_EINVAL
    r.map("to", A, -1, 3)
    r.map("from", np.zeros_like(A))
    with pytest.raises(pp.PPError) as e:
        r.launch(1, 9, "stencil7", c0=1.0, c1=1.0)    # host-only region cannot launch
    assert e.value.status == pp.PP_ESTATE
    with pytest.raises(pp.PPError) as e:
        r.plan_dump(0, 9)                             # window k-1 = -1
    assert e.value.status == pp.PP_ERANGE
    with pytest.raises(pp.PPError) as e:
        r.plan_dump(1, 10)                            # window k+1 = 10 = nz
    assert e.value.status == pp.PP_ERANGE
    r.close()


def test_aliased_input_output_rejected():
    r = pp.Region(-1)
    A = np.zeros((10, 4, 4))
    r.map("to", A, -1, 3)
    with pytest.raises(pp.PPError) as e:
        r.map("from", A)                              # same host memory (reading S24)
    assert e.value.status == pp.PP_EINVAL
    r.map("to", A, 0, 1)                              # two read-only views may overlap
    r.close()


def test_too_many_arrays():
    r = pp.Region(-1)
    xs = [np.zeros(4) for _ in range(9)]
    for x in xs[:8]:
        r.map("to", x)
    with pytest.raises(pp.PPError):
        r.map("to", xs[8])
    r.close()


# ------------------------------------------------------------------ planner rules
def test_ring_capacity_formula_and_chunking():
    r, A0, An = region(nz=40)
    r.set_option(pp.PP_OPT_STREAM_POLICY, 0)          # the paper's chunk -> stream mapping
    for c, S in [(1, 3), (2, 3), (3, 2), (5, 4)]:
        r.pipeline(c, S)
        hdr, ops = parse_plan(r.plan_dump(1, 39))
        R = [int(x) for x in hdr["R"].split(",")]
        iters = 38
        assert R[0] == min(S * c + 2, iters + 2) and R[1] == min(S * c, iters)   # reading S10
        assert int(hdr["N"]) == -(-iters // c)                                     # ceil
        kers = [o for o in ops if o["kind"] == "KER"]
        assert [(o["p0"], o["p1"]) for o in kers] == [(1 + j * c, min(1 + (j + 1) * c, 39)) for j in range(len(kers))]
        # last chunk holds the remainder (reading S7); chunk j on stream j mod S (reading S8)
        assert all(o["st"] == o["j"] % S for o in ops)
    r.close()


def test_halo_reuse_each_input_plane_copied_once_and_slots_mod_R():
    r, A0, An = region(nz=50)
    r.pipeline(3, 2)
    hdr, ops = parse_plan(r.plan_dump(1, 49))
    R = [int(x) for x in hdr["R"].split(",")]
    loaded = []
    for o in ops:
        if o["kind"] == "H2D":
            loaded += list(range(o["p0"], o["p1"]))
            # index handler: slot = (p - base) mod R, base = lo + off = 0
            assert o["s"] == (o["p0"] - 0) % R[0]
            assert o["s"] + (o["p1"] - o["p0"]) <= R[0]
        if o["kind"] == "D2H":
            assert o["s"] == (o["p0"] - 1) % R[1]
    assert loaded == list(range(0, 50))               # every input plane once, in order (S13)
    segs = {}
    for o in ops:
        if o["kind"] != "KER":
            segs[(o["kind"], o["j"], o["a"])] = segs.get((o["kind"], o["j"], o["a"]), 0) + 1
    assert max(segs.values()) <= 2
    r.close()


def test_budget_shrinks_chunk_first_then_streams():
    r, A0, An = region(nz=100, ny=8, nx=8)            # plane = 512 B
    P = 8 * 8 * 8
    r.pipeline(8, 3)
    r.mem_limit(14 * P)                               # fits c=2,S=3 (8+6 planes), not c=3 (11+9)
    hdr, _ = parse_plan(r.plan_dump(1, 99))
    assert (hdr["c"], hdr["S"]) == ("2", "3")
    r.mem_limit(6 * P)                                # c=1: S=3 needs 5+3 > 6 -> S=2 needs 4+2 = 6
    hdr, _ = parse_plan(r.plan_dump(1, 99))
    assert (hdr["c"], hdr["S"]) == ("1", "2")
    r.mem_limit(3 * P)
    with pytest.raises(pp.PPError) as e:
        r.plan_dump(1, 99)
    assert e.value.status == pp.PP_EBUDGET
    r.close()


def test_auto_chunk_and_empty_range():
    r, A0, An = region(nz=512, ny=512, nx=64)         # plane 256 KiB
    r.pipeline(0, 3)
    hdr, _ = parse_plan(r.plan_dump(1, 511))
    c = int(hdr["c"])
    assert 1 <= c and int(hdr["N"]) >= 8 * 3 or c == 1
    hdr, ops = parse_plan(r.plan_dump(5, 5))
    assert ops == [] and hdr["N"] == "0"
    r.close()


def test_auto_chunk_targets_more_input_per_chunk_for_chains():
    """Automatic chunk size: >= 16 MiB of input per chunk for a single sweep, >= 256 MiB for a
    multi-sweep chain (each chunk also pays ceil(T/L) level kernels), both capped at >= 8*S chunks."""
    r, A0, An = region(nz=1000, ny=512, nx=256, dtype=np.float64)   # plane 1 MiB, 998 iterations
    r.pipeline(0, 3)
    hdr, _ = parse_plan(r.plan_dump(1, 999))
    assert int(hdr["c"]) == 16
    r.set_option(pp.PP_OPT_SWEEPS, 4)
    hdr, _ = parse_plan(r.plan_dump(1, 999))
    assert int(hdr["c"]) == (998 + 8 * 3 - 1) // (8 * 3)                 # 256 MiB target, capped: 42
    r.close()


def test_partition_balanced_contiguous():
    for lo, hi, G in [(1, 511, 1), (1, 4479, 8), (0, 7, 8), (3, 3, 4), (1, 2239 * 2 + 1, 2)]:
        parts = [pp.pp_partition(lo, hi, G, g) for g in range(G)]
        assert parts[0][0] == lo and parts[-1][1] == hi
        assert all(parts[g][1] == parts[g + 1][0] for g in range(G - 1))
        sizes = [b - a for a, b in parts]
        assert max(sizes) - min(sizes) <= 1 and sorted(sizes, reverse=True) == sizes
    with pytest.raises(pp.PPError):
        pp.pp_partition(0, 10, 2, 2)


# ------------------------------------------------------------------ schedule checker (brute force)
@pytest.mark.parametrize("nz", [3, 4, 5, 8, 12])
def test_every_schedule_passes_the_checker(nz):
    r, A0, An = region(nz=nz, ny=3, nx=3)
    iters = nz - 2
    for c in range(1, iters + 1):
        for S in range(1, 9):
            for extra in (0, 1, -1, 1000):
                for pol in (0, 1, 2, 3, 4, 5):
                    r.pipeline(c, S)
                    r.set_option(pp.PP_OPT_RING_EXTRA, extra)
                    r.set_option(pp.PP_OPT_STREAM_POLICY, pol)
                    v, why = r.plan_check(1, nz - 1, orders=6, seed=c * 131 + S)
                    assert v == 0, (nz, c, S, extra, pol, why)
    r.close()


@pytest.mark.parametrize("off,size", [(-1, 3), (0, 1), (-2, 5), (-3, 7), (0, 2)])
def test_other_window_shapes_pass_the_checker(off, size):
    nz = 31
    r = pp.Region(-1)
    A = np.zeros((nz, 2, 2))
    O = np.zeros_like(A)
    r.map("to", A, off, size)
    r.map("from", O)
    lo, hi = -off, nz - (off + size - 1)
    for c in (1, 2, 3, 5, 8):
        for S in (1, 2, 3, 5, 16):
            for extra in (0, 1, 2, -1):
                r.pipeline(c, S)
                r.set_option(pp.PP_OPT_RING_EXTRA, extra)
                v, why = r.plan_check(lo, hi, orders=4, seed=7)
                assert v == 0, (off, size, c, S, extra, why)
    r.close()


def test_tofrom_and_triad_plans_pass_the_checker():
    n = 97
    r = pp.Region(-1)
    a, b, c = np.zeros(n, np.float32), np.zeros(n, np.float32), np.zeros(n, np.float32)
    r.map("to", a)
    r.map("to", b)
    r.map("from", c)
    for ch in (1, 4, 13, 97):
        for S in (1, 2, 4):
            r.pipeline(ch, S)
            assert r.plan_check(0, n, orders=4)[0] == 0
    r.close()
    r = pp.Region(-1)
    x = np.zeros((40, 3))
    y = np.zeros((40, 3))
    r.map("tofrom", x, 1, 1)
    r.map("to", y, -1, 3)
    for ch in (1, 2, 5):
        for S in (1, 3):
            for extra in (0, -1):
                r.pipeline(ch, S)
                r.set_option(pp.PP_OPT_RING_EXTRA, extra)
                assert r.plan_check(1, 38, orders=4)[0] == 0
    r.close()


@pytest.mark.parametrize("fault,what", [(1, "race"), (2, "slot"), (3, "race"), (4, "race")])
def test_checker_catches_planted_faults(fault, what):
    # the checker is not vacuous: each planted planner bug is reported
    r, A0, An = region(nz=30, ny=3, nx=3)
    r.pipeline(2, 3)
    r.set_option(pp.PP_OPT_FAULT_INJECT, fault)
    v, why = r.plan_check(1, 29, orders=4)
    assert v > 0 and what in why, (fault, v, why)
    r.close()


@pytest.mark.parametrize("fault,what", [(1, "race"), (2, "slot"), (3, "race"), (4, "race")])
def test_checker_catches_planted_faults_on_mirrored_rings(fault, what):
    # the same planted bugs with every ring mirrored (granule = one plane): copies run past the
    # ring end into the second mapping, and the checker still reports each bug
    r, A0, An = region(nz=30, ny=3, nx=3)
    r.pipeline(2, 3)
    r.set_option(pp.PP_OPT_MIRROR, 3 * 3 * A0.itemsize)
    assert r.plan_check(1, 29, orders=4)[0] == 0
    r.set_option(pp.PP_OPT_FAULT_INJECT, fault)
    v, why = r.plan_check(1, 29, orders=4)
    assert v > 0 and what in why, (fault, v, why)
    r.close()


def test_fault_injection_also_breaks_semantics_check():
    # with only one stream (FIFO orders everything) a too-small ring still shows up in the
    # random-order semantic simulation, not only in the race check
    r, A0, An = region(nz=30, ny=3, nx=3)
    r.pipeline(3, 1)
    r.set_option(pp.PP_OPT_FAULT_INJECT, 2)
    v, why = r.plan_check(1, 29, orders=2)
    assert v > 0
    r.close()


# ------------------------------------------------------------------ in-place mode (reading S24)
def test_inplace_alias_rules_and_schedules_pass_checker():
    A = np.zeros((40, 3, 4))
    r = pp.Region(-1)
    r.set_option(pp.PP_OPT_INPLACE, 1)
    r.map("to", A, -1, 3)
    r.map("from", A)                                   # exact alias: allowed in in-place mode
    for c in (1, 2, 3, 7, 38):
        for S in (1, 2, 3, 5):
            for pol in (0, 1, 2, 3, 4, 5):
                for extra in (0, -1):
                    r.pipeline(c, S)
                    r.set_option(pp.PP_OPT_STREAM_POLICY, pol)
                    r.set_option(pp.PP_OPT_RING_EXTRA, extra)
                    v, why = r.plan_check(1, 39, orders=3)
                    assert v == 0, (c, S, pol, extra, why)
    r.close()
    r = pp.Region(-1)
    r.set_option(pp.PP_OPT_INPLACE, 1)
    r.map("to", A, -1, 3)
    with pytest.raises(pp.PPError):
        r.map("from", A[1:])                           # partial overlap is never allowed
    r.close()


def test_inplace_checker_flags_output_that_overtakes_its_input():
    # iteration k writes host plane k+2 in place, but plane k+2 is only copied in by a LATER chunk:
    # the checker must report the overwrite-before-read hazard (it is not vacuous for aliases)
    A = np.zeros((30, 2, 2))
    r = pp.Region(-1)
    r.set_option(pp.PP_OPT_INPLACE, 1)
    r.map("to", A, -1, 3)
    r.map("from", A, 2, 1)
    r.pipeline(1, 2)
    v, why = r.plan_check(1, 27, orders=2)
    assert v > 0 and "in-place" in why
    r.close()


def test_autotune_argument_errors():
    r, A0, An = region(nz=20)
    with pytest.raises(pp.PPError) as e:
        r.autotune(1, 19, "stencil7", c0=1.0, c1=1.0)          # host-only region
    assert e.value.status == pp.PP_ESTATE
    r.close()


# ------------------------------------------------------------------ multi-sweep chains (NEXT-1)
@pytest.mark.parametrize("T", [2, 3, 5, 9])
def test_chain_plans_pass_the_checker(T):
    nz = 17
    r, A0, An = region(nz=nz, ny=3, nx=3)
    r.set_option(pp.PP_OPT_SWEEPS, T)
    for c in (1, 2, 3, 5, 15):
        for S in (1, 2, 3):
            for pol in (0, 1, 3, 5):
                r.pipeline(c, S)
                r.set_option(pp.PP_OPT_STREAM_POLICY, pol)
                v, why = r.plan_check(1, nz - 1, orders=3, seed=c * 7 + S)
                assert v == 0, (T, c, S, pol, why)
    # and on a sub-range (boundary planes lo-1, hi are interior planes of the array)
    r.pipeline(2, 2)
    v, why = r.plan_check(4, 12, orders=3)
    assert v == 0, why
    r.close()


def test_chain_plan_shape():
    nz, T, c, S = 40, 4, 2, 2
    r, A0, An = region(nz=nz, ny=3, nx=3)
    r.set_option(pp.PP_OPT_SWEEPS, T)
    r.pipeline(c, S)
    hdr, ops = parse_plan(r.plan_dump(1, nz - 1))
    R = [int(x) for x in hdr["R"].split(",")]
    assert len(R) == T + 1                             # A0, output, T-1 level rings
    assert R[0] == S * c + T + 1 and R[1] == S * c
    assert R[2:] == [S * c + T - t + 1 for t in range(1, T)]
    h2d = [p for o in ops if o["kind"] == "H2D" for p in range(o["p0"], o["p1"])]
    assert h2d == list(range(0, nz))                   # every input plane crosses the link once
    kers = [o for o in ops if o["kind"] == "KER"]
    assert len({o["a"] for o in kers}) == T            # kernels at every level 1..T
    d2h = [p for o in ops if o["kind"] == "D2H" for p in range(o["p0"], o["p1"])]
    assert d2h == list(range(1, nz - 1))
    r.close()


@pytest.mark.parametrize("T,L", [(2, 2), (3, 2), (4, 2), (5, 2), (4, 3), (7, 3), (4, 4), (9, 4), (6, 4), (3, 4)])
def test_fused_chain_plans_pass_the_checker(T, L):
    """PP_OPT_FUSE: stages of up to L levels, each one kernel op with an L-plane halo; every schedule,
    also at the correctness-minimum ring capacity (ring extra 0), passes the race + semantics check."""
    nz = 19
    r, A0, An = region(nz=nz, ny=3, nx=3)
    r.set_option(pp.PP_OPT_SWEEPS, T)
    r.set_option(pp.PP_OPT_FUSE, L)
    for extra in (-1, 0):
        r.set_option(pp.PP_OPT_RING_EXTRA, extra)
        for c in (1, 2, 3, 5, 17):
            for S in (1, 2, 3):
                for pol in (0, 1):
                    r.pipeline(c, S)
                    r.set_option(pp.PP_OPT_STREAM_POLICY, pol)
                    v, why = r.plan_check(1, nz - 1, orders=2, seed=c * 7 + S)
                    assert v == 0, (T, L, extra, c, S, pol, why)
    r.set_option(pp.PP_OPT_RING_EXTRA, -1)
    r.pipeline(2, 2)
    v, why = r.plan_check(5, 13, orders=3)
    assert v == 0, why
    r.close()


def test_fused_chain_plan_shape():
    nz, T, L, c, S = 40, 7, 3, 2, 2
    r, A0, An = region(nz=nz, ny=3, nx=3)
    r.set_option(pp.PP_OPT_SWEEPS, T)
    r.set_option(pp.PP_OPT_FUSE, L)
    r.pipeline(c, S)
    hdr, ops = parse_plan(r.plan_dump(1, nz - 1))
    R = [int(x) for x in hdr["R"].split(",")]
    ends = [3, 6]                                      # stage ends 3, 6 (rings), 7 = output
    assert len(R) == len(ends) + 2
    assert R[0] == S * c + max(T + 1, 2 * L) and R[1] == S * c
    halos = [3, 1]                                     # next stage's halo after ends 3 and 6
    assert R[2:] == [S * c + max(T - e + 1, 2 * h) for e, h in zip(ends, halos)]
    kers = [o for o in ops if o["kind"] == "KER"]
    assert sorted({o["a"] for o in kers}) == [3, 6, 7]  # one op per stage and chunk
    h2d = [p for o in ops if o["kind"] == "H2D" for p in range(o["p0"], o["p1"])]
    assert h2d == list(range(0, nz))
    with pytest.raises(pp.PPError):
        r.set_option(pp.PP_OPT_FUSE, 5)
    r.close()


def test_chain_checker_catches_small_level_ring():
    r, A0, An = region(nz=30, ny=3, nx=3)
    r.set_option(pp.PP_OPT_SWEEPS, 4)
    r.pipeline(2, 1)
    r.set_option(pp.PP_OPT_RING_EXTRA, 0)
    assert r.plan_check(1, 29, orders=2)[0] == 0
    r.set_option(pp.PP_OPT_FAULT_INJECT, 1)            # drop cross-stream deps
    r.set_option(pp.PP_OPT_STREAM_POLICY, 0)
    r.pipeline(2, 3)
    v, why = r.plan_check(1, 29, orders=2)
    assert v > 0
    r.close()


# ------------------------------------------------------------------ 2-D block regions (NEXT-3)
def test_map_ex_split_dim_validation_and_plans():
    r = pp.Region(-1)
    A = np.zeros((37, 100))
    with pytest.raises(pp.PPError) as e:
        r.map("to", A, split_dim=2)
    assert e.value.status == pp.PP_EINVAL
    r.map("to", A, split_dim=1)
    r.map("to", np.zeros((37, 100)), split_dim=1)
    r.map("from", np.zeros((37, 100)), split_dim=1)
    for c in (1, 7, 16, 100):
        for S in (1, 3):
            r.pipeline(c, S)
            v, why = r.plan_check(0, 100, orders=2)
            assert v == 0, why
    with pytest.raises(pp.PPError) as e:
        r.plan_dump(0, 101)                                # window beyond extents[split_dim]
    assert e.value.status == pp.PP_ERANGE
    r.close()


def test_binding_enums_match_the_header():
    """Every PP_* enumerator the C header declares has the same value in the Python binding."""
    import os
    import re
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    src = open(os.path.join(root, "include", "ppipe.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    found = 0
    for body in re.findall(r"typedef enum \w+ \{(.*?)\}", src, flags=re.S):
        nxt = 0
        for item in body.split(","):
            item = item.strip()
            if not item:
                continue
            m = re.match(r"(PP_\w+)\s*(?:=\s*(-?\d+))?$", item)
            assert m, item
            name, val = m.group(1), int(m.group(2)) if m.group(2) is not None else nxt
            nxt = val + 1
            if hasattr(pp, name):
                assert getattr(pp, name) == val, (name, getattr(pp, name), val)
                found += 1
    assert found >= 20 and pp.PP_OPT_MIRROR == 11


def test_binding_struct_layouts_match_the_header(tmp_path):
    """ctypes mirrors of the header's structs have the C compiler's size and field offsets."""
    import ctypes
    import os
    import subprocess
    from paper_conf_ipps_cuissf17_b200 import _ffi
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    structs = ["pp_triad_args", "pp_stencil_args", "pp_view", "pp_chunk", "pp_info", "pp_tune_result", "pp_trace_rec"]
    lines = ['#include <stddef.h>', '#include <stdio.h>', '#include "ppipe.h"', "int main(void) {"]
    for st in structs:
        lines.append(f'printf("{st} size %zu\\n", sizeof({st}));')
        for name, _ in getattr(_ffi, st)._fields_:
            lines.append(f'printf("{st} {name} %zu\\n", offsetof({st}, {name}));')
    lines += ["return 0;", "}"]
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    subprocess.run(["gcc", "-I", os.path.join(root, "include"), "-o", str(exe), str(src)], check=True)
    out = subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout.split("\n")
    for line in filter(None, out):
        st, field, val = line.split()
        cls = getattr(_ffi, st)
        want = ctypes.sizeof(cls) if field == "size" else getattr(cls, field).offset
        assert int(val) == want, (st, field, int(val), want)


def test_view_plane_is_the_index_handler_slot_map():
    """pp_view_plane (the C index handler for custom bodies): slot (p - base) mod R, runs stop at the
    ring end, 2-D block regions step by one row's run; bad arguments are PP_EINVAL. Host-only."""
    from paper_conf_ipps_cuissf17_b200 import _ffi
    v = _ffi.pp_view()
    v.ring, v.R, v.base, v.plane_elems, v.plane_bytes, v.outer, v.outer_stride = 0x10000, 5, 7, 6, 48, 1, 0
    for p in range(-3, 30):
        addr, run = pp.pp_view_plane(v, p, 9)
        slot = (p - 7) % 5
        assert addr == 0x10000 + slot * 48 and run == min(9, 5 - slot)
    assert pp.ring_runs(type("C", (), {"view": [v]})(), 0, 7, 20) == [(7, 5), (12, 5), (17, 3)]
    v.outer, v.outer_stride = 3, 30                      # block region: 3 rows of 2 elements per plane
    addr, run = pp.pp_view_plane(v, 9, 1)
    assert addr == 0x10000 + 2 * 16 and run == 1
    with pytest.raises(pp.PPError):
        pp.pp_view_plane(v, 0, 0)


def test_round2_options_and_calls_validate_on_a_host_only_region():
    """Argument checks of the round-2 options and calls need no device: option ranges, the peer-halo
    calls on a host-only region (PP_ESTATE: they need a device), pp_halo_clear always legal."""
    r = pp.Region(-1)
    A = np.zeros((6, 4, 8))
    r.map("to", A, -1, 3)
    r.map("from", np.zeros((6, 4, 8)))
    for opt, good, bad in ((pp.PP_OPT_D2H_INTERIOR, 1, None), (pp.PP_OPT_DEBUG_TAGS, 1, None),
                           (pp.PP_OPT_BOUNCE, 8, 65), (pp.PP_OPT_SM_COPY, 1 << 20, -1),
                           (pp.PP_OPT_MERGE_COPIES, 1, None)):
        r.set_option(opt, good)
        r.set_option(opt, 0)
        if bad is not None:
            with pytest.raises(pp.PPError) as ei:
                r.set_option(opt, bad)
            assert ei.value.status == pp.PP_EINVAL
    with pytest.raises(pp.PPError) as ei:
        r.halo_export(0, 1, 0x1000, 0x2000, 1)
    assert ei.value.status == pp.PP_ESTATE
    with pytest.raises(pp.PPError) as ei:
        r.halo_import(0, 5, 0x1000, 0, 0x2000, 1)
    assert ei.value.status == pp.PP_ESTATE
    r.halo_clear()
    assert pp.pp_build_flags() & ~pp.PP_BUILD_TUNING == 0
    r.close()
