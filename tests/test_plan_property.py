"""Property-based tests of the planner + schedule checker (hypothesis): random array windows, loop
ranges, chunk sizes, stream counts, stream policies, ring slack and sweep counts — every generated plan
must pass pp_plan_check (race freedom, exact-once semantics, halo completeness, <= 2 segments)."""
import numpy as np
from hypothesis import given, settings
from hypothesis import strategies as st

import paper_conf_ipps_cuissf17_b200 as pp


@settings(max_examples=150, deadline=None)
@given(nz=st.integers(3, 40), off=st.integers(-3, 0), size=st.integers(1, 4), c=st.integers(1, 12),
       S=st.integers(1, 6), policy=st.integers(0, 5), extra=st.sampled_from([-1, 0, 1, 3]),
       out_off=st.integers(0, 1), data=st.data())
def test_random_single_sweep_plans_pass(nz, off, size, c, S, policy, extra, out_off, data):
    A = np.zeros((nz, 2, 2))
    O = np.zeros_like(A)
    lo_min = max(-off, -out_off, 0)
    hi_max = min(nz - (off + size - 1), nz - out_off)
    if hi_max <= lo_min:
        return
    lo = data.draw(st.integers(lo_min, hi_max - 1))
    hi = data.draw(st.integers(lo + 1, hi_max))
    r = pp.Region(-1)
    r.map("to", A, off, size)
    r.map("from", O, out_off, 1)
    r.pipeline(c, S)
    r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
    r.set_option(pp.PP_OPT_RING_EXTRA, extra)
    v, why = r.plan_check(lo, hi, orders=2, seed=nz * 31 + c)
    r.close()
    assert v == 0, why


@settings(max_examples=100, deadline=None)
@given(nz=st.integers(3, 36), T=st.integers(2, 7), c=st.integers(1, 10), S=st.integers(1, 4),
       policy=st.integers(0, 5), extra=st.sampled_from([-1, 0, 2]), data=st.data())
def test_random_chain_plans_pass(nz, T, c, S, policy, extra, data):
    A = np.zeros((nz, 2, 3))
    O = np.zeros_like(A)
    lo = data.draw(st.integers(1, nz - 2))
    hi = data.draw(st.integers(lo + 1, nz - 1))
    r = pp.Region(-1)
    r.map("to", A, -1, 3)
    r.map("from", O)
    r.pipeline(c, S)
    r.set_option(pp.PP_OPT_SWEEPS, T)
    r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
    r.set_option(pp.PP_OPT_RING_EXTRA, extra)
    v, why = r.plan_check(lo, hi, orders=2, seed=T * 101 + c)
    r.close()
    assert v == 0, why


@settings(max_examples=60, deadline=None)
@given(n=st.integers(1, 300), c=st.integers(1, 64), S=st.integers(1, 5), policy=st.integers(0, 5))
def test_random_triad_plans_pass(n, c, S, policy):
    a, b, cc = np.zeros(n, np.float32), np.zeros(n, np.float32), np.zeros(n, np.float32)
    r = pp.Region(-1)
    r.map("to", a)
    r.map("to", b)
    r.map("from", cc)
    r.pipeline(c, S)
    r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
    v, why = r.plan_check(0, n, orders=2)
    r.close()
    assert v == 0, why


@settings(max_examples=120, deadline=None)
@given(nz=st.integers(3, 40), c=st.integers(1, 12), S=st.integers(1, 6), policy=st.integers(0, 5),
       extra=st.sampled_from([-1, 0, 1, 3]), gran_planes=st.sampled_from([1, 2, 3]), T=st.sampled_from([1, 1, 3]),
       data=st.data())
def test_random_mirrored_ring_plans_pass(nz, c, S, policy, extra, gran_planes, T, data):
    """PP_OPT_MIRROR forced on a host-only region (granule = gran_planes planes): rings whose size is a
    multiple get one copy per chunk and array (copies may run past the ring end into the mirror);
    the checker must still find every plan race-free and exact, with slots taken mod R."""
    A = np.zeros((nz, 2, 2))
    O = np.zeros_like(A)
    lo = data.draw(st.integers(1, max(1, nz - 2)))
    hi = data.draw(st.integers(lo, nz - 1)) if nz > 2 else lo
    r = pp.Region(-1)
    r.map("to", A, -1, 3)
    r.map("from", O)
    r.pipeline(c, S)
    r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
    r.set_option(pp.PP_OPT_RING_EXTRA, extra)
    r.set_option(pp.PP_OPT_SWEEPS, T)
    r.set_option(pp.PP_OPT_MIRROR, gran_planes * 2 * 2 * 8)
    v, why = r.plan_check(lo, hi, orders=2, seed=nz * 7 + c)
    r.close()
    assert v == 0, why


def _h2d_ops_per_chunk(dump):
    per = {}
    for line in dump.splitlines():
        if line.startswith("H2D"):
            j = int(line.split()[1][2:])
            per[j] = per.get(j, 0) + 1
    return per


def test_mirrored_ring_never_splits_a_copy():
    A = np.zeros((40, 2, 2))
    O = np.zeros_like(A)
    r = pp.Region(-1)
    r.map("to", A, -1, 3)
    r.map("from", O)
    r.pipeline(6, 1)                        # R_in = 8 planes, 6 new planes per chunk: wraps often
    r.set_option(pp.PP_OPT_MIRROR, 0)
    split = _h2d_ops_per_chunk(r.plan_dump(1, 39))
    assert max(split.values()) == 2
    r.set_option(pp.PP_OPT_MIRROR, 32)      # granule = one plane: every ring mirrored
    one = _h2d_ops_per_chunk(r.plan_dump(1, 39))
    assert set(one.values()) == {1} and sorted(one) == sorted(split)
    assert r.plan_check(1, 39)[0] == 0
    r.set_option(pp.PP_OPT_MIRROR, 3 * 32)  # 8-plane input ring is not a multiple of 3 planes
    assert max(_h2d_ops_per_chunk(r.plan_dump(1, 39)).values()) == 2
    r.close()


def test_only_rings_whose_copies_wrap_are_mirrored():
    """A ring is mirrored only when one of its copies would cross the ring end: the stencil's input
    ring (8 planes, 6 new per chunk) wraps, its output ring (6 planes, drained 6 at a time from slot 0)
    never does; the triad's rings (S*c elements, chunks at multiples of c) never wrap either."""
    A = np.zeros((40, 2, 2))
    O = np.zeros_like(A)
    r = pp.Region(-1)
    r.map("to", A, -1, 3)
    r.map("from", O)
    r.pipeline(6, 1)
    r.set_option(pp.PP_OPT_MIRROR, 32)       # granule = one plane: every ring could be mirrored
    head = r.plan_dump(1, 39).splitlines()[0]
    assert head.endswith("R=8,6 mirror=1,0"), head
    assert r.plan_check(1, 39)[0] == 0
    r.pipeline(5, 1)                          # 5 planes drained into a 5-plane ring: slot 0 each time
    assert r.plan_dump(1, 39).splitlines()[0].endswith("mirror=1,0")
    r.set_option(pp.PP_OPT_RING_EXTRA, 1)     # 6-plane output ring, 5 planes per drain: wraps
    assert r.plan_dump(1, 39).splitlines()[0].endswith("mirror=1,1")
    assert r.plan_check(1, 39)[0] == 0
    r.close()
    a, b, c = (np.zeros(1 << 12, np.float32) for _ in range(3))
    t = pp.Region(-1)
    t.map("to", a)
    t.map("to", b)
    t.map("from", c)
    t.pipeline(1 << 10, 2)
    t.set_option(pp.PP_OPT_MIRROR, 4)
    assert t.plan_dump(0, 1 << 12).splitlines()[0].endswith("mirror=0,0,0")
    t.close()
