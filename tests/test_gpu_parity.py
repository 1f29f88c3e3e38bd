"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, element by element.

Bar (BASELINE.json north_star): bit-exact for integer/index work and for floating point
in the default (no-FMA, Fig. 2 order) build; with PP_OPT_FMAD within 1e-12 (fp64) / 1e-5 (fp32)
of the per-element term scale (reading S17). Inputs are seeded synthetic fields (synth/).
"""
import itertools
import sys

import numpy as np
import pytest
import torch

import oracle
import paper_conf_ipps_cuissf17_b200 as pp
import synth

pytestmark = pytest.mark.gpu

C0_64 = 1.0 / 6.0
C1_64 = C0_64 / 6.0
C0_32 = np.float32(1) / np.float32(6)
C1_32 = C0_32 / np.float32(6)


def coeffs(dt):
    if dt == torch.float32:
        return float(C0_32), float(C1_32)
    if dt == torch.int64:
        return 3.0, 5.0
    return C0_64, C1_64


def host(shape, dtype, kind="random", seed=synth.SEED_A, pinned=True, sentinel=False):
    t = torch.empty(shape, dtype=dtype, pin_memory=pinned)
    if sentinel:
        synth.fill_sentinel(t)
    else:
        nx = shape[-1] if len(shape) > 1 else 1
        ny = shape[-2] if len(shape) > 2 else 1
        synth.fill(t, kind, seed=seed, nx=nx, ny=ny)
    return t


def as_bits(x):
    a = x.numpy() if isinstance(x, torch.Tensor) else x
    return a.view(np.uint32 if a.dtype == np.float32 else np.uint64)


def oracle_stencil(A0, lo, hi, c0, c1):
    ref = np.empty(tuple(A0.shape), dtype=A0.numpy().dtype)
    synth.fill_sentinel(ref)
    if A0.dtype == torch.int64:
        oracle.stencil7(A0.numpy(), ref, lo, hi, int(c0), int(c1))
    else:
        oracle.stencil7(A0.numpy(), ref, lo, hi, c0, c1)
    return ref


def run_stencil(A0, lo, hi, c, S, extra=-1, policy=0, graph=0, path=0, fmad=0, budget=0, out=None):
    An = out if out is not None else host(tuple(A0.shape), A0.dtype, sentinel=True)
    c0, c1 = coeffs(A0.dtype)
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(c, S)
        if budget:
            r.mem_limit(budget)
        r.set_option(pp.PP_OPT_RING_EXTRA, extra)
        r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
        r.set_option(pp.PP_OPT_GRAPH, graph)
        r.set_option(pp.PP_OPT_KERNEL_PATH, path)
        r.set_option(pp.PP_OPT_FMAD, fmad)
        r.launch(lo, hi, "stencil7", c0=c0, c1=c1)
        info = r.query()
    return An, info


# ------------------------------------------------------------------ brute force, tiny grids
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32, torch.int64])
@pytest.mark.parametrize("shape", [(3, 3, 3), (5, 4, 3), (9, 5, 8), (13, 33, 4), (12, 8, 36)])
def test_stencil_every_schedule_bit_exact(dtype, shape):
    nz = shape[0]
    A0 = host(shape, dtype)
    lo, hi = 1, nz - 1
    ref = oracle_stencil(A0, lo, hi, *coeffs(dtype))
    iters = hi - lo
    cs = sorted(set(range(1, iters + 1)))
    for c, S, extra, policy in itertools.product(cs, (1, 2, 3, 8), (0, 1, -1, 1000), (0, 1, 2, 3, 4, 5)):
        if policy != 0 and S not in (1, 3):
            continue
        An, info = run_stencil(A0, lo, hi, c, S, extra=extra, policy=policy)
        assert np.array_equal(as_bits(An), as_bits(ref)), (shape, c, S, extra, policy)
        assert info["nchunks"] == (iters + info["chunk_size"] - 1) // info["chunk_size"]


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_stencil_subrange_and_sentinels(dtype):
    A0 = host((20, 17, 24), dtype)
    An, _ = run_stencil(A0, 5, 14, 3, 2)
    ref = oracle_stencil(A0, 5, 14, *coeffs(dtype))
    assert np.array_equal(as_bits(An), as_bits(ref))
    assert synth.count_sentinel(An[:5]) == 5 * 17 * 24 and synth.count_sentinel(An[14:]) == 6 * 17 * 24


def test_stencil_empty_launch_is_noop():
    A0 = host((6, 5, 5), torch.float64)
    An, info = run_stencil(A0, 3, 3, 1, 1)
    assert synth.count_sentinel(An) == An.numel()


# ------------------------------------------------------------------ TMA-staged path, forced
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
@pytest.mark.parametrize("shape", [(5, 3, 4), (9, 17, 8), (21, 40, 264), (7, 35, 132), (40, 64, 64)])
@pytest.mark.parametrize("c,S,extra", [(1, 1, 0), (2, 3, -1), (3, 2, 1), (100, 1, -1)])
def test_stencil_tma_path_bit_exact(dtype, shape, c, S, extra):
    A0 = host(shape, dtype)
    lo, hi = 1, shape[0] - 1
    ref = oracle_stencil(A0, lo, hi, *coeffs(dtype))
    An, info = run_stencil(A0, lo, hi, c, S, extra=extra, path=pp.KPATH_TMA)
    assert info["kernel_path"] == pp.KPATH_TMA
    assert np.array_equal(as_bits(An), as_bits(ref)), (shape, c, S, extra)


def test_stencil_tma_forced_on_unaligned_shape_is_unsupported():
    A0 = host((6, 5, 7), torch.float64)                  # nx = 7: rows are not 16-byte multiples
    with pytest.raises(pp.PPError) as e:
        run_stencil(A0, 1, 5, 2, 2, path=pp.KPATH_TMA)
    assert e.value.status == pp.PP_EUNSUPPORTED


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_resident_tma_long_march_bit_exact(dtype):
    # one launch marching many planes per CTA (the bench's value mode), ragged tiles in x and y
    A0 = host((130, 70, 200), dtype)
    ref = oracle_stencil(A0, 1, 129, *coeffs(dtype))
    dA = A0.cuda()
    dN = torch.empty_like(dA)
    c0, c1 = coeffs(dtype)
    with pp.Region(0) as r:
        r.map("to", dA, -1, 3)
        r.map("from", dN)
        r.pipeline(0, 1)
        r.launch(1, 129, "stencil7", c0=c0, c1=c1)
        assert r.query()["kernel_path"] == pp.KPATH_TMA
    got = dN.cpu()
    assert np.array_equal(as_bits(got)[1:129], as_bits(ref)[1:129])


# ------------------------------------------------------------------ closed-form fields on GPU
@pytest.mark.parametrize("kind,expect", [("const", 0.0), ("linear", 0.0), ("quad", 6.0)])
def test_stencil_closed_forms_gpu(kind, expect):
    A0 = host((10, 12, 16), torch.float64, kind=kind, seed=5)
    An = host((10, 12, 16), torch.float64, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(3, 2)
        r.launch(1, 9, "stencil7", c0=6.0, c1=1.0)
    assert torch.all(An[1:9, 1:-1, 1:-1] == expect)


# ------------------------------------------------------------------ paper-sized: configs[1]
def test_config2_512cubed_fp64_bit_exact():
    nz = ny = nx = 512
    A0 = host((nz, ny, nx), torch.float64)
    ref = oracle_stencil(A0, 1, nz - 1, C0_64, C1_64)
    for path in (0, 1):
        An, info = run_stencil(A0, 1, nz - 1, 2, 3, path=path)
        assert info["ring_planes"] == [8, 6] and info["nchunks"] == 255
        assert info["h2d_bytes"] == 512 * 512 * 512 * 8 and info["d2h_bytes"] == 510 * 512 * 512 * 8
        assert np.array_equal(as_bits(An), as_bits(ref)), path
        del An


def test_config2_bench_launch_configuration_bit_exact():
    """bench.py's e2e leg exactly: 512^3 fp64, the 8 + 6-plane (28 MiB) budget, pp_autotune's pick
    (c = 6, one chunk in flight on the B200 box; mirrored rings), repeated launches — whole output
    bit-exact against the oracle after the tuner's trial launches and after the timed ones."""
    n = 512
    A0 = host((n, n, n), torch.float64)
    An = host((n, n, n), torch.float64, sentinel=True)
    ref = oracle_stencil(A0, 1, n - 1, C0_64, C1_64)
    plane = n * n * 8
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(2, 3)
        r.mem_limit((3 * 2 + 2 + 3 * 2) * plane)
        tune = r.autotune(1, n - 1, "stencil7", trials=8, c0=C0_64, c1=C1_64)
        assert np.array_equal(as_bits(An), as_bits(ref))          # the trials wrote the loop's results
        for _ in range(3):
            synth.fill_sentinel(An)
            r.launch(1, n - 1, "stencil7", c0=C0_64, c1=C1_64)
        q = r.query()
    assert q["ring_bytes"] <= 28 << 20 and q["chunk_size"] == tune["chunk_size"]
    assert np.array_equal(as_bits(An), as_bits(ref))


def test_config2_graph_and_per_stage_policy_identical():
    A0 = host((64, 128, 96), torch.float64)
    ref = oracle_stencil(A0, 1, 63, C0_64, C1_64)
    for graph, policy in ((1, 0), (0, 1), (1, 1)):
        An, info = run_stencil(A0, 1, 63, 2, 3, graph=graph, policy=policy)
        assert np.array_equal(as_bits(An), as_bits(ref)), (graph, policy)


def test_graph_replay_reuses_and_stays_exact():
    A0 = host((40, 64, 64), torch.float32)
    An = host((40, 64, 64), torch.float32, sentinel=True)
    c0, c1 = coeffs(torch.float32)
    ref = oracle_stencil(A0, 1, 39, c0, c1)
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(4, 3)
        r.set_option(pp.PP_OPT_GRAPH, 1)
        r.launch(1, 39, "stencil7", c0=c0, c1=c1)
        assert r.query()["graph_replayed"] == 0
        synth.fill_sentinel(An)
        r.launch(1, 39, "stencil7", c0=c0, c1=c1)
        assert r.query()["graph_replayed"] == 1
    assert np.array_equal(as_bits(An), as_bits(ref))


# ------------------------------------------------------------------ FMAD build: tolerance
@pytest.mark.parametrize("dtype,tol", [(torch.float64, 1e-12), (torch.float32, 1e-5)])
def test_stencil_fmad_within_tolerance(dtype, tol):
    A0 = host((18, 40, 36), dtype)
    An, _ = run_stencil(A0, 1, 17, 4, 3, fmad=1)
    c0, c1 = coeffs(dtype)
    ref = oracle_stencil(A0, 1, 17, c0, c1)
    a = A0.numpy().astype(np.float64)
    g = An.numpy()[1:17].astype(np.float64)
    rr = ref[1:17].astype(np.float64)
    # scale-relative (reading S17): |g - r| <= tol * (|c1| * sum|nbr| + |c0| * |ctr|)
    nb = np.zeros_like(a)
    nb[1:-1, 1:-1, 1:-1] = (np.abs(a[2:, 1:-1, 1:-1]) + np.abs(a[:-2, 1:-1, 1:-1]) + np.abs(a[1:-1, 2:, 1:-1])
                            + np.abs(a[1:-1, :-2, 1:-1]) + np.abs(a[1:-1, 1:-1, 2:]) + np.abs(a[1:-1, 1:-1, :-2]))
    scale = abs(c1) * nb[1:17] + abs(c0) * np.abs(a[1:17])
    assert np.all(np.abs(g - rr) <= tol * scale + 0.0)


# ------------------------------------------------------------------ resident (HBM) and naive
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_resident_arrays_bit_exact(dtype):
    A0 = host((33, 64, 72), dtype)
    ref = oracle_stencil(A0, 1, 32, *coeffs(dtype))
    dA = A0.cuda()
    dN = torch.empty_like(dA)
    synth.fill_sentinel(An := host(tuple(A0.shape), dtype, sentinel=True))
    dN.copy_(An)
    c0, c1 = coeffs(dtype)
    with pp.Region(0) as r:
        r.map("to", dA, -1, 3)
        r.map("from", dN)
        r.pipeline(0, 3)
        r.launch(1, 32, "stencil7", c0=c0, c1=c1)
        info = r.query()
    assert info["resident"] == [1, 1] and info["ring_bytes"] == 0 and info["h2d_bytes"] == 0
    assert np.array_equal(as_bits(dN.cpu()), as_bits(ref))


def test_naive_matches_oracle_and_pipelined():
    A0 = host((30, 48, 40), torch.float64)
    An = host((30, 48, 40), torch.float64, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.naive(1, 29, "stencil7", c0=C0_64, c1=C1_64)
        info = r.query()
    assert info["naive_bytes"] == 2 * 30 * 48 * 40 * 8
    assert np.array_equal(as_bits(An), as_bits(oracle_stencil(A0, 1, 29, C0_64, C1_64)))


@pytest.mark.parametrize("auto_pin", [1, 0])
def test_pageable_host_memory(auto_pin):
    A0 = host((16, 20, 24), torch.float64, pinned=False)
    An = host((16, 20, 24), torch.float64, pinned=False, sentinel=True)
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_AUTO_PIN, auto_pin)
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(3, 2)
        r.launch(1, 15, "stencil7", c0=C0_64, c1=C1_64)
        assert r.query()["pinned"] == [auto_pin, auto_pin]
    assert np.array_equal(as_bits(An), as_bits(oracle_stencil(A0, 1, 15, C0_64, C1_64)))


@pytest.mark.parametrize("bounce", [1, 3, 0])
@pytest.mark.parametrize("dtype,shape", [(torch.float64, (21, 33, 40)), (torch.float32, (30, 256, 512))])
def test_pageable_bounce_ring_bit_exact(bounce, dtype, shape):
    """Row a4: pageable arrays left pageable (PP_OPT_AUTO_PIN = 0) go through the pinned bounce ring
    (host memcpy workers; 1 = auto, 3 workers) or the driver's pageable path (0); every schedule is exact,
    also repeated async launches (staging slots reused across launches) and an in-place sweep."""
    A0 = host(shape, dtype, pinned=False)
    c0, c1 = coeffs(dtype)
    ref = oracle_stencil(A0, 1, shape[0] - 1, c0, c1)
    for c, S, pol in ((1, 1, 1), (3, 2, 0), (4, 3, 1), (7, 2, 3)):
        An = host(shape, dtype, pinned=False, sentinel=True)
        with pp.Region(0) as r:
            r.set_option(pp.PP_OPT_AUTO_PIN, 0)
            r.set_option(pp.PP_OPT_BOUNCE, bounce)
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.pipeline(c, S)
            r.set_option(pp.PP_OPT_STREAM_POLICY, pol)
            r.set_option(pp.PP_OPT_DEBUG_TAGS, 1)
            for _ in range(2):
                r.launch_async(1, shape[0] - 1, "stencil7", c0=c0, c1=c1)
            r.wait()
            q = r.query()
            assert q["pinned"] == [0, 0] and q["debug_violations"] == 0
        assert np.array_equal(as_bits(An), as_bits(ref)), (bounce, c, S, pol)
    B = A0.clone()
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_AUTO_PIN, 0)
        r.set_option(pp.PP_OPT_INPLACE, 1)
        r.set_option(pp.PP_OPT_BOUNCE, bounce)
        r.map("to", B, -1, 3)
        r.map("from", B)
        r.pipeline(2, 3)
        r.launch(1, shape[0] - 1, "stencil7", c0=c0, c1=c1)
    want = as_bits(ref).copy()
    want[0], want[-1] = as_bits(A0)[0], as_bits(A0)[-1]
    assert np.array_equal(as_bits(B), want)


def test_pageable_bounce_triad_and_launch_fn():
    n = 1 << 20
    a, b = host((n,), torch.float32, pinned=False), host((n,), torch.float32, seed=synth.SEED_B, pinned=False)
    cc = host((n,), torch.float32, pinned=False, sentinel=True)
    refc = np.empty(n, np.float32)
    oracle.triad(a.numpy(), b.numpy(), np.float32(3.0), refc)
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_AUTO_PIN, 0)
        r.map("to", a)
        r.map("to", b)
        r.map("from", cc)
        r.pipeline(1 << 18, 2)
        r.launch(0, n, "triad", s=3.0)
    assert np.array_equal(as_bits(cc), refc.view(np.uint32))


@pytest.mark.parametrize("policy,graph", [(1, 0), (0, 1), (3, 0)])
def test_sm_copy_path_bit_exact(policy, graph):
    """PP_OPT_SM_COPY: copies up to the threshold are SM kernels over the host-mapped pages (pinned
    and registered arrays); stencil and triad stay exact, the tag check sees the right planes."""
    A0 = host((26, 64, 96), torch.float64)
    ref = oracle_stencil(A0, 1, 25, C0_64, C1_64)
    An = host((26, 64, 96), torch.float64, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(3, 2)
        r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
        r.set_option(pp.PP_OPT_GRAPH, graph)
        r.set_option(pp.PP_OPT_SM_COPY, 1 << 20)
        r.set_option(pp.PP_OPT_DEBUG_TAGS, 0 if graph else 1)
        for _ in range(2):
            synth.fill_sentinel(An)
            r.launch(1, 25, "stencil7", c0=C0_64, c1=C1_64)
        assert r.query()["debug_violations"] in (0, -1)
    assert np.array_equal(as_bits(An), as_bits(ref))
    n = (1 << 20) + 12                                   # ragged: not a multiple of the chunk or of 16 B
    a = host((n,), torch.float32, pinned=False)          # registered in place by pp_map
    b = host((n,), torch.float32, seed=synth.SEED_B)
    cc = host((n,), torch.float32, sentinel=True)
    refc = np.empty(n, np.float32)
    oracle.triad(a.numpy(), b.numpy(), np.float32(3.0), refc)
    with pp.Region(0) as r:
        r.map("to", a)
        r.map("to", b)
        r.map("from", cc)
        r.pipeline(1 << 18, 2)
        r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
        r.set_option(pp.PP_OPT_GRAPH, graph)
        r.set_option(pp.PP_OPT_SM_COPY, 4 << 20)
        for _ in range(2):                               # the bench's configs[0] row: graph replayed
            synth.fill_sentinel(cc)
            r.launch(0, n, "triad", s=3.0)
            assert np.array_equal(as_bits(cc), refc.view(np.uint32))


def test_budget_shrinks_chunk_then_streams():
    A0 = host((40, 32, 32), torch.float64)
    plane = 32 * 32 * 8
    # budget for exactly c=2 at S=3 (R_in = 8, R_out = 6) even though c=8 was requested
    An, info = run_stencil(A0, 1, 39, 8, 3, budget=14 * plane)
    assert info["chunk_size"] == 2 and info["num_streams"] == 3
    assert np.array_equal(as_bits(An), as_bits(oracle_stencil(A0, 1, 39, C0_64, C1_64)))
    An, info = run_stencil(A0, 1, 39, 8, 3, budget=4 * plane)   # c=1,S=1: R_in=3, R_out=1
    assert info["chunk_size"] == 1 and info["num_streams"] == 1
    assert np.array_equal(as_bits(An), as_bits(oracle_stencil(A0, 1, 39, C0_64, C1_64)))
    with pytest.raises(pp.PPError) as e:
        run_stencil(A0, 1, 39, 8, 3, budget=3 * plane)
    assert e.value.status == pp.PP_EBUDGET


# ------------------------------------------------------------------ triad (configs[0])
@pytest.mark.parametrize("dtype", [torch.float32, torch.float64])
@pytest.mark.parametrize("n,c,S", [(1 << 20, 1 << 18, 2), (1000003, 4099, 3), (17, 1, 5), (64, 64, 1),
                                   (1, 1, 1), (5, 100, 2), (4099, 0, 3)])
def test_triad_bit_exact(dtype, n, c, S):
    a = host((n,), dtype, seed=synth.SEED_A)
    b = host((n,), dtype, seed=synth.SEED_B)
    ref = np.empty(n, dtype=a.numpy().dtype)
    oracle.triad(a.numpy(), b.numpy(), a.numpy().dtype.type(3.0), ref)
    for policy in (0, 1, 5):
        cc = host((n,), dtype, sentinel=True)
        with pp.Region(0) as r:
            r.map("to", a)
            r.map("to", b)
            r.map("from", cc)
            r.pipeline(c, S)
            r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
            r.launch(0, n, "triad", s=3.0)
        assert np.array_equal(as_bits(cc), as_bits(ref)), policy


@pytest.mark.parametrize("c,S,graph", [(1 << 18, 2, 0), (1 << 18, 2, 1), (70001, 3, 0), (1 << 20, 1, 0)])
def test_triad_merged_copies_bit_exact(c, S, graph):
    """PP_OPT_MERGE_COPIES: a and b as the two halves of one pinned buffer -> each chunk's two H2D copies
    go out as one 2-D copy (merged_copies = one per chunk); reversed order (negative host distance),
    per-array copy streams (policy 5) and the option off issue one copy per array; every result bit-exact."""
    n = 1 << 20
    buf = torch.empty(2 * n, dtype=torch.float32).pin_memory()
    synth.fill(buf[:n].numpy(), "random", seed=synth.SEED_A)
    synth.fill(buf[n:].numpy(), "random", seed=synth.SEED_B)
    for order, policy, merge, want in (("ab", 1, 1, True), ("ba", 1, 1, False), ("ab", 5, 1, False),
                                       ("ab", 1, 0, False)):
        first, second = (buf[:n], buf[n:]) if order == "ab" else (buf[n:], buf[:n])
        exp = np.empty(n, dtype=np.float32)
        oracle.triad(first.numpy(), second.numpy(), np.float32(3.0), exp)
        cc = host((n,), torch.float32, sentinel=True)
        with pp.Region(0) as r:
            r.map("to", first)
            r.map("to", second)
            r.map("from", cc)
            r.pipeline(c, S)
            r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
            r.set_option(pp.PP_OPT_MERGE_COPIES, merge)
            r.set_option(pp.PP_OPT_GRAPH, graph)
            r.set_option(pp.PP_OPT_MIRROR, 0)          # (a mirrored ring is its own mapping: no merge)
            for _ in range(2 if graph else 1):
                r.launch(0, n, "triad", s=3.0)
                info = r.query()
        assert np.array_equal(as_bits(cc), as_bits(exp)), (order, policy, merge)
        assert info["merged_copies"] == (info["nchunks"] if want else 0), (order, policy, merge, info["merged_copies"])
        assert info["graph_replayed"] == graph


def test_merged_copies_off_for_single_input_and_traced_launches():
    """One input array (stencil) has nothing to merge; a traced launch keeps one copy per array so each
    op gets its own interval."""
    n = 1 << 16
    buf = torch.empty(2 * n, dtype=torch.float64).pin_memory()
    synth.fill(buf.numpy(), "random", seed=synth.SEED_A)
    cc = host((n,), torch.float64, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", buf[:n])
        r.map("to", buf[n:])
        r.map("from", cc)
        r.pipeline(1 << 12, 2)
        r.set_option(pp.PP_OPT_TRACE, 1)
        r.launch(0, n, "triad", s=3.0)
        assert r.query()["merged_copies"] == 0
        assert len(r.trace()) == r.query()["n_h2d"] + r.query()["n_d2h"] + r.query()["n_kernels"]
    A0 = host((24, 16, 20), torch.float64)
    An = host((24, 16, 20), torch.float64, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(4, 2)
        r.launch(1, 23, "stencil7", c0=1 / 6, c1=1 / 36)
        assert r.query()["merged_copies"] == 0


def test_triad_closed_form_config1():
    n = 1 << 20
    a = torch.arange(n, dtype=torch.float32).pin_memory()
    b = (2 * torch.arange(n)).to(torch.float32).pin_memory()
    c = host((n,), torch.float32, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", a)
        r.map("to", b)
        r.map("from", c)
        r.pipeline(1 << 18, 2)
        r.launch(0, n, "triad", s=3.0)
        info = r.query()
    assert info["nchunks"] == 4 and info["ring_planes"] == [1 << 19] * 3
    assert torch.equal(c, (7 * torch.arange(n)).to(torch.float32))


# ------------------------------------------------------------------ probe: index handler, int64
@pytest.mark.parametrize("c,S,extra", [(1, 1, 0), (1, 3, -1), (2, 3, -1), (5, 2, 1), (7, 4, 0), (30, 1, -1)])
def test_probe_plane_index_13k_plus_8(c, S, extra):
    nz = 40
    A = host((nz, 3, 70), torch.int64, kind="plane")
    O = torch.full((nz, 3, 70), -1, dtype=torch.int64).pin_memory()
    with pp.Region(0) as r:
        r.map("to", A, -1, 3)
        r.map("from", O)
        r.pipeline(c, S)
        r.set_option(pp.PP_OPT_RING_EXTRA, extra)
        r.launch(1, nz - 1, "probe")
    k = torch.arange(1, nz - 1).view(-1, 1, 1)
    assert torch.all(O[1:nz - 1] == 13 * k + 8)
    assert torch.all(O[0] == -1) and torch.all(O[nz - 1] == -1)


def test_probe_random_int64_matches_oracle():
    A = host((25, 7, 9), torch.int64)
    O = torch.zeros((25, 7, 9), dtype=torch.int64).pin_memory()
    with pp.Region(0) as r:
        r.map("to", A, -1, 3)
        r.map("from", O)
        r.pipeline(3, 3)
        r.launch(1, 24, "probe")
    ref = np.zeros((25, 7, 9), dtype=np.int64)
    oracle.probe(A.numpy(), ref, 1, 24)
    assert np.array_equal(O.numpy(), ref)


# ------------------------------------------------------------------ errors on the GPU path
def test_errors_and_poisoning():
    A0 = host((10, 8, 8), torch.float64)
    An = host((10, 8, 8), torch.float64, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(2, 2)
        with pytest.raises(pp.PPError) as e:
            r.launch(0, 9, "stencil7", c0=1.0, c1=1.0)      # window k-1 = -1
        assert e.value.status == pp.PP_ERANGE
        with pytest.raises(pp.PPError) as e:
            r.launch(1, 9, "triad", s=1.0)                  # wrong binding
        assert e.value.status == pp.PP_EINVAL
        r.launch(1, 9, "stencil7", c0=C0_64, c1=C1_64)      # region still usable
    assert np.array_equal(as_bits(An), as_bits(oracle_stencil(A0, 1, 9, C0_64, C1_64)))


# ------------------------------------------------------------------ in-place mode (configs[2] path)
@pytest.mark.parametrize("dtype", [torch.float32, torch.float64])
@pytest.mark.parametrize("c,S,policy", [(1, 1, 0), (2, 3, 1), (3, 2, 2), (8, 3, 1)])
def test_inplace_sweep_equals_oracle_on_original(dtype, c, S, policy):
    shape = (37, 24, 40)
    A = host(shape, dtype)
    orig = A.clone()
    ref = oracle_stencil(orig, 1, shape[0] - 1, *coeffs(dtype))
    c0, c1 = coeffs(dtype)
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_INPLACE, 1)
        r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
        r.map("to", A, -1, 3)
        r.map("from", A)
        r.pipeline(c, S)
        r.mem_limit(10 * 24 * 40 * A.element_size() * (S * c + 2))
        r.launch(1, shape[0] - 1, "stencil7", c0=c0, c1=c1)
    got = as_bits(A)
    want = as_bits(ref).copy()
    want[0] = as_bits(orig)[0]
    want[-1] = as_bits(orig)[-1]
    assert np.array_equal(got, want)


# ------------------------------------------------------------------ custom loop body (pp_launch_fn)
def test_launch_fn_custom_body_with_torch_ops():
    # a user body built from torch ops on the ring views: out[k] = in[k-1] - 2 in[k] + in[k+1]
    # (1-D second difference along the split dim); must match numpy on the host arrays
    nz, P = 41, 1000
    A = host((nz, P), torch.float64)
    O = host((nz, P), torch.float64, sentinel=True)

    def body(chunk, stream):
        st = torch.cuda.ExternalStream(stream)
        with torch.cuda.stream(st):
            for k in range(chunk.k0, chunk.k1):
                win = [torch.as_tensor(pp.chunk_view(chunk, 0, q), device="cuda") for q in (k - 1, k, k + 1)]
                out = torch.as_tensor(pp.chunk_view(chunk, 1, k), device="cuda")
                out.copy_(win[0] - 2.0 * win[1] + win[2])
        return 0

    with pp.Region(0) as r:
        r.map("to", A, -1, 3)
        r.map("from", O)
        r.pipeline(3, 2)
        r.launch_fn(1, nz - 1, body)
    a = A.numpy()
    want = a[:-2] - 2.0 * a[1:-1] + a[2:]
    assert np.array_equal(O.numpy()[1:nz - 1], want)


def test_launch_fn_merged_copies_both_directions():
    """Two inputs and two outputs, each pair the halves of one pinned buffer: every chunk's two H2D
    copies and two D2H copies go out as one 2-D copy each (wrap-free rings stay unmirrored, so no
    MIRROR override is needed); u = x + y, v = x - y exact."""
    nz, P = 40, 4096
    XY = host((2 * nz, P), torch.float32)
    UV = host((2 * nz, P), torch.float32, sentinel=True)
    X, Y, U, V = XY[:nz], XY[nz:], UV[:nz], UV[nz:]

    def body(chunk, stream):
        st = torch.cuda.ExternalStream(stream)
        with torch.cuda.stream(st):
            n = chunk.k1 - chunk.k0
            x, y, u, v = (torch.as_tensor(pp.chunk_view(chunk, a, chunk.k0, n, typestr="<f4"), device="cuda")
                          for a in range(4))
            u.copy_(x + y)
            v.copy_(x - y)
        return 0

    for c, S in ((4, 2), (5, 1), (8, 3)):
        synth.fill_sentinel(UV)
        with pp.Region(0) as r:
            for t in (X, Y):
                r.map("to", t)
            for t in (U, V):
                r.map("from", t)
            r.pipeline(c, S)
            r.launch_fn(0, nz, body)
            q = r.query()
        assert q["merged_copies"] == 2 * q["nchunks"], (c, S, q["merged_copies"])
        assert torch.equal(U, X + Y) and torch.equal(V, X - Y), (c, S)


def test_launch_fn_error_aborts():
    A = host((10, 8), torch.float64)
    O = host((10, 8), torch.float64, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", A, -1, 3)
        r.map("from", O)
        r.pipeline(2, 2)
        with pytest.raises(pp.PPError) as e:
            r.launch_fn(1, 9, lambda chunk, stream: 1)
        assert e.value.status == pp.PP_EINVAL


# ------------------------------------------------------------------ borrowed device buffer / streams
def test_use_device_buffer_and_streams():
    A0 = host((30, 32, 32), torch.float64)
    An = host((30, 32, 32), torch.float64, sentinel=True)
    buf = torch.empty(64 << 20, dtype=torch.uint8, device="cuda")
    streams = [torch.cuda.Stream() for _ in range(7)]      # policy 3 with S = 3 uses 2S + 1 streams
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(2, 3)
        r.use_device_buffer(buf.data_ptr(), buf.numel())
        r.use_streams([s.cuda_stream for s in streams])
        r.launch(1, 29, "stencil7", c0=C0_64, c1=C1_64)
        assert r.query()["ring_bytes"] <= buf.numel()
    assert np.array_equal(as_bits(An), as_bits(oracle_stencil(A0, 1, 29, C0_64, C1_64)))


@pytest.mark.parametrize("dtype,tol", [(torch.float32, 1e-5), (torch.float64, 1e-12)])
def test_triad_fmad_within_tolerance(dtype, tol):
    n = 100003
    a = host((n,), dtype, seed=synth.SEED_A)
    b = host((n,), dtype, seed=synth.SEED_B)
    c = host((n,), dtype, sentinel=True)
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_FMAD, 1)
        r.map("to", a)
        r.map("to", b)
        r.map("from", c)
        r.pipeline(4096, 3)
        r.launch(0, n, "triad", s=3.0)
    ref = np.empty(n, dtype=a.numpy().dtype)
    oracle.triad(a.numpy(), b.numpy(), a.numpy().dtype.type(3.0), ref)
    scale = np.abs(a.numpy().astype(np.float64)) + 3.0 * np.abs(b.numpy().astype(np.float64))
    assert np.all(np.abs(c.numpy().astype(np.float64) - ref.astype(np.float64)) <= tol * scale)


# ------------------------------------------------------------------ autotuner (NEXT-4)
def test_autotune_picks_a_fitting_schedule_and_stays_exact():
    A0 = host((96, 128, 128), torch.float64)
    An = host((96, 128, 128), torch.float64, sentinel=True)
    plane = 128 * 128 * 8
    ref = oracle_stencil(A0, 1, 95, C0_64, C1_64)
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.mem_limit(14 * plane)                      # the configs[1]-style 14-plane budget
        res = r.autotune(1, 95, "stencil7", trials=3, c0=C0_64, c1=C1_64)
        assert res["candidates"] > 0 and res["trials"] == 3 and res["measured_ms"] > 0
        synth.fill_sentinel(An)
        r.launch(1, 95, "stencil7", c0=C0_64, c1=C1_64)
        q = r.query()
        assert q["chunk_size"] == res["chunk_size"] and q["ring_bytes"] <= 14 * plane
        assert res["graph"] in (0, 1)
        assert res["graph"] == 0 or res["policy"] == 4 or (res["policy"] == 1 and res["num_streams"] == 1)
        if res["graph"]:                             # the second launch replays the tuned graph
            synth.fill_sentinel(An)
            r.launch(1, 95, "stencil7", c0=C0_64, c1=C1_64)
            assert r.query()["graph_replayed"]
    assert np.array_equal(as_bits(An), as_bits(ref))


def test_autotune_graph_candidates_only_with_pinned_arrays():
    A0 = torch.from_numpy(np.empty((40, 64, 64)))    # pageable: graph replay is not allowed
    synth.fill(A0, "random", seed=synth.SEED_A, nx=64, ny=64)
    An = torch.from_numpy(np.empty((40, 64, 64)))
    synth.fill_sentinel(An)
    ref = oracle_stencil(A0, 1, 39, C0_64, C1_64)
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_AUTO_PIN, 0)
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.mem_limit(14 * 64 * 64 * 8)
        res = r.autotune(1, 39, "stencil7", trials=8, c0=C0_64, c1=C1_64)
        assert res["graph"] == 0
        synth.fill_sentinel(An)
        r.launch(1, 39, "stencil7", c0=C0_64, c1=C1_64)
    assert np.array_equal(as_bits(An), as_bits(ref))


def test_autotune_rejects_inplace():
    A = host((20, 16, 16), torch.float64)
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_INPLACE, 1)
        r.map("to", A, -1, 3)
        r.map("from", A)
        with pytest.raises(pp.PPError) as e:
            r.autotune(1, 19, "stencil7", c0=C0_64, c1=C1_64)
        assert e.value.status == pp.PP_EUNSUPPORTED
        res = r.autotune(1, 19, "stencil7", trials=0, c0=C0_64, c1=C1_64)   # the model's pick only
        assert res["trials"] == 0 and res["chunk_size"] >= 1
        B = A.clone()
        r.launch(1, 19, "stencil7", c0=C0_64, c1=C1_64)                     # the array was not touched
    ref = oracle_stencil(B, 1, 19, C0_64, C1_64)
    want = as_bits(ref).copy()
    want[0], want[-1] = as_bits(B)[0], as_bits(B)[-1]
    assert np.array_equal(as_bits(A), want)


# ------------------------------------------------------------------ multi-sweep chains (NEXT-1)
def oracle_sweeps(A0, lo, hi, c0, c1, T):
    ref = np.empty(tuple(A0.shape), dtype=A0.numpy().dtype)
    synth.fill_sentinel(ref)
    if A0.dtype == torch.int64:
        oracle.stencil7_sweeps(A0.numpy(), ref, lo, hi, int(c0), int(c1), T)
    else:
        oracle.stencil7_sweeps(A0.numpy(), ref, lo, hi, c0, c1, T)
    return ref


def run_sweeps(A0, lo, hi, T, c, S, policy=1, path=0, inplace=False, out=None, fuse=1, fmad=0):
    An = A0 if inplace else (out if out is not None else host(tuple(A0.shape), A0.dtype, sentinel=True))
    c0, c1 = coeffs(A0.dtype)
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_INPLACE, int(inplace))
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(c, S)
        r.set_option(pp.PP_OPT_SWEEPS, T)
        r.set_option(pp.PP_OPT_FUSE, fuse)
        r.set_option(pp.PP_OPT_FMAD, fmad)
        r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
        r.set_option(pp.PP_OPT_KERNEL_PATH, path)
        r.launch(lo, hi, "stencil7", c0=c0, c1=c1)
        info = r.query()
    return An, info


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32, torch.int64])
@pytest.mark.parametrize("T", [2, 3, 5, 8])
def test_sweeps_chain_bit_exact(dtype, T):
    shape = (29, 20, 36)
    A0 = host(shape, dtype)
    ref = oracle_sweeps(A0, 1, shape[0] - 1, *coeffs(dtype), T)
    for c, S, pol in ((1, 1, 1), (2, 3, 1), (3, 2, 0), (5, 2, 3), (27, 1, 1)):
        An, info = run_sweeps(A0, 1, shape[0] - 1, T, c, S, policy=pol)
        assert np.array_equal(as_bits(An), as_bits(ref)), (T, c, S, pol)
        assert info["n_kernels"] >= T and info["h2d_bytes"] == A0.numel() * A0.element_size()


@pytest.mark.parametrize("path", [pp.KPATH_GENERIC, pp.KPATH_TMA])
def test_sweeps_chain_subrange_both_paths(path):
    A0 = host((40, 34, 64), torch.float64)
    ref = oracle_sweeps(A0, 6, 30, C0_64, C1_64, 6)
    An, info = run_sweeps(A0, 6, 30, 6, 4, 2, path=path)
    assert info["kernel_path"] == path
    assert np.array_equal(as_bits(An), as_bits(ref))


def test_sweeps_naive_and_inplace_match():
    A0 = host((26, 24, 32), torch.float32)
    ref = oracle_sweeps(A0, 1, 25, *coeffs(torch.float32), 4)
    An = host((26, 24, 32), torch.float32, sentinel=True)
    c0, c1 = coeffs(torch.float32)
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.set_option(pp.PP_OPT_SWEEPS, 4)
        r.naive(1, 25, "stencil7", c0=c0, c1=c1)
        assert r.query()["n_kernels"] == 4
    assert np.array_equal(as_bits(An), as_bits(ref))
    B = A0.clone().pin_memory()
    run_sweeps(B, 1, 25, 4, 3, 2, inplace=True)
    want = as_bits(ref).copy()
    want[0], want[-1] = as_bits(A0)[0], as_bits(A0)[-1]
    assert np.array_equal(as_bits(B), want)


# ------------------------------------------------------------------ fused multi-level chains (PP_OPT_FUSE)
# shapes span several overlapped tiles (output tiles of 64-2L columns x 32 or 36-2L rows) with ragged tails
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
@pytest.mark.parametrize("T,L", [(2, 2), (3, 2), (5, 2), (3, 3), (8, 3), (4, 4), (9, 4), (6, 4)])
def test_fused_chain_bit_exact(dtype, T, L):
    shape = (23, 70, 132)
    A0 = host(shape, dtype)
    ref = oracle_sweeps(A0, 1, shape[0] - 1, *coeffs(dtype), T)
    for c, S, pol in ((1, 1, 1), (2, 3, 1), (3, 2, 0), (21, 1, 1)):
        An, info = run_sweeps(A0, 1, shape[0] - 1, T, c, S, policy=pol, fuse=L)
        assert np.array_equal(as_bits(An), as_bits(ref)), (T, L, c, S, pol)
        assert info["h2d_bytes"] == A0.numel() * A0.element_size()


def test_fused_chain_subrange_tiny_and_large_planes():
    # sub-range: planes lo-1 and hi are interior planes of the array, kept fixed
    A0 = host((40, 34, 64), torch.float64)
    ref = oracle_sweeps(A0, 6, 30, C0_64, C1_64, 7)
    An, _ = run_sweeps(A0, 6, 30, 7, 4, 2, fuse=3)
    assert np.array_equal(as_bits(An), as_bits(ref))
    # planes smaller than one tile, and a single-plane launch
    A1 = host((9, 5, 4), torch.float32)
    for lo, hi in ((1, 8), (4, 5)):
        ref = oracle_sweeps(A1, lo, hi, *coeffs(torch.float32), 5)
        An, _ = run_sweeps(A1, lo, hi, 5, 2, 2, fuse=4)
        assert np.array_equal(as_bits(An), as_bits(ref)), (lo, hi)
    # planes wider than one tile row in both directions, many z-segments per launch
    A2 = host((70, 130, 260), torch.float32)
    ref = oracle_sweeps(A2, 1, 69, *coeffs(torch.float32), 4)
    An, _ = run_sweeps(A2, 1, 69, 4, 68, 1, fuse=2)
    assert np.array_equal(as_bits(An), as_bits(ref))


def test_fused_fmad_matches_unfused_fmad():
    A0 = host((20, 40, 68), torch.float64)
    a, _ = run_sweeps(A0, 1, 19, 6, 3, 2, fmad=1)
    b, _ = run_sweeps(A0, 1, 19, 6, 3, 2, fmad=1, fuse=3)
    assert np.array_equal(as_bits(a), as_bits(b))


def test_fused_naive_matches_oracle():
    for dtype, L in ((torch.float32, 3), (torch.float64, 4)):
        A0 = host((26, 24, 32), dtype)
        ref = oracle_sweeps(A0, 1, 25, *coeffs(dtype), 7)
        An = host((26, 24, 32), dtype, sentinel=True)
        c0, c1 = coeffs(dtype)
        with pp.Region(0) as r:
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.set_option(pp.PP_OPT_SWEEPS, 7)
            r.set_option(pp.PP_OPT_FUSE, L)
            r.naive(1, 25, "stencil7", c0=c0, c1=c1)
            assert r.query()["n_kernels"] == (7 + L - 1) // L
        assert np.array_equal(as_bits(An), as_bits(ref)), (dtype, L)


# ------------------------------------------------------------------ FMAD chains: T-scaled tolerance
# Reading S17 per sweep: |g - r| <= tol * (|c1| sum|nbr| + |c0| |ctr|). Over T sweeps the per-sweep
# differences propagate through the linear sweep operator, whose max-norm gain is
# rho = 6|c1| + |c0| (= 1/3 with the Parboil coefficients), so with rho <= 1 and every level bounded
# by max|A0|: |g_T - r_T| <= tol * T * rho * max|A0| at every point. A dropped term,
# wrong sign or stale halo plane changes results by ~|c1| * |A| (1/36), far above the bound.
@pytest.mark.parametrize("dtype,tol", [(torch.float64, 1e-12), (torch.float32, 1e-5)])
@pytest.mark.parametrize("T,L", [(2, 1), (4, 1), (8, 1), (2, 2), (4, 2), (8, 2), (4, 4), (8, 4)])
def test_sweeps_fmad_within_T_scaled_tolerance(dtype, tol, T, L):
    shape = (23, 70, 132)
    A0 = host(shape, dtype)
    c0, c1 = coeffs(dtype)
    ref = oracle_sweeps(A0, 1, shape[0] - 1, c0, c1, T)
    rho = 6 * abs(c1) + abs(c0)
    assert rho <= 1
    bound = tol * T * rho * float(np.abs(A0.numpy()).max())
    for c, S, pol in ((3, 2, 1), (1, 1, 0)):
        An, info = run_sweeps(A0, 1, shape[0] - 1, T, c, S, policy=pol, fuse=L, fmad=1)
        g = An.numpy()[1:-1].astype(np.float64)          # planes 0 and nz-1 keep the sentinel
        r = ref[1:-1].astype(np.float64)
        assert np.abs(g - r).max() <= bound, (T, L, c, S, np.abs(g - r).max(), bound)
        # untouched planes and each plane's edge ring (copies) are exact
        gb, rb = as_bits(An), as_bits(ref)
        assert np.array_equal(gb[0], rb[0]) and np.array_equal(gb[-1], rb[-1])
        assert np.array_equal(gb[:, 0, :], rb[:, 0, :]) and np.array_equal(gb[:, :, -1], rb[:, :, -1])
        # the option took effect: contraction changes the last bit somewhere (~half the points)
        assert not np.array_equal(gb, rb)


def test_fused_unsupported_shapes_rejected():
    for dtype, shape in ((torch.int64, (8, 6, 8)), (torch.float64, (8, 6, 7)), (torch.float32, (8, 6, 6))):
        A0 = host(shape, dtype)
        An = host(shape, dtype, sentinel=True)
        with pp.Region(0) as r:
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.set_option(pp.PP_OPT_SWEEPS, 3)
            r.set_option(pp.PP_OPT_FUSE, 2)
            with pytest.raises(pp.PPError) as ei:
                r.launch(1, shape[0] - 1, "stencil7", c0=3.0, c1=5.0)
            assert ei.value.status == pp.PP_EUNSUPPORTED


@pytest.mark.skipif(not (pp.pp_build_flags() & pp.PP_BUILD_TUNING),
                    reason="alternative tilings are compiled only in a tuning build (make TUNING=1)")
@pytest.mark.parametrize("variant", ["1", "2"])
def test_fused_tiling_variants_bit_exact(variant):
    """The alternative tilings (PP_FUSE_VARIANT, read once per process) give the same bits."""
    import os
    import subprocess
    code = (
        "import sys; sys.path.insert(0, %r); sys.path.insert(0, %r)\n"
        "import numpy as np, torch, test_gpu_parity as t\n"
        "for dt in (torch.float64, torch.float32):\n"
        "    for T, L in ((4, 2), (7, 3), (8, 4)):\n"
        "        A0 = t.host((21, 70, 132), dt)\n"
        "        ref = t.oracle_sweeps(A0, 1, 20, *t.coeffs(dt), T)\n"
        "        An, _ = t.run_sweeps(A0, 1, 20, T, 3, 2, fuse=L)\n"
        "        assert np.array_equal(t.as_bits(An), t.as_bits(ref)), (dt, T, L)\n"
        "print('ok')\n") % (os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                              os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, PP_FUSE_VARIANT=variant)
    res = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=600)
    assert res.returncode == 0 and res.stdout.strip().endswith("ok"), res.stderr[-3000:]


# ------------------------------------------------------------------ 3-D convolution (NEXT-2)
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
@pytest.mark.parametrize("shape", [(5, 4, 3), (17, 33, 40), (40, 64, 64)])
def test_conv3d_bit_exact_every_schedule(dtype, shape):
    A = host(shape, dtype)
    ref = np.empty(shape, dtype=A.numpy().dtype)
    synth.fill_sentinel(ref)
    oracle.conv3d(A.numpy(), ref, 1, shape[0] - 1)
    for c, S, pol in ((1, 1, 1), (2, 3, 1), (3, 2, 0), (100, 1, 1)):
        B = host(shape, dtype, sentinel=True)
        with pp.Region(0) as r:
            r.map("to", A, -1, 3)
            r.map("from", B)
            r.pipeline(c, S)
            r.set_option(pp.PP_OPT_STREAM_POLICY, pol)
            r.launch(1, shape[0] - 1, "conv3d")
        assert np.array_equal(as_bits(B), as_bits(ref)), (shape, c, S, pol)


def test_conv3d_naive_and_resident():
    A = host((24, 40, 48), torch.float32)
    ref = np.empty((24, 40, 48), dtype=np.float32)
    synth.fill_sentinel(ref)
    oracle.conv3d(A.numpy(), ref, 1, 23)
    B = host((24, 40, 48), torch.float32, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", A, -1, 3)
        r.map("from", B)
        r.naive(1, 23, "conv3d")
    assert np.array_equal(as_bits(B), as_bits(ref))
    dA, dB = A.cuda(), torch.empty_like(A, device="cuda")
    with pp.Region(0) as r:
        r.map("to", dA, -1, 3)
        r.map("from", dB)
        r.pipeline(0, 1)
        r.launch(1, 23, "conv3d")
    assert np.array_equal(as_bits(dB.cpu())[1:23], as_bits(ref)[1:23])


@pytest.mark.parametrize("dtype", [torch.float32, torch.float64])
@pytest.mark.parametrize("nz,ny,nx", [(130, 512, 512), (75, 200, 392)])
def test_conv3d_tma_resident_long_segments_bit_exact(dtype, nz, ny, nx):
    """One resident launch of the TMA kernel the bench times (kernels record): every CTA marches a
    z-segment of tens of planes, so each stage is refilled many times (fp32: by the last consumer warp
    to release it; fp64: by the producer warp); the second shape has ragged x and y tiles."""
    A = host((nz, ny, nx), dtype)
    ref = np.empty((nz, ny, nx), dtype=A.numpy().dtype)
    synth.fill_sentinel(ref)
    oracle.conv3d(A.numpy(), ref, 1, nz - 1)
    dA = A.cuda()
    dB = torch.empty_like(dA)
    with pp.Region(0) as r:
        r.map("to", dA, -1, 3)
        r.map("from", dB)
        r.pipeline(0, 1)
        r.set_option(pp.PP_OPT_KERNEL_PATH, pp.KPATH_TMA)
        r.launch(1, nz - 1, "conv3d")
        assert r.query()["kernel_path"] == pp.KPATH_TMA
    assert np.array_equal(as_bits(dB.cpu())[1:nz - 1], as_bits(ref)[1:nz - 1])


@pytest.mark.parametrize("c,S", [(32, 2), (30, 1)])
def test_conv3d_fp32_slot_filling_map_through_rings_bit_exact(c, S):
    """fp32 chunk launches long enough for the slot-filling z-segment map (>= 4 planes per segment at
    512^2: 64 tiles, q + 1 = 7 segments), through input/output rings that wrap, vs the oracle."""
    shape = (70, 512, 512)
    A = host(shape, torch.float32)
    ref = np.empty(shape, dtype=np.float32)
    synth.fill_sentinel(ref)
    oracle.conv3d(A.numpy(), ref, 1, shape[0] - 1)
    B = host(shape, torch.float32, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", A, -1, 3)
        r.map("from", B)
        r.pipeline(c, S)
        r.set_option(pp.PP_OPT_KERNEL_PATH, pp.KPATH_TMA)
        r.launch(1, shape[0] - 1, "conv3d")
        q = r.query()
    assert q["ring_planes"][0] < shape[0]                          # the input ring wraps
    assert np.array_equal(as_bits(B), as_bits(ref))


# ------------------------------------------------------------------ conv3d worked rounding examples
def _conv3d_worked_examples():
    import os
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    from test_oracle import conv3d_worked_examples
    return conv3d_worked_examples()


@pytest.mark.parametrize("path", [pp.KPATH_GENERIC, pp.KPATH_TMA])
def test_conv3d_worked_rounding_examples_gpu(path):
    """Both conv3d kernels reproduce the exact-rational hand derivation (tests/golden/
    conv3d_worked_examples.txt) bit for bit: Polybench order, no FMA. The 3x3x3 example sits inside a
    larger array (TMA rows must be 16-byte multiples) and the point is computed in a pipelined launch."""
    for (fmt, seed), (blk, want, _) in _conv3d_worked_examples().items():
        dtype = torch.float64 if fmt == "f64" else torch.float32
        A = torch.zeros((3, 16, 64), dtype=dtype).pin_memory()
        A[0:3, 4:7, 8:11] = torch.from_numpy(blk)
        B = host((3, 16, 64), dtype, sentinel=True)
        with pp.Region(0) as r:
            r.map("to", A, -1, 3)
            r.map("from", B)
            r.pipeline(1, 1)
            r.set_option(pp.PP_OPT_KERNEL_PATH, path)
            r.launch(1, 2, "conv3d")
            assert r.query()["kernel_path"] == path
        got = int(as_bits(B)[1, 5, 9])
        assert got == want, (fmt, seed, hex(got), hex(want))


# ------------------------------------------------------------------ interior-only copy-back (PP_OPT_D2H_INTERIOR)
def oracle_fig2(A0, lo, hi, c0, c1):
    ref = np.empty(tuple(A0.shape), dtype=A0.numpy().dtype)
    synth.fill_sentinel(ref)
    oracle.stencil7_fig2(A0.numpy(), ref, lo, hi, c0, c1)
    return ref


@pytest.mark.parametrize("dtype,shape", [(torch.float64, (21, 33, 40)), (torch.float32, (19, 70, 132)),
                                         (torch.float64, (30, 256, 256))])
@pytest.mark.parametrize("c,S,policy,graph,mirror", [(1, 1, 1, 0, 1), (2, 3, 1, 0, 1), (3, 2, 0, 0, 0),
                                                     (4, 3, 4, 1, 1), (6, 1, 1, 0, 1)])
def test_interior_d2h_equals_fig2_literal(dtype, shape, c, S, policy, graph, mirror):
    """Reading S5b: with PP_OPT_D2H_INTERIOR the host output equals Fig. 2 as printed — interior points
    of every computed plane, the host's edge points (sentinel here) and other planes untouched."""
    A0 = host(shape, dtype)
    c0, c1 = coeffs(dtype)
    lo, hi = 1, shape[0] - 1
    ref = oracle_fig2(A0, lo, hi, c0, c1)
    An = host(shape, dtype, sentinel=True)
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_MIRROR, mirror)
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(c, S)
        r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
        r.set_option(pp.PP_OPT_GRAPH, graph)
        r.set_option(pp.PP_OPT_D2H_INTERIOR, 1)
        for _ in range(2 if graph else 1):
            synth.fill_sentinel(An)
            r.launch(lo, hi, "stencil7", c0=c0, c1=c1)
        q = r.query()
    assert np.array_equal(as_bits(An), as_bits(ref))
    assert q["d2h_bytes"] == (hi - lo) * (shape[1] - 2) * (shape[2] - 2) * A0.element_size()


def test_interior_d2h_conv3d_chain_naive_inplace():
    # conv3d: interior = the oracle's interior, host edges untouched
    A = host((18, 40, 64), torch.float32)
    ref = np.empty((18, 40, 64), np.float32)
    synth.fill_sentinel(ref)
    oracle.conv3d(A.numpy(), ref, 1, 17)
    B = host((18, 40, 64), torch.float32, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", A, -1, 3)
        r.map("from", B)
        r.pipeline(3, 2)
        r.set_option(pp.PP_OPT_D2H_INTERIOR, 1)
        r.launch(1, 17, "conv3d")
    want = as_bits(ref).copy()
    sent = np.empty_like(ref)
    synth.fill_sentinel(sent)
    want[:, 0, :] = want[:, -1, :] = as_bits(sent)[:, 0, :]
    want[:, :, 0] = want[:, :, -1] = as_bits(sent)[:, :, 0]
    assert np.array_equal(as_bits(B), want)
    # a 4-sweep chain (fused L = 2) and the naive baseline: interior of A^T, edges untouched
    A0 = host((22, 34, 64), torch.float64)
    full = oracle_sweeps(A0, 1, 21, C0_64, C1_64, 4)
    want = as_bits(full).copy()
    sent = np.empty_like(full)
    synth.fill_sentinel(sent)
    want[:, 0, :] = want[:, -1, :] = as_bits(sent)[:, 0, :]
    want[:, :, 0] = want[:, :, -1] = as_bits(sent)[:, :, 0]
    for naive in (False, True):
        An = host((22, 34, 64), torch.float64, sentinel=True)
        with pp.Region(0) as r:
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.pipeline(2, 2)
            r.set_option(pp.PP_OPT_SWEEPS, 4)
            r.set_option(pp.PP_OPT_FUSE, 2)
            r.set_option(pp.PP_OPT_D2H_INTERIOR, 1)
            (r.naive if naive else r.launch)(1, 21, "stencil7", c0=C0_64, c1=C1_64)
            assert r.query()["d2h_bytes"] == 20 * 32 * 62 * 8
        assert np.array_equal(as_bits(An), want), naive
    # in place, interior-only copy-back gives the same host array as whole planes (edges = A0 there)
    outs = []
    for interior in (0, 1):
        B = A0.clone().pin_memory()
        with pp.Region(0) as r:
            r.set_option(pp.PP_OPT_INPLACE, 1)
            r.map("to", B, -1, 3)
            r.map("from", B)
            r.pipeline(3, 2)
            r.set_option(pp.PP_OPT_D2H_INTERIOR, interior)
            r.launch(1, 21, "stencil7", c0=C0_64, c1=C1_64)
        outs.append(as_bits(B).copy())
    assert np.array_equal(outs[0], outs[1])


def test_interior_d2h_unsupported_outputs():
    a = host((1 << 12,), torch.float32)
    b = host((1 << 12,), torch.float32)
    c = host((1 << 12,), torch.float32, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", a)
        r.map("to", b)
        r.map("from", c)
        r.set_option(pp.PP_OPT_D2H_INTERIOR, 1)
        with pytest.raises(pp.PPError) as ei:
            r.launch(0, 1 << 12, "triad", s=3.0)
        assert ei.value.status == pp.PP_EUNSUPPORTED


# ------------------------------------------------------------------ peer halo exchange (pp_halo_*)
def _slab(A, lo_g, hi_g, dtype):
    """Host buffer of global planes [lo_g - 1, hi_g + 1) (one rank's slab with its re-read halos)."""
    return torch.from_numpy(np.ascontiguousarray(A[lo_g - 1:hi_g + 1])).clone().pin_memory()


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
def test_peer_halo_same_device_functional(dtype):
    """configs[3] with the opt-in peer halo: two slab regions (ranks g-1, g) on cuda:0. Region g exports
    its first loaded plane lo_g into a side slot; region g-1 imports it as its upper halo instead of
    re-reading it from host memory (its host copy of that plane is poisoned, so the result is right
    only if the plane came from the side slot). Both slabs must equal the oracle's sweep of the whole
    array, over two launches with a bumped epoch."""
    nz, ny, nx = 40, 48, 64
    c0, c1 = coeffs(dtype)
    A = host((nz, ny, nx), dtype).numpy()
    ref = np.empty_like(A)
    synth.fill_sentinel(ref)
    oracle.stencil7(A, ref, 1, nz - 1, c0, c1)
    (l0, h0), (l1, h1) = pp.pp_partition(1, nz - 1, 2, 0), pp.pp_partition(1, nz - 1, 2, 1)
    lower, upper = _slab(A, l0, h0, dtype), _slab(A, l1, h1, dtype)
    lower[-1].fill_(12345.0)                      # the upper halo (global plane h0 = l1): must not be read
    out_lo = host(tuple(lower.shape), dtype, sentinel=True)
    out_up = host(tuple(upper.shape), dtype, sentinel=True)
    side = torch.empty((ny, nx), dtype=dtype, device="cuda")
    flag = torch.zeros(1, dtype=torch.int32, device="cuda")
    with pp.Region(0) as rl, pp.Region(0) as ru:
        for r, hb, ob in ((rl, lower, out_lo), (ru, upper, out_up)):
            r.map("to", hb, -1, 3)
            r.map("from", ob)
            r.pipeline(3, 2)
        for epoch in (1, 2):
            ru.halo_export(0, 1, side.data_ptr(), flag.data_ptr(), epoch)          # local 1 = global l1
            rl.halo_import(0, lower.shape[0] - 1, side.data_ptr(), 0, flag.data_ptr(), epoch)
            ru.launch_async(1, upper.shape[0] - 1, "stencil7", c0=c0, c1=c1)
            rl.launch_async(1, lower.shape[0] - 1, "stencil7", c0=c0, c1=c1)
            ru.wait()
            rl.wait()
            ql, qu = rl.query(), ru.query()
            assert ql["peer_bytes"] == ny * nx * lower.element_size() and qu["peer_bytes"] == 0
            assert ql["h2d_bytes"] == (lower.shape[0] - 1) * ny * nx * lower.element_size()
            assert int(flag.item()) == epoch
            assert np.array_equal(as_bits(out_lo)[1:-1], as_bits(ref)[l0:h0])
            assert np.array_equal(as_bits(out_up)[1:-1], as_bits(ref)[l1:h1])
        rl.halo_clear()
        with pytest.raises(pp.PPError):               # the plain re-read now sees the poisoned plane
            rl.halo_import(0, 0, 0, 0, 0, 0)
        rl.launch(1, lower.shape[0] - 1, "stencil7", c0=c0, c1=c1)
        assert not np.array_equal(as_bits(out_lo)[1:-1], as_bits(ref)[l0:h0])
        # a plane the launch does not load is rejected
        rl.halo_import(0, 0, side.data_ptr(), 0, flag.data_ptr(), 3)
        with pytest.raises(pp.PPError) as ei:
            rl.launch(2, lower.shape[0] - 1, "stencil7", c0=c0, c1=c1)
        assert ei.value.status == pp.PP_ERANGE


def test_peer_halo_missing_peer_fails_instead_of_hanging():
    """An import whose flag never reaches the epoch gives up after ~10 s and the launch fails with
    PP_ECUDA (no hang, no trap: the region stays usable and a plain re-read launch is exact)."""
    A = host((8, 16, 32), torch.float64)
    B = host((8, 16, 32), torch.float64, sentinel=True)
    side = torch.empty((16, 32), dtype=torch.float64, device="cuda")
    flag = torch.zeros(1, dtype=torch.int32, device="cuda")
    with pp.Region(0) as r:
        r.map("to", A, -1, 3)
        r.map("from", B)
        r.pipeline(2, 2)
        r.halo_import(0, 7, side.data_ptr(), 0, flag.data_ptr(), 1)
        with pytest.raises(pp.PPError) as ei:
            r.launch(1, 7, "stencil7", c0=C0_64, c1=C1_64)
        assert ei.value.status == pp.PP_ECUDA and "epoch" in ei.value.msg
        r.halo_clear()
        r.launch(1, 7, "stencil7", c0=C0_64, c1=C1_64)
    assert np.array_equal(as_bits(B), as_bits(oracle_stencil(A, 1, 7, C0_64, C1_64)))


# ------------------------------------------------------------------ device-side schedule check (PP_OPT_DEBUG_TAGS)
@pytest.mark.parametrize("dtype,shape", [(torch.float64, (21, 33, 40)), (torch.float64, (30, 512, 512)),
                                         (torch.float32, (19, 70, 132))])
@pytest.mark.parametrize("c,S,policy,mirror", [(1, 1, 0, 1), (2, 3, 1, 1), (3, 2, 3, 0), (4, 3, 4, 1), (6, 1, 1, 1)])
def test_debug_tags_see_a_correct_device_execution(dtype, shape, c, S, policy, mirror):
    """With slot tags checked by the device around every op, every schedule's real execution reads
    exactly the planned planes at the planned level, drains every output plane once, and stays exact."""
    A0 = host(shape, dtype)
    c0, c1 = coeffs(dtype)
    ref = oracle_stencil(A0, 1, shape[0] - 1, c0, c1)
    An = host(shape, dtype, sentinel=True)
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_MIRROR, mirror)
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(c, S)
        r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
        r.set_option(pp.PP_OPT_DEBUG_TAGS, 1)
        r.launch(1, shape[0] - 1, "stencil7", c0=c0, c1=c1)
        assert r.query()["debug_violations"] == 0, pp.pp_last_error()
        r.set_option(pp.PP_OPT_DEBUG_TAGS, 0)
        r.launch(1, shape[0] - 1, "stencil7", c0=c0, c1=c1)
        assert r.query()["debug_violations"] == -1
    assert np.array_equal(as_bits(An), as_bits(ref))


def test_debug_tags_chains_triad_conv_inplace():
    # a fused chain (level rings, levels 0..T), the triad, conv3d, and an in-place sweep
    A0 = host((23, 70, 132), torch.float32)
    c0, c1 = coeffs(torch.float32)
    for L in (1, 2):
        An = host((23, 70, 132), torch.float32, sentinel=True)
        with pp.Region(0) as r:
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.pipeline(3, 2)
            r.set_option(pp.PP_OPT_SWEEPS, 5)
            r.set_option(pp.PP_OPT_FUSE, L)
            r.set_option(pp.PP_OPT_DEBUG_TAGS, 1)
            r.launch(1, 22, "stencil7", c0=c0, c1=c1)
            assert r.query()["debug_violations"] == 0, pp.pp_last_error()
        assert np.array_equal(as_bits(An), as_bits(oracle_sweeps(A0, 1, 22, c0, c1, 5)))
    n = 1 << 16
    a, b = host((n,), torch.float32), host((n,), torch.float32, seed=synth.SEED_B)
    cc = host((n,), torch.float32, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", a)
        r.map("to", b)
        r.map("from", cc)
        r.pipeline(n // 7, 3)
        r.set_option(pp.PP_OPT_DEBUG_TAGS, 1)
        r.launch(0, n, "triad", s=3.0)
        assert r.query()["debug_violations"] == 0, pp.pp_last_error()
    B = host((23, 70, 132), torch.float32, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", B)
        r.pipeline(4, 2)
        r.set_option(pp.PP_OPT_DEBUG_TAGS, 1)
        r.launch(1, 22, "conv3d")
        assert r.query()["debug_violations"] == 0, pp.pp_last_error()
    C = A0.clone().pin_memory()
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_INPLACE, 1)
        r.map("to", C, -1, 3)
        r.map("from", C)
        r.pipeline(2, 3)
        r.set_option(pp.PP_OPT_DEBUG_TAGS, 1)
        r.launch(1, 22, "stencil7", c0=c0, c1=c1)
        assert r.query()["debug_violations"] == 0, pp.pp_last_error()


@pytest.mark.parametrize("fault", [2, 4])
def test_debug_tags_catch_planted_planner_bugs_on_the_device(fault):
    """The planner bugs pp_plan_check catches on the host are also caught by the DEVICE when executed:
    2 = input ring one plane too small (a kernel window reads an overwritten slot), 4 = drain from the
    wrong slot (mirrored rings, so the shifted copy stays inside the mapping)."""
    A0 = host((30, 512, 512), torch.float64)
    An = host((30, 512, 512), torch.float64, sentinel=True)
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_MIRROR, 1)
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(2, 3)
        r.set_option(pp.PP_OPT_FAULT_INJECT, fault)
        r.set_option(pp.PP_OPT_DEBUG_TAGS, 1)
        r.launch(1, 29, "stencil7", c0=C0_64, c1=C1_64)
        assert r.query()["debug_violations"] > 0
        assert "PP_OPT_DEBUG_TAGS" in pp.pp_last_error()


# ------------------------------------------------------------------ persistent pipeline kernel (PP_OPT_PERSISTENT)
@pytest.mark.parametrize("dtype,shape", [(torch.float64, (21, 64, 96)), (torch.float32, (19, 70, 132)),
                                         (torch.float64, (30, 512, 512))])
@pytest.mark.parametrize("c,S,mirror", [(1, 1, 1), (2, 3, 1), (3, 2, 0), (6, 1, 1), (4, 2, 1)])
def test_persistent_pipeline_bit_exact(dtype, shape, c, S, mirror):
    """One resident kernel for every chunk, handed over by flag words (stream memory operations):
    bit-exact against the oracle, repeated launches, one kernel launch per sweep."""
    A0 = host(shape, dtype)
    c0, c1 = coeffs(dtype)
    ref = oracle_stencil(A0, 1, shape[0] - 1, c0, c1)
    An = host(shape, dtype, sentinel=True)
    with pp.Region(0) as r:
        r.set_option(pp.PP_OPT_MIRROR, mirror)
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(c, S)
        r.set_option(pp.PP_OPT_PERSISTENT, 1)
        for _ in range(3):
            synth.fill_sentinel(An)
            r.launch(1, shape[0] - 1, "stencil7", c0=c0, c1=c1)
            q = r.query()
            assert q["n_kernels"] == 1 and q["kernel_path"] == pp.KPATH_TMA
            assert np.array_equal(as_bits(An), as_bits(ref)), (c, S, mirror)


def test_persistent_pipeline_configs1_and_rejections():
    n = 512
    A0 = host((n, n, n), torch.float64)
    ref = oracle_stencil(A0, 1, n - 1, C0_64, C1_64)
    An = host((n, n, n), torch.float64, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(6, 1)
        r.mem_limit(((8 + 6) * n * n) * 8)
        r.set_option(pp.PP_OPT_PERSISTENT, 1)
        r.launch(1, n - 1, "stencil7", c0=C0_64, c1=C1_64)
        assert r.query()["ring_planes"] == [8, 6]
    assert np.array_equal(as_bits(An), as_bits(ref))
    # the device really ran ONE pipeline kernel for the 85 chunks (CUPTI, not the library's own count)
    from torch.profiler import ProfilerActivity, profile
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.pipeline(6, 1)
        r.set_option(pp.PP_OPT_PERSISTENT, 1)
        r.launch(1, n - 1, "stencil7", c0=C0_64, c1=C1_64)
        torch.cuda.synchronize()
        with profile(activities=[ProfilerActivity.CUDA]) as prof:
            r.launch(1, n - 1, "stencil7", c0=C0_64, c1=C1_64)
            torch.cuda.synchronize()
    names = [e.name for e in prof.events() if "stencil7" in e.name]
    assert len([x for x in names if "pipe_kernel" in x]) == 1 and not [x for x in names if "tma_kernel" in x], names
    assert np.array_equal(as_bits(An), as_bits(ref))
    small = host((12, 16, 32), torch.float64)
    out = host((12, 16, 32), torch.float64, sentinel=True)
    for opt, val in ((pp.PP_OPT_SWEEPS, 2), (pp.PP_OPT_KERNEL_PATH, pp.KPATH_GENERIC), (pp.PP_OPT_DEBUG_TAGS, 1)):
        with pp.Region(0) as r:
            r.map("to", small, -1, 3)
            r.map("from", out)
            r.pipeline(2, 2)
            r.set_option(pp.PP_OPT_PERSISTENT, 1)
            r.set_option(opt, val)
            with pytest.raises(pp.PPError) as ei:
                r.launch(1, 11, "stencil7", c0=C0_64, c1=C1_64)
            assert ei.value.status == pp.PP_EUNSUPPORTED
    with pp.Region(0) as r:                           # pageable arrays: copies must be pinned
        r.set_option(pp.PP_OPT_AUTO_PIN, 0)
        r.map("to", small.numpy().copy(), -1, 3)
        r.map("from", np.zeros((12, 16, 32)))
        r.pipeline(2, 2)
        r.set_option(pp.PP_OPT_PERSISTENT, 1)
        with pytest.raises(pp.PPError) as ei:
            r.launch(1, 11, "stencil7", c0=C0_64, c1=C1_64)
        assert ei.value.status == pp.PP_EUNSUPPORTED


# ------------------------------------------------------------------ plain-C caller of the C ABI
@pytest.mark.parametrize("sweeps", [1, 3])
def test_c_example_matches_oracle(tmp_path, sweeps):
    import os
    import subprocess
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    exe = os.path.join(root, "examples", "stencil_offload")
    nz, ny, nx = 23, 30, 34
    out = tmp_path / "an.bin"
    res = subprocess.run([exe, str(nz), str(ny), str(nx), str(out), str(sweeps)], capture_output=True, text=True)
    assert res.returncode == 0, res.stderr
    got = np.fromfile(out, dtype=np.float64).reshape(nz, ny, nx)
    A0 = (np.arange(nz * ny * nx) % 1000 / 1000.0).reshape(nz, ny, nx)
    ref = A0.copy()
    oracle.stencil7_sweeps(A0, ref, 1, nz - 1, 1.0 / 6.0, (1.0 / 6.0) / 6.0, sweeps)
    assert np.array_equal(got.view(np.uint64), ref.view(np.uint64))


def test_autotune_chain_stays_exact():
    A0 = host((60, 64, 64), torch.float64)
    An = host((60, 64, 64), torch.float64, sentinel=True)
    ref = oracle_sweeps(A0, 1, 59, C0_64, C1_64, 6)
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        r.set_option(pp.PP_OPT_SWEEPS, 6)
        r.mem_limit(80 * 64 * 64 * 8)
        res = r.autotune(1, 59, "stencil7", trials=3, c0=C0_64, c1=C1_64)
        assert res["trials"] == 3
        synth.fill_sentinel(An)
        r.launch(1, 59, "stencil7", c0=C0_64, c1=C1_64)
        assert r.query()["ring_bytes"] <= 80 * 64 * 64 * 8
    assert np.array_equal(as_bits(An), as_bits(ref))


# ------------------------------------------------------------------ out-of-core tool (configs[2] path)
def test_ooc_tool_in_place_16GB_fully_verified():
    import json
    import os
    import subprocess
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    res = subprocess.run([sys.executable, os.path.join(root, "tests", "ooc_run.py"), "--gb", "16"],
                         capture_output=True, text=True, timeout=600)
    assert res.returncode == 0, res.stderr[-2000:]
    rec = json.loads(res.stdout.strip().splitlines()[-1])
    assert rec["verify"]["mismatches"] == 0 and rec["verify"]["planes_checked"] == rec["host_array_bytes"] // (4096 * 4096 * 4) - 2
    assert rec["ring_bytes"] <= 4e9 and rec["e2e_gbs"] > 20


def test_ooc_tool_exceeds_hbm_fully_verified():
    """The north_star target (BASELINE.json configs[2]): a host array LARGER THAN THE GPU's HBM (sized
    from MemAvailable, in place), 4e9 B device budget, every one of its planes bit-exact against the
    oracle's verify-in-place. Skipped only when the box has too little host RAM to exceed HBM."""
    import json
    import os
    import subprocess
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    res = subprocess.run([sys.executable, os.path.join(root, "tests", "ooc_run.py"), "--gb", "auto"],
                         capture_output=True, text=True, timeout=1200)
    assert res.returncode == 0, res.stderr[-2000:]
    rec = json.loads(res.stdout.strip().splitlines()[-1])
    if rec["size_capped_by_host_ram"] and not rec["exceeds_hbm"]:
        pytest.skip(f"host RAM ({rec['host_mem_available'] / 1e9:.0f} GB available) cannot exceed HBM")
    assert rec["exceeds_hbm"] and rec["host_array_bytes"] > rec["hbm_total_bytes"]
    nz = rec["host_array_bytes"] // (4096 * 4096 * 4)
    assert rec["verify"]["mismatches"] == 0 and rec["verify"]["planes_checked"] == nz - 2
    assert rec["ring_bytes"] <= 4e9 and rec["frac_of_duplex_roofline"] > 0.8


def test_ooc_tool_two_ranks_slab_partitioned_verified():
    """configs[3] path: two torchrun ranks (sharing cuda:0 here) each pipeline their slab of the global
    array from their own host buffer with re-read halo planes; every plane of both slabs bit-exact."""
    import json
    import os
    import random
    import subprocess
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, PP_BENCH_SHARE_GPU="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(random.randint(29600, 29900)),
           os.path.join(root, "tests", "ooc_run.py"), "--gb", "2", "--nx", "1024", "--ny", "1024", "--budget", "2e8"]
    res = subprocess.run(cmd, capture_output=True, text=True, timeout=600, env=env)
    assert res.returncode == 0, res.stderr[-3000:]
    rec = json.loads([ln for ln in res.stdout.strip().splitlines() if ln.startswith("{")][-1])
    nz = rec["host_array_bytes"] // (1024 * 1024 * 4)
    assert rec["ranks"] == 2 and rec["verify"]["mismatches"] == 0
    assert rec["verify"]["planes_checked"] == nz - 2          # the two slabs cover the loop exactly once
    assert rec["h2d_bytes"] == (nz + 2) * 1024 * 1024 * 4     # plus the two re-read halo planes


# ------------------------------------------------------------------ 2-D block regions (NEXT-3)
@pytest.mark.parametrize("shape,split_dim", [((37, 1000), 1), ((5, 6, 301), 2), ((9, 40, 33), 1)])
@pytest.mark.parametrize("c,S", [(1, 2), (16, 3), (64, 1)])
def test_triad_2d_block_region_bit_exact(shape, split_dim, c, S):
    a = host(shape, torch.float32, seed=synth.SEED_A)
    b = host(shape, torch.float32, seed=synth.SEED_B)
    cc = host(shape, torch.float32, sentinel=True)
    n = shape[split_dim]
    with pp.Region(0) as r:
        r.map("to", a, split_dim=split_dim)
        r.map("to", b, split_dim=split_dim)
        r.map("from", cc, split_dim=split_dim)
        r.pipeline(c, S)
        r.launch(0, n, "triad", s=3.0)
        q = r.query()
    ref = np.empty(a.numel(), np.float32)
    oracle.triad(a.numpy().ravel(), b.numpy().ravel(), np.float32(3.0), ref)
    assert np.array_equal(as_bits(cc).ravel(), ref.view(np.uint32))
    assert q["h2d_bytes"] == 2 * a.numel() * 4 and q["d2h_bytes"] == a.numel() * 4


def test_triad_2d_block_region_subrange_keeps_other_columns():
    a = host((20, 300), torch.float64, seed=1)
    b = host((20, 300), torch.float64, seed=2)
    cc = host((20, 300), torch.float64, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", a, split_dim=1)
        r.map("to", b, split_dim=1)
        r.map("from", cc, split_dim=1)
        r.pipeline(32, 2)
        r.launch(50, 250, "triad", s=3.0)
    ref = np.empty((20, 300))
    oracle.triad(a.numpy().ravel(), b.numpy().ravel(), 3.0, ref.ravel())
    assert np.array_equal(as_bits(cc)[:, 50:250], ref.view(np.uint64)[:, 50:250])
    assert synth.count_sentinel(cc[:, :50].contiguous()) == 20 * 50
    assert synth.count_sentinel(cc[:, 250:].contiguous()) == 20 * 50


def test_paper_matmul_pipeline_buffer_with_2d_regions():
    # PAPER.md §V.E "pipeline-buffer" matmul: per k-block task, the column block of A and
    # the row block of B are copied into small device buffers (A's block is non-contiguous: a 2-D
    # region) and C += A_blk @ B_blk. The GEMM itself is a library call inside a user body; integer
    # data keeps every sum exact, so the blocked result must equal A @ B bit for bit.
    M, K, N = 96, 512, 80
    g = torch.Generator().manual_seed(7)
    A = torch.randint(-8, 9, (M, K), generator=g).to(torch.float64).pin_memory()
    B = torch.randint(-8, 9, (K, N), generator=g).to(torch.float64).pin_memory()
    C = torch.zeros((M, N), dtype=torch.float64, device="cuda")

    def body(chunk, stream):
        st = torch.cuda.ExternalStream(stream)
        with torch.cuda.stream(st):
            for p, n in pp.ring_runs(chunk, 0, chunk.k0, chunk.k1):
                a_blk = torch.as_tensor(pp.block_view(chunk, 0, p, n), device="cuda")          # M x n
                b_blk = torch.as_tensor(pp.chunk_view(chunk, 1, p, n, plane_shape=(N,)), device="cuda")
                C.add_(a_blk @ b_blk.reshape(n, N))
        return 0

    with pp.Region(0) as r:
        r.map("to", A, split_dim=1)            # column blocks of A: 2-D region
        r.map("to", B)                         # row blocks of B: contiguous planes
        r.pipeline(32, 3)
        r.set_option(pp.PP_OPT_STREAM_POLICY, 1)   # one kernel stream: the C += ... updates are ordered
        r.launch_fn(0, K, body)
        q = r.query()
    torch.cuda.synchronize()
    assert torch.equal(C.cpu(), A @ B)
    assert q["ring_bytes"] < (M * K + K * N) * 8 / 4     # blocks, not whole matrices, on the device


@pytest.mark.parametrize("path", [pp.KPATH_GENERIC, pp.KPATH_TMA])
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32])
@pytest.mark.parametrize("shape,c,S", [((9, 17, 8), 1, 1), ((21, 40, 264), 3, 2), ((40, 70, 200), 100, 1)])
def test_conv3d_both_paths_bit_exact(path, dtype, shape, c, S):
    A = host(shape, dtype)
    ref = np.empty(shape, dtype=A.numpy().dtype)
    synth.fill_sentinel(ref)
    oracle.conv3d(A.numpy(), ref, 1, shape[0] - 1)
    B = host(shape, dtype, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", A, -1, 3)
        r.map("from", B)
        r.pipeline(c, S)
        r.set_option(pp.PP_OPT_KERNEL_PATH, path)
        r.launch(1, shape[0] - 1, "conv3d")
        assert r.query()["kernel_path"] == path
    assert np.array_equal(as_bits(B), as_bits(ref))


# ------------------------------------------------------------------ mirrored rings (PP_OPT_MIRROR)
@pytest.mark.parametrize("dtype,shape", [(torch.float64, (30, 512, 512)), (torch.float32, (30, 512, 1024))])
@pytest.mark.parametrize("c,S,policy,graph", [(6, 1, 1, 0), (3, 2, 1, 0), (5, 2, 3, 0), (2, 3, 4, 1), (4, 3, 0, 0)])
def test_mirrored_rings_bit_exact_one_copy_per_chunk(dtype, shape, c, S, policy, graph):
    """2 MiB planes: every ring is a whole number of VMM granules, so it is mapped twice and the
    chunks whose planes wrap past the ring end are copied with ONE cudaMemcpyAsync each."""
    A0 = host(shape, dtype)
    nz = shape[0]
    ref = oracle_stencil(A0, 1, nz - 1, *coeffs(dtype))
    outs = {}
    for mirror in (1, 0):
        An = host(shape, dtype, sentinel=True)
        c0, c1 = coeffs(dtype)
        with pp.Region(0) as r:
            r.set_option(pp.PP_OPT_MIRROR, mirror)
            r.map("to", A0, -1, 3)
            r.map("from", An)
            r.pipeline(c, S)
            r.set_option(pp.PP_OPT_STREAM_POLICY, policy)
            r.set_option(pp.PP_OPT_GRAPH, graph)
            for _ in range(2):                       # second launch replays the graph / reuses rings
                synth.fill_sentinel(An)
                r.launch(1, nz - 1, "stencil7", c0=c0, c1=c1)
            outs[mirror] = r.query()
        assert np.array_equal(as_bits(An), as_bits(ref)), (mirror, c, S)
    on, off = outs[1], outs[0]
    nch = on["nchunks"]
    assert on["n_h2d"] == nch and on["n_d2h"] == nch        # one copy per chunk and array
    assert off["n_h2d"] >= on["n_h2d"] and off["ring_bytes"] == on["ring_bytes"]


def test_mirrored_rings_reallocate_when_the_plan_changes():
    A0 = host((40, 512, 512), torch.float64)
    ref = oracle_stencil(A0, 1, 39, C0_64, C1_64)
    An = host((40, 512, 512), torch.float64, sentinel=True)
    with pp.Region(0) as r:
        r.map("to", A0, -1, 3)
        r.map("from", An)
        for c, S in ((3, 2), (6, 1), (2, 3), (7, 2)):
            r.pipeline(c, S)
            synth.fill_sentinel(An)
            r.launch(1, 39, "stencil7", c0=C0_64, c1=C1_64)
            q = r.query()
            assert np.array_equal(as_bits(An), as_bits(ref)), (c, S)
            assert q["n_h2d"] == q["nchunks"], (c, S, q["n_h2d"])


def test_mirrored_rings_chain_and_fused_bit_exact():
    A0 = host((36, 512, 512), torch.float64)
    ref = oracle_sweeps(A0, 1, 35, C0_64, C1_64, 4)
    for fuse in (1, 2):
        An, info = run_sweeps(A0, 1, 35, 4, 5, 2, fuse=fuse)
        assert np.array_equal(as_bits(An), as_bits(ref)), fuse
        assert info["n_h2d"] == info["nchunks"] and info["n_d2h"] == info["nchunks"]


def test_mirror_option_validation():
    with pp.Region(0) as r:
        with pytest.raises(pp.PPError) as e:
            r.set_option(pp.PP_OPT_MIRROR, -1)
        assert e.value.status == pp.PP_EINVAL


def test_mirrored_rings_are_released():
    """Regions with mirrored rings give their VMM memory back on destroy and on re-plans."""
    A0 = host((30, 512, 512), torch.float64)
    An = host((30, 512, 512), torch.float64, sentinel=True)
    torch.cuda.synchronize()
    free0 = torch.cuda.mem_get_info(0)[0]
    for c, S in ((6, 1), (3, 2), (4, 3), (6, 1), (2, 3)):
        with pp.Region(0) as r:
            r.map("to", A0, -1, 3)
            r.map("from", An)
            for cc in (c, 1 + c // 2):              # a re-plan inside the region, too
                r.pipeline(cc, S)
                r.launch(1, 29, "stencil7", c0=C0_64, c1=C1_64)
                q = r.query()
                assert q["n_h2d"] == q["nchunks"]
    torch.cuda.synchronize()
    assert torch.cuda.mem_get_info(0)[0] >= free0 - (64 << 20)


def test_mirror_refused_falls_back_to_split_copies():
    """If the driver refuses the VMM mapping, auto mode re-plans with plain rings (split copies) and
    the launch still succeeds bit-exactly (subprocess: the refusal switch is read once per process)."""
    import os
    import subprocess
    code = r'''
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import oracle, synth, paper_conf_ipps_cuissf17_b200 as pp
A0 = torch.empty((30, 512, 512), dtype=torch.float64, pin_memory=True)
synth.fill(A0, "random", seed=synth.SEED_A, nx=512, ny=512)
An = torch.empty_like(A0).pin_memory(); synth.fill_sentinel(An)
ref = np.empty((30, 512, 512)); synth.fill_sentinel(ref)
oracle.stencil7(A0.numpy(), ref, 1, 29, 1 / 6, 1 / 36)
with pp.Region(0) as r:
    r.map("to", A0, -1, 3); r.map("from", An); r.pipeline(6, 1)
    r.launch(1, 29, "stencil7", c0=1 / 6, c1=1 / 36)
    q = r.query()
assert q["n_h2d"] > q["nchunks"], q
assert np.array_equal(An.numpy().view(np.uint64), ref.view(np.uint64))
print("ok")
'''
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    res = subprocess.run([sys.executable, "-c", code, root], capture_output=True, text=True, timeout=300,
                         env=dict(os.environ, PP_TEST_REFUSE_VMM="1"))
    assert res.returncode == 0 and "ok" in res.stdout, res.stderr[-2000:]
