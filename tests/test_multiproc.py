"""World-size-2 CPU test (gloo) of the N>1 path's host logic: slab partition, halo re-read from each
rank's own host buffer, the barrier and the max-over-ranks reduction bench.py uses. Each rank plans
its slab with a host-only region (pp_plan_check) and produces its slab's output with the oracle;
rank 0 checks that the gathered slabs equal the oracle over the whole array."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, nz, ny, nx, q):
    import oracle
    import paper_conf_ipps_cuissf17_b200 as pp
    import synth
    from paper_conf_ipps_cuissf17_b200.slab import slab
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        s = slab(1, nz - 1, world, rank)
        # this rank's host buffer: planes [p0, p1) generated at their GLOBAL indices
        A = np.empty((s.nplanes, ny, nx))
        synth.fill(A, "random", seed=synth.SEED_A, g0=s.p0 * ny * nx, nx=nx, ny=ny)
        out = np.zeros_like(A)
        r = pp.Region(-1)
        r.map("to", A, -1, 3)
        r.map("from", out)
        r.pipeline(2, 3)
        v, why = r.plan_check(s.local(s.lo), s.local(s.hi), orders=4)
        r.close()
        c0 = 1.0 / 6.0
        oracle.stencil7(A, out, s.local(s.lo), s.local(s.hi), c0, c0 / 6.0)
        mine = torch.from_numpy(out[s.local(s.lo):s.local(s.hi)].copy())
        sizes = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(sizes, torch.tensor([mine.shape[0]]))
        m = int(max(sizes).item())                          # gloo all_gather needs equal shapes
        pad = torch.zeros((m, ny, nx), dtype=torch.float64)
        pad[: mine.shape[0]] = mine
        gathered = [torch.zeros((m, ny, nx), dtype=torch.float64) for _ in sizes]
        dist.all_gather(gathered, pad)
        gathered = [g[: int(n)] for g, n in zip(gathered, sizes)]
        t = torch.tensor([float(rank + 1)], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)           # bench.py's max-over-ranks timing
        dist.barrier()
        if rank == 0:
            full = np.empty((nz, ny, nx))
            synth.fill(full, "random", seed=synth.SEED_A, nx=nx, ny=ny)
            ref = np.zeros_like(full)
            oracle.stencil7(full, ref, 1, nz - 1, c0, c0 / 6.0)
            got = torch.cat(gathered).numpy()
            q.put((v, why, bool(np.array_equal(got.view(np.uint64), ref[1:nz - 1].view(np.uint64))),
                   float(t.item()), [tuple(x.shape) for x in gathered]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("nz", [21, 64])
def test_two_rank_slabs_equal_whole_array(nz):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, nz, 9, 12, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = q.get(timeout=120)
    for p in ps:
        p.join(60)
        assert p.exitcode == 0
    v, why, equal, tmax, shapes = res
    assert v == 0, why
    assert equal
    assert tmax == 2.0
    assert sum(s[0] for s in shapes) == nz - 2


def test_slab_halo_windows():
    from paper_conf_ipps_cuissf17_b200.slab import slab
    s0, s1 = slab(1, 511, 2, 0), slab(1, 511, 2, 1)
    assert (s0.lo, s0.hi, s1.lo, s1.hi) == (1, 256, 256, 511)
    assert (s0.p0, s0.p1) == (0, 257) and (s1.p0, s1.p1) == (255, 512)   # planes 255,256 read twice


def _sizing_worker(rank, world, port, avail, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench
    import paper_conf_ipps_cuissf17_b200 as pp
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        cx = bench.Ctx(torch, dist, world, rank, 0, share=True)
        plane = 4096 * 4096 * 4
        want, limit = bench.ooc_global_planes("auto", 192_265_846_784, plane, avail[rank], 12.0, world)
        nz = int(cx.reduce(float(min(want, limit)), "min"))
        lo, hi = pp.pp_partition(1, nz - 1, world, rank)
        spans = [torch.zeros(2, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(spans, torch.tensor([lo, hi]))
        q.put((rank, nz, [tuple(x.tolist()) for x in spans]))
    finally:
        dist.destroy_process_group()


def test_bench_ooc_sizing_agrees_across_ranks():
    """bench.py's configs[3] sizing: ranks that read different MemAvailable values agree on ONE global
    array (all-reduce MIN) before allocating, and their slabs tile [1, nz-1) without gap or overlap."""
    world, port = 2, _free_port()
    avail = [260e9, 230e9]                    # rank 1 reads less free memory than rank 0
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_sizing_worker, args=(r, world, port, avail, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    plane = 4096 * 4096 * 4
    nz = {r[1] for r in res}
    assert len(nz) == 1
    nz = nz.pop()
    assert nz == min(int(-(-192_265_846_784 * 1.005 // plane)) + 2, int((230e9 - 12e9) // plane) - 2)
    spans = res[0][2]
    assert spans == res[1][2] and spans[0][0] == 1 and spans[0][1] == spans[1][0] and spans[1][1] == nz - 1
