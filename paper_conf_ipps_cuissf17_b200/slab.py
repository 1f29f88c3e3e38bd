"""Slab sharding of the split dimension across ranks (BASELINE.json configs[3]).

Each rank pipelines a contiguous, balanced slab of the loop [lo, hi) (pp_partition) through its own
host link. Its host buffer holds the planes its windows touch — the slab plus the halo planes, which
are RE-READ from host memory (generated or copied by the owner of that process) rather than
exchanged between GPUs (north_star: NCCL only if a measured peer exchange beats the re-read).
"""
from dataclasses import dataclass

from . import pp_partition


@dataclass(frozen=True)
class Slab:
    lo: int          # global first iteration of this rank
    hi: int          # global end iteration
    p0: int          # first global plane held in this rank's host buffer
    p1: int          # end global plane held
    halo_planes: int  # planes this rank re-reads that another rank's slab also reads

    @property
    def nplanes(self):
        return self.p1 - self.p0

    def local(self, k):
        """Global plane/iteration k -> index into this rank's host buffer."""
        return k - self.p0


def slab(lo, hi, world, rank, split_offset=-1, split_size=3):
    """Slab of rank `rank` for a loop [lo,hi) whose input windows are [k+off, k+off+size)."""
    a, b = pp_partition(lo, hi, world, rank)
    p0 = a + split_offset
    p1 = b + split_offset + split_size - 1
    halo = (split_size - 1) if world > 1 else 0
    if world > 1 and rank in (0, world - 1):
        halo = (split_size - 1) // 2 if split_size > 1 else 0
    return Slab(a, b, p0, p1, halo)
