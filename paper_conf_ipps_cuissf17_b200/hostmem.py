"""Host arrays for out-of-core sweeps.

The copy engines translate host addresses page by page. Measured on the B200 box: a
192 GB pinned array backed by 4 KiB pages streams at 11/21 GB/s (H2D/D2H); the same array backed by
2 MiB transparent huge pages streams at 48/50 GB/s. `alloc_host` returns a numpy array on an
anonymous mapping advised MADV_HUGEPAGE (allocate it before other large allocations, while memory is
unfragmented); pp_map page-locks it (cudaHostRegister) when mapped.
"""
import mmap

import numpy as np


def alloc_host(shape, dtype=np.float32):
    nbytes = int(np.prod(shape)) * np.dtype(dtype).itemsize
    m = mmap.mmap(-1, max(nbytes, 1), flags=mmap.MAP_PRIVATE | mmap.MAP_ANONYMOUS)
    try:
        m.madvise(mmap.MADV_HUGEPAGE)
    except (AttributeError, OSError):
        pass
    return np.frombuffer(m, dtype=dtype, count=int(np.prod(shape))).reshape(shape)


def bind_local_cpus(device):
    """Restrict this process to the CPUs NVML reports as local to CUDA device `device` (its NUMA
    node), so the pinned host slab this rank first-touches lands in memory next to the GPU's PCIe
    root. One process per GPU (bench.py under torchrun) calls it before allocating host arrays.
    Returns the sorted CPU list it bound to, or None when NVML cannot say (nothing changed)."""
    import os
    try:
        import pynvml
        import torch
        props = torch.cuda.get_device_properties(device)
        bus = "%08x:%02x:%02x.0" % (props.pci_domain_id, props.pci_bus_id, props.pci_device_id)
        pynvml.nvmlInit()
        try:
            h = pynvml.nvmlDeviceGetHandleByPciBusId(bus)
            words = pynvml.nvmlDeviceGetCpuAffinity(h, (os.cpu_count() + 63) // 64)
        finally:
            pynvml.nvmlShutdown()
        cpus = [64 * w + b for w, m in enumerate(words) for b in range(64) if (int(m) >> b) & 1]
        cpus = [c for c in cpus if c in os.sched_getaffinity(0)]
        if not cpus:
            return None
        os.sched_setaffinity(0, cpus)
        return sorted(cpus)
    except Exception:
        return None
