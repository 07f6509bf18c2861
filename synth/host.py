"""Host-side storage, schedule and placement of the synthetic workloads.

Neutral module: it holds none of the method's arithmetic and never loads libgd.so, so both
bench.py arms (the CUDA path and the oracle reference arm), the tests and the product's
multigpu helpers can use it.

  * batch_schedule: GNNDrive "divides the entire training set into segments for subprocesses
    to execute": rank r runs the contiguous segment r of the global batch list
    (synth.segment), wrapping with one epoch per wrap.
  * SharedArray / HostTable: "topological data and staging buffer are shared among
    subprocesses": world == 1 -> private anonymous memory; world > 1 -> one /dev/shm
    file created by rank 0 and mapped by every rank (capacity checked before creation).
  * NUMA placement: each rank's threads bound to the CPUs local to its GPU (the PCIe root
    complex's socket, /sys/bus/pci/devices/<bdf>/local_cpulist), and the shared table
    interleaved over the sockets while it is faulted in.
"""
from __future__ import annotations

import ctypes
import mmap
import os
import platform

import numpy as np
import torch

from . import segment


def batch_schedule(num_batches: int, rank: int, world: int, steps: int):
    """(global batch index, epoch) for this rank's first `steps` steps; wraps around the
    segment, one epoch per wrap.  The Philox batch key is epoch * num_batches + b, so every
    (epoch, batch) pair draws an independent sample regardless of the GPU count."""
    seg = segment(num_batches, rank, world)
    if len(seg) == 0:
        return []
    return [(seg[j % len(seg)], j // len(seg)) for j in range(steps)]


# ------------------------------------------------------------------------------ NUMA
def parse_cpulist(text: str):
    out = []
    for part in text.strip().split(","):
        if part:
            lo, _, hi = part.partition("-")
            out.extend(range(int(lo), int(hi or lo) + 1))
    return out


def numa_nodes():
    """Online NUMA node ids (empty if unknown)."""
    try:
        with open("/sys/devices/system/node/online") as f:
            return parse_cpulist(f.read())
    except OSError:
        return []


def set_interleave(enable: bool) -> bool:
    """Interleave this thread's future page allocations over all online NUMA nodes
    (set_mempolicy(MPOL_INTERLEAVE)), or restore the default policy.  Used while rank 0
    faults the shared host table in, so that on a multi-socket box the random row reads of
    all GPUs' miss streams spread over every socket's memory controllers.  Returns False (and
    changes nothing) on a single-node host or where the syscall is unavailable."""
    nodes = numa_nodes()
    if len(nodes) < 2 and enable:
        return False
    nr = {"x86_64": 238, "aarch64": 237}.get(platform.machine())
    if nr is None:
        return False
    try:
        libc = ctypes.CDLL(None, use_errno=True)
        mask = (ctypes.c_ulong * 16)()
        for n in nodes:
            mask[n // 64] |= 1 << (n % 64)
        mode = 3 if enable else 0                      # MPOL_INTERLEAVE / MPOL_DEFAULT
        rc = libc.syscall(nr, mode, mask if enable else None, ctypes.c_ulong(1024 if enable else 0))
        return rc == 0
    except (OSError, AttributeError):
        return False


def gpu_pci_bdf(device_index: int) -> str | None:
    """PCI address (dddd:bb:dd.f, lower case) of CUDA device `device_index`, from NVML."""
    try:
        import pynvml as N
        N.nvmlInit()
        uuid = torch.cuda.get_device_properties(device_index).uuid
        h = None
        for i in range(N.nvmlDeviceGetCount()):
            hi = N.nvmlDeviceGetHandleByIndex(i)
            u = N.nvmlDeviceGetUUID(hi)
            u = u.decode() if isinstance(u, bytes) else u
            if u.replace("GPU-", "") == str(uuid).replace("GPU-", ""):
                h = hi
                break
        if h is None:
            h = N.nvmlDeviceGetHandleByIndex(device_index)
        bus = N.nvmlDeviceGetPciInfo(h).busId
        bus = bus.decode() if isinstance(bus, bytes) else bus
        dom, rest = bus.split(":", 1)
        return f"{int(dom, 16) & 0xFFFF:04x}:{rest.lower()}"
    except Exception:  # noqa: BLE001
        return None


def gpu_local_cpus(device_index: int):
    """(CPUs local to the GPU's PCIe root, its NUMA node, bdf); ([], -1, bdf) if unknown."""
    bdf = gpu_pci_bdf(device_index)
    if not bdf:
        return [], -1, None
    base = f"/sys/bus/pci/devices/{bdf}"
    try:
        with open(f"{base}/local_cpulist") as f:
            cpus = parse_cpulist(f.read())
    except OSError:
        cpus = []
    try:
        with open(f"{base}/numa_node") as f:
            node = int(f.read().strip())
    except (OSError, ValueError):
        node = -1
    return cpus, node, bdf


def bind_to_gpu_socket(device_index: int) -> dict:
    """Restrict this process (and the threads it creates afterwards: the host-gather pool,
    the CUDA callback thread) to the CPUs local to its GPU, intersected with the current
    affinity mask, so its pinned staging memory is first-touched on the GPU's socket (SURVEY
    §8(e)).  No-op on a single-socket host or when the topology is unknown."""
    have = sorted(os.sched_getaffinity(0))
    cpus, node, bdf = gpu_local_cpus(device_index)
    use = sorted(set(cpus) & set(have))
    rep = {"gpu_bdf": bdf, "gpu_numa_node": node, "numa_nodes": len(numa_nodes()), "cpus_before": len(have)}
    if len(numa_nodes()) < 2 or not use or len(use) == len(have):
        rep.update(bound=False, cpus=len(have))
        return rep
    os.sched_setaffinity(0, use)
    rep.update(bound=True, cpus=len(use))
    return rep


# ------------------------------------------------------------------------ shared memory
def shm_free_bytes(path: str) -> int:
    st = os.statvfs(path)
    return st.f_bavail * st.f_frsize


class SharedArray:
    """A C-contiguous numpy array.  world == 1: private anonymous memory.  world > 1: one
    file under `shm_dir` (env GD_SHM_DIR, default /dev/shm) created by rank 0 and mapped by
    every rank; rank 0 checks the filesystem's free space first and fails with a clear
    message instead of letting a short tmpfs SIGBUS a rank mid-fill."""

    def __init__(self, shape, dtype, name: str, rank: int = 0, world: int = 1, shm_dir: str | None = None):
        self.shape = tuple(int(x) for x in shape)
        self.dtype = np.dtype(dtype)
        nbytes = int(np.prod(self.shape)) * self.dtype.itemsize
        self.path = None
        self._mm = None
        self.owner = rank == 0
        self.thp = False
        if world == 1:
            # private anonymous mapping with transparent huge pages requested (env GD_THP=0: off):
            # the host gather's random row reads then miss the TLB far less (measured on this
            # pool's boxes, 57 GB table, 512 B rows, 16 threads: 46.4 -> 53.5 GB/s)
            self._mm = mmap.mmap(-1, max(1, nbytes), flags=mmap.MAP_PRIVATE | mmap.MAP_ANONYMOUS)
            if os.environ.get("GD_THP", "1") == "1" and hasattr(mmap, "MADV_HUGEPAGE"):
                try:
                    self._mm.madvise(mmap.MADV_HUGEPAGE)
                    self.thp = True
                except OSError:
                    pass
            self.array = np.frombuffer(self._mm, dtype=self.dtype, count=int(np.prod(self.shape))).reshape(self.shape)
            return
        shm_dir = shm_dir or os.environ.get("GD_SHM_DIR", "/dev/shm")
        self.path = os.path.join(shm_dir, f"gd_{name}_{'x'.join(map(str, self.shape))}_{self.dtype.str[1:]}")
        err = None
        if rank == 0:
            free = shm_free_bytes(shm_dir)
            if free < nbytes:
                err = (f"{shm_dir} has {free / 2**30:.1f} GiB free but the shared {name} needs "
                       f"{nbytes / 2**30:.1f} GiB: enlarge it (mount -o remount,size=...) or set GD_SHM_DIR")
            else:
                with open(self.path, "wb") as f:
                    f.truncate(nbytes)
        flag = torch.tensor([1 if err else 0], dtype=torch.int32)
        import torch.distributed as dist
        if dist.is_available() and dist.is_initialized():
            if dist.get_backend() != "gloo":
                flag = flag.cuda()
            dist.broadcast(flag, 0)
        if int(flag.item()):
            raise RuntimeError(err or f"rank 0 could not create the shared {name} under {shm_dir} (see rank 0)")
        fd = os.open(self.path, os.O_RDWR)
        try:
            self._mm = mmap.mmap(fd, nbytes, mmap.MAP_SHARED, mmap.PROT_READ | mmap.PROT_WRITE)
        finally:
            os.close(fd)
        self.array = np.frombuffer(self._mm, dtype=self.dtype).reshape(self.shape)

    def close(self, unlink: bool = True):
        self.array = None
        if self._mm is not None:
            try:
                self._mm.close()
            except BufferError:
                pass
            self._mm = None
        if unlink and self.owner and self.path and os.path.exists(self.path):
            os.unlink(self.path)


class HostTable(SharedArray):
    """The [P, R] uint8 host feature table (the SSD stand-in), shared by all ranks."""

    def __init__(self, num_rows: int, row_bytes: int, name: str, rank: int = 0, world: int = 1,
                 shm_dir: str | None = None):
        super().__init__((num_rows, row_bytes), np.uint8, name, rank, world, shm_dir)
        self.tensor = torch.from_numpy(self.array)

    def close(self, unlink: bool = True):
        self.tensor = None
        super().close(unlink)
