"""Data-parallel host logic for the sample + extract path.

GNNDrive "divides the entire training set into segments for subprocesses to execute"
(P:140); "topological data and staging buffer are shared among subprocesses. A subprocess
has its own feature buffer".  On B200: one process per GPU, each with a private
HBM topology replica and feature buffer; one host feature table (the SSD stand-in) is
shared by all processes through a /dev/shm file that each process registers with CUDA.
There is NO collective on the data path: mini-batches are independent.  torch.distributed
is used only for start-up barriers and the off-path max-over-ranks of the timings.
"""
from __future__ import annotations

import ctypes
import mmap
import os
import platform

import numpy as np
import torch
import torch.distributed as dist


def segment(num_batches: int, rank: int, world: int) -> range:
    """Contiguous segment [rank*nb/world, (rank+1)*nb/world) of the global batch list."""
    lo = num_batches * rank // world
    hi = num_batches * (rank + 1) // world
    return range(lo, hi)


def batch_schedule(num_batches: int, rank: int, world: int, steps: int):
    """(global batch index, epoch) for this rank's first `steps` steps; wraps around the
    segment, one epoch per wrap.  The Philox batch key is epoch * num_batches + b, so
    every (epoch, batch) pair draws an independent sample regardless of the GPU count."""
    seg = segment(num_batches, rank, world)
    if len(seg) == 0:
        return []
    return [(seg[j % len(seg)], j // len(seg)) for j in range(steps)]


def barrier():
    if dist.is_available() and dist.is_initialized():
        dist.barrier()


def max_over_ranks(x: float, device=None) -> float:
    """Max of a per-rank scalar (timings are reported as the slowest rank)."""
    if not (dist.is_available() and dist.is_initialized()):
        return float(x)
    if dist.get_backend() == "gloo":
        device = None
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(x: float, device=None) -> float:
    if not (dist.is_available() and dist.is_initialized()):
        return float(x)
    if dist.get_backend() == "gloo":
        device = None
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


def _parse_list(text: str):
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
            return _parse_list(f.read())
    except OSError:
        return []


def set_interleave(enable: bool) -> bool:
    """Interleave this thread's future page allocations over all online NUMA nodes
    (set_mempolicy(MPOL_INTERLEAVE)), or restore the default policy.  Used while rank 0
    faults the shared host table in, so that on a multi-socket box the random row reads of
    all GPUs' miss streams spread over every socket's memory controllers.
    Returns False (and changes nothing) on a single-node host or where the syscall is
    unavailable."""
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


class HostTable:
    """A [N, R] uint8 host table.  world == 1: private anonymous memory.  world > 1: one
    /dev/shm file created by rank 0 and mapped by every rank (P:142 shared host data)."""

    def __init__(self, num_rows: int, row_bytes: int, name: str, rank: int = 0, world: int = 1,
                 shm_dir: str = "/dev/shm"):
        self.shape = (int(num_rows), int(row_bytes))
        nbytes = self.shape[0] * self.shape[1]
        self.path = None
        if world == 1:
            self.array = np.empty(self.shape, dtype=np.uint8)
            self._mm = None
        else:
            self.path = os.path.join(shm_dir, f"gd_{name}_{num_rows}x{row_bytes}")
            if rank == 0:
                with open(self.path, "wb") as f:
                    f.truncate(nbytes)
            barrier()
            fd = os.open(self.path, os.O_RDWR)
            try:
                self._mm = mmap.mmap(fd, nbytes, mmap.MAP_SHARED, mmap.PROT_READ | mmap.PROT_WRITE)
            finally:
                os.close(fd)
            self.array = np.frombuffer(self._mm, dtype=np.uint8).reshape(self.shape)
        self.tensor = torch.from_numpy(self.array)
        self.owner = rank == 0

    def close(self, unlink: bool = True):
        self.tensor = None
        self.array = None
        if self._mm is not None:
            try:
                self._mm.close()
            except BufferError:
                pass
            self._mm = None
        if unlink and self.owner and self.path and os.path.exists(self.path):
            os.unlink(self.path)
