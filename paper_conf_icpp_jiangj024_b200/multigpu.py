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

import torch
import torch.distributed as dist


# The shared host table, the segment schedule and the NUMA placement live in the neutral
# synth.host module (no libgd), so that bench.py's oracle reference arm uses them without
# loading this package; re-exported here as part of the data-parallel API.
from synth import segment  # noqa: E402,F401
from synth.host import (HostTable, SharedArray, batch_schedule, bind_to_gpu_socket,  # noqa: E402,F401
                        numa_nodes, set_interleave)


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
