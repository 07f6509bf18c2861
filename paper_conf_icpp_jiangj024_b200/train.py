"""f4: the train stage (GraphSAGE on the sampled blocks), a thin binding of gd_sage_* (include/gd.h).

Argument marshalling only: every step of forward, loss, backward and SGD runs in libgd.so.
Data parallelism follows the paper's subprocess-per-GPU model: each rank trains on
its own batches and the flat gradient buffer is summed across ranks (NCCL all-reduce)
before the SGD step with grad_scale = 1 / world.
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch

from ._lib import check, lib

GD_SAGE_W, GD_SAGE_B, GD_SAGE_DW, GD_SAGE_DB, GD_SAGE_A16, GD_SAGE_Z, GD_SAGE_H = range(7)


def _stream_ptr(stream, device):
    s = stream if stream is not None else torch.cuda.current_stream(device)
    return ctypes.c_void_p(s.cuda_stream)


class SageModel:
    """gd_sage: L-layer GraphSAGE (mean aggregator, root weight), widths dims[0..L]."""

    def __init__(self, dims, init_params, max_nodes, device: int = 0):
        self.dims = [int(d) for d in dims]
        self.L = len(self.dims) - 1
        self.device = device
        assert len(init_params) == self.L and len(max_nodes) == self.L + 1
        self._init = [(np.ascontiguousarray(W, dtype=np.float32), np.ascontiguousarray(b, dtype=np.float32))
                      for W, b in init_params]
        for j, (W, b) in enumerate(self._init):
            assert W.shape == (2 * self.dims[j], self.dims[j + 1]) and b.shape == (self.dims[j + 1],)
        d = (ctypes.c_int32 * (self.L + 1))(*self.dims)
        ws = (ctypes.c_void_p * self.L)(*[W.ctypes.data for W, _ in self._init])
        bs = (ctypes.c_void_p * self.L)(*[b.ctypes.data for _, b in self._init])
        mn = (ctypes.c_int64 * (self.L + 1))(*[int(x) for x in max_nodes])
        h = ctypes.c_void_p()
        check(lib.gd_sage_create(self.L, d, ws, bs, mn, device, ctypes.byref(h)))
        self._h = h
        g = ctypes.c_void_p()
        n = ctypes.c_int64()
        check(lib.gd_sage_grads(h, ctypes.byref(g), ctypes.byref(n)))
        self.num_params = n.value
        # zero-copy torch view of the flat gradient buffer (for the all-reduce)
        self.grad_flat = _device_view(g.value, n.value, device)
        self.loss = torch.zeros(1, dtype=torch.float32, device=torch.device("cuda", device))

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            lib.gd_sage_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass

    def step(self, sample_out, feats: torch.Tensor, labels: torch.Tensor, stream=None) -> torch.Tensor:
        """gd_sage_step on one batch: `sample_out` a SampleOut, `feats` the extracted rows
        (fp32 [>= n_L, dims[0]] or the uint8 [>= n_L, 4 dims[0]] out buffer), `labels`
        int32 [>= n_0] on the device.  Returns the device loss scalar (valid in stream order)."""
        K = sample_out.K
        assert K == self.L
        rp = (ctypes.c_void_p * K)(*[sample_out.rowptr[h].data_ptr() for h in range(K)])
        cl = (ctypes.c_void_p * K)(*[sample_out.col[h].data_ptr() for h in range(K)])
        assert feats.is_cuda and labels.is_cuda and labels.dtype == torch.int32
        check(lib.gd_sage_step(self._h, rp, cl, ctypes.c_void_p(sample_out.sizes.data_ptr()),
                               ctypes.c_void_p(feats.data_ptr()), ctypes.c_void_p(labels.data_ptr()),
                               ctypes.c_void_p(self.loss.data_ptr()), _stream_ptr(stream, self.device)))
        return self.loss

    def apply_sgd(self, lr: float, grad_scale: float = 1.0, stream=None):
        check(lib.gd_sage_apply_sgd(self._h, float(lr), float(grad_scale), _stream_ptr(stream, self.device)))

    def allreduce_grads(self, group=None) -> float:
        """Sum the flat gradients over the process group (NCCL on GPUs); returns the
        grad_scale (1 / world) for apply_sgd."""
        return allreduce_flat(self.grad_flat, group)

    def get(self, what: int, layer: int) -> np.ndarray:
        di, do = self.dims[layer], self.dims[layer + 1]
        shapes = {GD_SAGE_W: ((2 * di, do), np.float32), GD_SAGE_B: ((do,), np.float32),
                  GD_SAGE_DW: ((2 * di, do), np.float32), GD_SAGE_DB: ((do,), np.float32)}
        if what in shapes:
            shp, dt = shapes[what]
            a = np.zeros(shp, dtype=dt)
        else:
            raise ValueError("use get_activation for A16 / Z")
        check(lib.gd_sage_get(self._h, what, layer, a.ctypes.data_as(ctypes.c_void_p), a.nbytes))
        return a

    def get_activation(self, what: int, layer: int, n_dst_max: int) -> np.ndarray:
        di, do = self.dims[layer], self.dims[layer + 1]
        if what in (GD_SAGE_A16, GD_SAGE_H):     # bf16 -> float32 (bf16 is the top half of an fp32)
            raw = np.zeros((n_dst_max, 2 * di if what == GD_SAGE_A16 else do), dtype=np.uint16)
            check(lib.gd_sage_get(self._h, what, layer, raw.ctypes.data_as(ctypes.c_void_p), raw.nbytes))
            return (raw.astype(np.uint32) << 16).view(np.float32)
        a = np.zeros((n_dst_max, do), dtype=np.float32)
        check(lib.gd_sage_get(self._h, what, layer, a.ctypes.data_as(ctypes.c_void_p), a.nbytes))
        return a


def allreduce_flat(flat: torch.Tensor, group=None) -> float:
    """DDP's gradient step: SUM-all-reduce one flat gradient tensor in place and
    return the scale (1 / world) that turns the sum into the mean."""
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()):
        return 1.0
    dist.all_reduce(flat, group=group)
    return 1.0 / dist.get_world_size(group)


def flatten_params(pairs) -> np.ndarray:
    """[(W_0, b_0), (W_1, b_1), ...] in the flat layout of gd_sage's parameter / gradient
    buffers ([W_0 b_0 W_1 b_1 ...], row-major W)."""
    return np.concatenate([np.concatenate([np.ravel(W), np.ravel(b)]) for W, b in pairs])


def _device_view(ptr: int, n: int, device: int) -> torch.Tensor:
    """A float32 torch tensor over device memory owned by libgd (no copy)."""
    class _CAI:
        __cuda_array_interface__ = {"shape": (n,), "typestr": "<f4", "data": (ptr, False), "version": 3,
                                    "strides": None, "stream": None}
    with torch.cuda.device(device):
        return torch.as_tensor(_CAI(), device=torch.device("cuda", device))
