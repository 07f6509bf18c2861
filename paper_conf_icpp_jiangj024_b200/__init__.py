"""B200-native sample + extract hot path of GNNDrive (Jiang, Jia, Wang, ICPP'24).

Thin Python binding over libgd.so (include/gd.h): argument marshalling only.  Every step
of the path runs in the library's sm_100a kernels; torch provides device memory, streams
and events.  Importing the package loads libgd.so and raises if it is missing.

    g = Graph(indptr, indices, device=0)
    out = g.sample(seeds, fanouts=(15, 10, 5), rng_seed=3, batch_id=b)     # gd_sample
    buf = FeatureBuffer(host_feat_u8, capacity=S, max_inflight=4, max_nodes_per_batch=out.max_nodes)
    feats, alias, done = buf.extract(out.n_id, out.num_nodes_dev, out.max_nodes)    # gd_extract
    ...                                   # consumer waits `done`, trains on feats
    buf.release(out.n_id, out.num_nodes_dev, out.max_nodes)                # gd_buffer_release
"""
from __future__ import annotations

import ctypes

import torch

from . import _lib
from ._lib import GD_MAX_HOPS, GdError, SampleOutC, check, lib

__all__ = ["Graph", "SampleOut", "Workspace", "FeatureBuffer", "GdError", "sample_bounds", "check_device_status", "lib"]


def _ptr(t):
    return ctypes.c_void_p(t.data_ptr()) if t is not None else None


def _stream_ptr(stream, device):
    s = stream if stream is not None else torch.cuda.current_stream(device)
    return ctypes.c_void_p(s.cuda_stream)


def sample_bounds(num_seeds: int, fanouts, num_nodes: int, num_edges: int):
    """gd_sample_bounds: (max_nodes[K+1], max_edges[K]) as Python lists."""
    K = len(fanouts)
    f = (ctypes.c_int32 * K)(*fanouts)
    nm = (ctypes.c_int64 * (K + 1))()
    em = (ctypes.c_int64 * K)()
    check(lib.gd_sample_bounds(num_seeds, f, K, num_nodes, num_edges, nm, em))
    return list(nm), list(em)


class SampleOut:
    """Device outputs of one gd_sample call, allocated at the worst-case bounds."""

    def __init__(self, max_nodes, max_edges, device, with_eid=False):
        K = len(max_edges)
        self.K = K
        self.max_nodes_list = list(max_nodes)
        self.max_edges_list = list(max_edges)
        self.max_nodes = int(max_nodes[-1])
        dev = torch.device("cuda", device)
        self.n_id = torch.empty(max(1, self.max_nodes), dtype=torch.int32, device=dev)
        self.rowptr = [torch.empty(max_nodes[h] + 1, dtype=torch.int64, device=dev) for h in range(K)]
        self.col = [torch.empty(max(1, max_edges[h]), dtype=torch.int32, device=dev) for h in range(K)]
        self.eid = [torch.empty(max(1, max_edges[h]), dtype=torch.int64, device=dev) for h in range(K)] if with_eid else None
        self.sizes = torch.zeros(2 * K + 1, dtype=torch.int64, device=dev)

    @property
    def num_nodes_dev(self) -> torch.Tensor:
        """Device int64 scalar n_K (a view of sizes[K]) for gd_extract / gd_buffer_release."""
        return self.sizes[self.K:self.K + 1]

    def cstruct(self) -> SampleOutC:
        c = getattr(self, "_cs", None)   # the arrays never move: build the struct once
        if c is not None:
            return c
        c = SampleOutC()
        c.n_id = self.n_id.data_ptr()
        for h in range(self.K):
            c.rowptr[h] = self.rowptr[h].data_ptr()
            c.col[h] = self.col[h].data_ptr()
            c.eid[h] = self.eid[h].data_ptr() if self.eid is not None else None
        c.sizes = self.sizes.data_ptr()
        self._cs = c
        return c

    def to_host(self):
        """Synchronising copy of the trimmed result (tests / inspection only)."""
        sizes = self.sizes.cpu()
        K = self.K
        nK = int(sizes[K])
        res = {"sizes": sizes.numpy(), "n_id": self.n_id[:nK].cpu().numpy(), "rowptr": [], "col": [], "eid": []}
        for h in range(K):
            n_prev, e_h = int(sizes[h]), int(sizes[K + 1 + h])
            res["rowptr"].append(self.rowptr[h][:n_prev + 1].cpu().numpy())
            res["col"].append(self.col[h][:e_h].cpu().numpy())
            res["eid"].append(self.eid[h][:e_h].cpu().numpy() if self.eid is not None else None)
        return res


class Graph:
    """gd_graph: an HBM replica of a CSR topology (int64 indptr, int32 indices)."""

    def __init__(self, indptr: torch.Tensor, indices: torch.Tensor, device: int = 0, validate: bool = True):
        assert indptr.dtype == torch.int64 and indices.dtype == torch.int32
        indptr = indptr.contiguous()
        indices = indices.contiguous()
        self.num_nodes = indptr.numel() - 1
        self.num_edges = indices.numel()
        self.device = device
        h = ctypes.c_void_p()
        check(lib.gd_graph_create(_ptr(indptr), _ptr(indices), self.num_nodes, self.num_edges, device,
                                  int(validate), ctypes.byref(h)))
        self._h = h

    @property
    def handle(self):
        return self._h

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            lib.gd_graph_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass

    def bounds(self, num_seeds: int, fanouts):
        return sample_bounds(num_seeds, fanouts, self.num_nodes, self.num_edges)

    def alloc_out(self, num_seeds: int, fanouts, with_eid=False) -> SampleOut:
        nm, em = self.bounds(num_seeds, fanouts)
        return SampleOut(nm, em, self.device, with_eid)

    def sample(self, seeds: torch.Tensor, fanouts, rng_seed: int, batch_id: int, out: SampleOut | None = None,
               stream=None, with_eid: bool = False, workspace: "Workspace | None" = None) -> SampleOut:
        """gd_sample (gd_sample_ws with a workspace).  `seeds` int32 on the device or in (pinned) host memory."""
        assert seeds.dtype == torch.int32 and seeds.is_contiguous()
        fanouts = list(fanouts)
        if out is None:
            out = self.alloc_out(seeds.numel(), fanouts, with_eid)
        K = len(fanouts)
        key = tuple(fanouts)
        f = self._fan_cache.get(key) if hasattr(self, "_fan_cache") else None
        if f is None:
            if not hasattr(self, "_fan_cache"):
                self._fan_cache = {}
            f = self._fan_cache[key] = (ctypes.c_int32 * K)(*fanouts)
        cs = out.cstruct()
        if workspace is None:
            check(lib.gd_sample(self._h, _ptr(seeds), seeds.numel(), f, K, ctypes.c_uint64(rng_seed),
                                ctypes.c_uint32(batch_id & 0xFFFFFFFF), ctypes.byref(cs),
                                _stream_ptr(stream, self.device)))
        else:
            check(lib.gd_sample_ws(self._h, workspace.handle, _ptr(seeds), seeds.numel(), f, K,
                                   ctypes.c_uint64(rng_seed), ctypes.c_uint32(batch_id & 0xFFFFFFFF),
                                   ctypes.byref(cs), _stream_ptr(stream, self.device)))
        return out

    def workspace(self) -> "Workspace":
        return Workspace(self)

    def check(self):
        return check_device_status(self._h)

    def sampler(self, padded: bool):
        """gd_graph_sampler: padded hops (default) or count-scan hops; identical outputs."""
        check(lib.gd_graph_sampler(self._h, int(padded)))

    def timing(self, enable: bool):
        check(lib.gd_graph_timing(self._h, int(enable)))

    def timing_read(self):
        ms = ctypes.c_double()
        n = ctypes.c_int64()
        check(lib.gd_graph_timing_read(self._h, ctypes.byref(ms), ctypes.byref(n)))
        return {"sample_ms": ms.value, "calls": n.value}


class Workspace:
    """gd_workspace: sampling scratch for one concurrently sampling stream."""

    def __init__(self, graph: Graph):
        h = ctypes.c_void_p()
        check(lib.gd_workspace_create(graph.handle, ctypes.byref(h)))
        self._h = h
        self.graph = graph      # keep the graph alive

    @property
    def handle(self):
        return self._h

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            lib.gd_workspace_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass


class FeatureBuffer:
    """gd_buffer: slot-managed HBM feature buffer over a pinned host table (the SSD stand-in)."""

    def __init__(self, host_feat: torch.Tensor, capacity: int, max_inflight: int, max_nodes_per_batch: int,
                 preload: bool = False, device: int = 0, num_nodes: int | None = None):
        """`host_feat` [P, R] uint8; node v's row is host_feat[v mod P] when num_nodes > P
        (gd_buffer_init_mod), else P = num_nodes (gd_buffer_init)."""
        assert host_feat.device.type == "cpu" and host_feat.dtype == torch.uint8 and host_feat.dim() == 2
        assert host_feat.is_contiguous()
        self.host_feat = host_feat          # keep alive until destroy
        self.table_rows, self.row_bytes = host_feat.shape
        self.num_nodes = int(num_nodes) if num_nodes is not None else self.table_rows
        self.capacity = int(capacity)
        self.max_inflight = int(max_inflight)
        self.max_nodes_per_batch = int(max_nodes_per_batch)
        self.device = device
        h = ctypes.c_void_p()
        check(lib.gd_buffer_init_mod(_ptr(host_feat), self.table_rows, self.num_nodes, self.row_bytes, self.capacity,
                                     self.max_inflight, self.max_nodes_per_batch, int(preload), device,
                                     ctypes.byref(h)))
        self._h = h
        sp = lib.gd_buffer_side_stream(h)
        self.side_stream = torch.cuda.ExternalStream(sp, device=torch.device("cuda", device))

    @property
    def handle(self):
        return self._h

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            lib.gd_buffer_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass

    def alloc_out(self, n_max: int) -> torch.Tensor:
        return torch.empty((max(1, n_max), self.row_bytes), dtype=torch.uint8, device=torch.device("cuda", self.device))

    def extract(self, node_ids: torch.Tensor, n_dev: torch.Tensor, n_max: int, out: torch.Tensor | None = None,
                alias: torch.Tensor | None = None, stats: torch.Tensor | None = None, stream=None,
                done: torch.cuda.Event | None = None):
        """gd_extract.  Returns (out, alias, done); `out` is valid after `done`."""
        if out is None:
            out = self.alloc_out(n_max)
        if done is None:
            done = torch.cuda.Event()
        if done.cuda_event == 0:        # torch creates events lazily on first record
            done.record(torch.cuda.current_stream(self.device))
        check(lib.gd_extract(self._h, _ptr(node_ids), _ptr(n_dev), int(n_max), _ptr(out), _ptr(alias), _ptr(stats),
                             _stream_ptr(stream, self.device), ctypes.c_void_p(done.cuda_event)))
        return out, alias, done

    def release(self, node_ids: torch.Tensor, n_dev: torch.Tensor, n_max: int, stream=None):
        check(lib.gd_buffer_release(self._h, _ptr(node_ids), _ptr(n_dev), int(n_max), _stream_ptr(stream, self.device)))

    def snapshot(self):
        import numpy as np
        N, S = self.num_nodes, self.capacity
        ms = np.zeros(N, dtype=np.int32)
        mr = np.zeros(N, dtype=np.int32)
        mv = np.zeros(N, dtype=np.uint8)
        rv = np.zeros(S, dtype=np.int32)
        sb = np.zeros(S, dtype=np.int32)
        k = ctypes.c_int64()
        p = lambda a: a.ctypes.data_as(ctypes.c_void_p)  # noqa: E731
        check(lib.gd_buffer_snapshot(self._h, p(ms), p(mr), p(mv), p(rv), p(sb), ctypes.byref(k)))
        return {"slot": ms, "rc": mr, "valid": mv, "reverse": rv, "standby": sb[:k.value].copy()}

    def set_state(self, slot, rc, valid, reverse, standby):
        import numpy as np
        a = [np.ascontiguousarray(x, dtype=t) for x, t in
             ((slot, np.int32), (rc, np.int32), (valid, np.uint8), (reverse, np.int32), (standby, np.int32))]
        p = lambda x: x.ctypes.data_as(ctypes.c_void_p)  # noqa: E731
        check(lib.gd_buffer_set_state(self._h, p(a[0]), p(a[1]), p(a[2]), p(a[3]), p(a[4]), len(a[4])))

    def check(self):
        return check_device_status(self._h)

    def timing(self, enable: bool):
        check(lib.gd_buffer_timing(self._h, int(enable)))

    def timing_read(self):
        ms = (ctypes.c_double * 7)()
        n = ctypes.c_int64()
        check(lib.gd_buffer_timing_read(self._h, ms, ctypes.byref(n)))
        return {"bookkeeping_ms": ms[0], "gather_ms": ms[1], "miss_zero_copy_ms": ms[2], "miss_staged_ms": ms[3],
                "host_gather_ms": ms[4], "zero_copy_share": ms[5], "staged_copy_ms": ms[6], "batches": n.value}

    # ---- f2: NVLink peer feature buffers
    PEER_BLOB_BYTES = 256

    def peer_attach(self, peers):
        """gd_buffer_peer_attach: in-process peer buffers ([] detaches)."""
        arr = (ctypes.c_void_p * max(1, len(peers)))(*[p._h.value for p in peers])
        check(lib.gd_buffer_peer_attach(self._h, len(peers), arr))
        self._peers = list(peers)      # keep them alive while attached

    def peer_export_ipc(self) -> bytes:
        """gd_buffer_peer_export_ipc: this buffer's descriptor for other processes."""
        blob = ctypes.create_string_buffer(self.PEER_BLOB_BYTES)
        check(lib.gd_buffer_peer_export_ipc(self._h, blob, self.PEER_BLOB_BYTES))
        return blob.raw

    def peer_attach_ipc(self, blobs):
        """gd_buffer_peer_attach_ipc: attach other processes' buffers (their export blobs)."""
        data = b"".join(blobs)
        buf = ctypes.create_string_buffer(data, max(1, len(data)))
        check(lib.gd_buffer_peer_attach_ipc(self._h, len(blobs), buf))

    def peer_stats(self):
        """gd_buffer_peer_stats: (rows served by peers, misses probed) since init."""
        s, p = ctypes.c_int64(), ctypes.c_int64()
        check(lib.gd_buffer_peer_stats(self._h, ctypes.byref(s), ctypes.byref(p)))
        return s.value, p.value

    def stage_mode(self, copy_engine: bool):
        """gd_buffer_stage_mode: phase 2 of the staged share by copy engine (True) or SM pull."""
        check(lib.gd_buffer_stage_mode(self._h, int(bool(copy_engine))))

    def policy_read(self):
        """gd_buffer_policy_read: the miss-path split policy's current inputs and decision."""
        v = (ctypes.c_double * 12)()
        check(lib.gd_buffer_policy_read(self._h, v, 12))
        return {"zero_copy_share": v[0], "r_host_GBps": v[1], "r_zc_GBps": v[2], "r_link_GBps": v[3],
                "misses_est": v[4], "rate_samples": int(v[5]), "model_share_cap": v[6], "rated_batch": int(v[7]),
                "tuner_on": bool(v[8]), "tuner_windows": int(v[9]), "tuner_frozen": bool(v[10]),
                "tuner_best_ns_per_miss": v[11]}

    def config(self, host_threads: int, zero_copy_share: float = -1.0, zc_blocks: int = 0, pull_blocks: int = 0):
        """gd_buffer_config: staged miss path width, zero-copy share (< 0: adaptive), copy grids."""
        check(lib.gd_buffer_config(self._h, int(host_threads), float(zero_copy_share), int(zc_blocks),
                                   int(pull_blocks)))


def check_device_status(handle) -> int:
    """gd_check_device_status: raises GdError if a device-side check tripped."""
    bits = ctypes.c_uint32()
    check(lib.gd_check_device_status(handle, ctypes.byref(bits)))
    return bits.value
