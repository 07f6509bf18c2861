#!/usr/bin/env python
"""Benchmark of the GNNDrive sample + extract hot path on B200 (BASELINE.json metric:
sampled+extracted mini-batches/s; gather GB/s vs HBM, misses vs the host link).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config papers100m]
    python -m torch.distributed.run --nnodes=1 --nproc-per-node N --master-addr 127.0.0.1 \\
        --master-port P bench.py --gpus N ...
    python bench.py --impl reference ...      # the CPU oracle as the reference arm

One step = one mini-batch through every §8(a) row: gd_sample (seed intake, counts,
Floyd/Philox sampling, relabel) -> gd_extract (lookup, LRU alloc/evict, hit gather, miss
stream from the pinned host table) -> gd_buffer_release of the batch Q=4 steps earlier
(P:177 training-queue depth).  Inputs are synthetic (synth/), shaped like the paper's
workloads; the default workload is the Papers100M-shaped config (BASELINE.json configs[2]).
Rank 0 prints ONE JSON line.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from synth.host import HostTable, SharedArray, batch_schedule, bind_to_gpu_socket, set_interleave  # noqa: E402

Q = 4   # release lag = training-queue capacity


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=200)
    p.add_argument("--warmup", type=int, default=16)
    p.add_argument("--config", default="papers100m", choices=sorted(synth.CONFIGS))
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--batch-size", type=int, default=None, help="f3 sweep override (Fig. 10)")
    p.add_argument("--feat-dim", type=int, default=None, help="f3 sweep override (Fig. 8)")
    p.add_argument("--buffer-frac", type=float, default=None, help="f3 sweep override (Fig. 12)")
    p.add_argument("--table-rows", type=int, default=None,
                   help="bounded physical host table (node v -> row v mod P, reading R15), e.g. for the dim-512 sweep point "
                        "whose full table exceeds host RAM")
    p.add_argument("--cpu-seconds", type=float, default=12.0, help="budget of the oracle cpu_baseline sample")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--train", action="store_true", help="f4: add the train stage (3-layer GraphSAGE, hidden 256, "
                   "P:173) to every step on its own stream; the host table holds numeric fp32 features")
    p.add_argument("--lr", type=float, default=0.01, help="f4 SGD learning rate")
    p.add_argument("--peer", action="store_true", help="f2: attach every other rank's feature buffer as an NVLink "
                   "peer (CUDA IPC); misses are served from peers' HBM before the host link")
    p.add_argument("--sample-ahead", type=int, default=None,
                   help="batches sampled ahead of extraction (per-batch buffer ring = Q + 1 + this); default: 3 "
                        "when every feature is resident (sampling bounds the step), 0 with a miss path (the host "
                        "link bounds it; sampling further ahead only adds contention for the hit gather)")
    p.add_argument("--samplers", type=int, default=2,
                   help="sampler streams (P:94 'a pool of threads as samplers'), each with its own gd_workspace: "
                        "batch j is sampled on stream j mod S, so the next batch's sampling overlaps this batch's "
                        "(extraction stays in batch order on the caller's stream)")
    p.add_argument("--no-peer-leg", action="store_true",
                   help="N > 1: skip the extra f2 leg (every rank's buffer attached as NVLink peers, W + K more "
                        "timed steps) that runs after the main measurement")
    p.add_argument("--parity-batches", type=int, default=None,
                   help="first batches of each rank checked in full (sample outputs, alias, hits/misses, rows) vs the "
                        "oracle; default 8 (papers100m/friendster/mag240m; 4 per rank at >= 8 ranks), 16 (products), "
                        "all of the rank's segment (tiny)")
    p.add_argument("--no-replay", action="store_true",
                   help="skip the steady-state parity: the oracle's Alg. 1 replayed over the rank's whole schedule")
    p.add_argument("--prewarm-max", type=int, default=1000,
                   help="untimed buffer pre-warm: batches until cumulative misses >= S (SURVEY 8(d)), at most this")
    p.add_argument("--out", default=None, help="also write the JSON line to this file")
    p.add_argument("--timeline", default=None, help="after the measurement, 16 more steps under torch.profiler "
                   "(CUPTI): per-activity busy time and the overlap of the miss stream with sampling -> this .md "
                   "(tools/timeline.py)")
    p.add_argument("--window", type=int, default=0, help="also report batches/s per window of this many timed steps "
                   "(device events on the caller's stream; sustained-rate evidence)")
    p.add_argument("--pipeline-sweep", default="", help="f1: 'samplers:reorder,...' SET pipeline runs "
                   "(concurrent sampler streams, out-of-order extraction), results under 'pipeline'")
    p.add_argument("--miss-sweep", default="", help="tuning: 'threads:share:zc_blocks:pull_blocks,...' timed "
                   "one after another in this process (results under 'sweep')")
    return p.parse_args()


# ----------------------------------------------------------------------------- helpers
# (torch.distributed directly: the reference arm must not load the product package / libgd.so)

def _dist_on():
    import torch.distributed as dist
    return dist.is_available() and dist.is_initialized()


def barrier():
    if _dist_on():
        import torch.distributed as dist
        dist.barrier()


def _reduce(x: float, op, device=None) -> float:
    if not _dist_on():
        return float(x)
    import torch.distributed as dist
    t = torch.tensor([float(x)], dtype=torch.float64, device=None if dist.get_backend() == "gloo" else device)
    dist.all_reduce(t, op=op)
    return float(t.item())


def max_over_ranks(x: float, device=None) -> float:
    import torch.distributed as dist
    return _reduce(x, dist.ReduceOp.MAX, device)


def sum_over_ranks(x: float, device=None) -> float:
    import torch.distributed as dist
    return _reduce(x, dist.ReduceOp.SUM, device)


def gather_objects(obj, world):
    """Every rank's `obj` (a list indexed by rank) on every rank."""
    if world == 1 or not _dist_on():
        return [obj]
    import torch.distributed as dist
    out = [None] * world
    dist.all_gather_object(out, obj)
    return out


def default_parity_batches(cfg, world, seg_len):
    """SURVEY 8(d) parity plan: all batches (tiny), the first 16 (products), the first 8 per GPU
    (papers100m / friendster / mag240m; 4 per GPU at 8 GPUs)."""
    if cfg.name == "tiny":
        return seg_len
    if cfg.name == "products":
        return 16
    return 4 if world >= 8 else 8


def loaded_native_libs():
    """Shared objects of this repo mapped into this process (reference-arm hygiene)."""
    libs = set()
    try:
        with open("/proc/self/maps") as f:
            for line in f:
                path = line.split()[-1] if line.strip() else ""
                if path.startswith(ROOT) and ".so" in path:
                    libs.add(os.path.relpath(path, ROOT))
    except OSError:
        pass
    return sorted(libs)


def log(*a):
    if int(os.environ.get("RANK", "0")) == 0:
        print("[bench]", *a, file=sys.stderr, flush=True)


class ClockSampler:
    """SM clocks and throttle reasons sampled every 200 ms during the timed region, in-process
    through NVML (spawning nvidia-smi would steal a host core from the miss-path gather).
    NVML is initialised (and queried once) when the sampler is constructed, before the timed
    region: nvmlInit inside the region stalled the copy-engine miss path for ~100 ms in some
    runs (20-step papers100m: 149 batches/s vs 444-485), visible only in short regions."""

    BITS = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40, "sw_power_cap": 0x4}

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.rows = []
        self._stop = threading.Event()
        self._t = None
        self._N = self._h = None
        try:
            import pynvml as N
            N.nvmlInit()
            self._N, self._h = N, N.nvmlDeviceGetHandleByIndex(gpu_index)
            self._query()
            self.rows.clear()
        except Exception:  # noqa: BLE001
            self._N = None

    def _query(self):
        N, h = self._N, self._h
        sm = N.nvmlDeviceGetClockInfo(h, N.NVML_CLOCK_SM)
        mx = N.nvmlDeviceGetMaxClockInfo(h, N.NVML_CLOCK_SM)
        r = N.nvmlDeviceGetCurrentClocksEventReasons(h) if hasattr(N, "nvmlDeviceGetCurrentClocksEventReasons") \
            else N.nvmlDeviceGetCurrentClocksThrottleReasons(h)
        self.rows.append((sm, mx, [k for k, b in self.BITS.items() if r & b]))

    def _run(self):
        if self._N is None:
            return
        period = float(os.environ.get("GD_CLOCK_PERIOD_S", "0.2"))
        while not self._stop.is_set():
            try:
                self._query()
            except Exception:  # noqa: BLE001
                pass
            if period <= 0:
                break
            self._stop.wait(period)

    def __enter__(self):
        self._stop.clear()
        self.rows = []
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join(timeout=10)

    def summary(self):
        sm = [r[0] for r in self.rows]
        mx = [r[1] for r in self.rows]
        reasons = sorted({x for r in self.rows for x in r[2]})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows), "source": "NVML, 200 ms"}


def h2d_peak_gbps(device, sync=None, reps: int = 10) -> float:
    """Host-link roofline measured in-run: pinned 1 GiB cudaMemcpyAsync H2D, best of `reps`.
    sync: called before every repetition (a barrier, so that all ranks copy at once)."""
    n = 1 << 30
    h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    h.fill_(1)
    d = torch.empty(n, dtype=torch.uint8, device=device)
    s = torch.cuda.Stream(device)
    best = 0.0
    with torch.cuda.stream(s):
        for _ in range(reps):
            if sync is not None:
                sync()
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record(s)
            d.copy_(h, non_blocking=True)
            b.record(s)
            b.synchronize()
            best = max(best, n / (a.elapsed_time(b) * 1e6))
    del h, d
    return best


def h2d_peaks(device, rank, world):
    """the host-link denominators at G GPUs.  `alone`: this rank's link with the
    other ranks idle (ranks take turns between barriers); `concurrent`: every rank copies at
    the same time (a barrier before each of the 10 repetitions), the per-GPU share of the
    links the G GPUs contend for (PCIe switch uplinks, host DRAM)."""
    if world == 1:
        v = h2d_peak_gbps(device)
        return {"alone": v, "concurrent": v}
    alone = 0.0
    for r in range(world):
        barrier()
        if r == rank:
            alone = h2d_peak_gbps(device)
        barrier()
    conc = h2d_peak_gbps(device, sync=barrier)
    return {"alone": alone, "concurrent": conc}


def anon_huge_gb():
    """AnonHugePages of /proc/meminfo in GB (transparent huge pages in use), or None."""
    try:
        for line in open("/proc/meminfo"):
            if line.startswith("AnonHugePages:"):
                return round(int(line.split()[1]) / 1e6, 2)
    except OSError:
        pass
    return None


def measured_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:  # noqa: BLE001
        return {}


NUM_CLASSES = {"papers100m": 172, "products": 47, "friendster": 64, "tiny": 16, "mag240m": 153}


def capacity_for(cfg, n_max: int) -> int:
    if cfg.preload:
        return cfg.num_nodes
    if cfg.buffer_frac < 0:                           # "miss heavy": the minimum legal size
        return min(cfg.num_nodes, Q * n_max)
    return max(int(cfg.buffer_frac * cfg.num_nodes), min(cfg.num_nodes, Q * n_max))


def train_batches(cfg, device):
    train = synth.train_nodes(cfg.num_nodes, cfg.train_frac, device=device)
    nb = max(1, len(train) // cfg.batch_size)
    return train, nb


class Workload:
    """Graph, host table, seeds of one config on this rank (setup, not timed)."""

    def __init__(self, cfg, rank, world, device, need_host_csr):
        self.cfg = cfg
        t0 = time.time()
        indptr, indices = synth.chung_lu_csr(cfg.num_nodes, cfg.num_edges, device=device)
        if device.type == "cuda":
            torch.cuda.synchronize(device)
        self.t_graph = time.time() - t0
        deg = (indptr[1:] - indptr[:-1])
        self.deg_stats = {"max": int(deg.max()), "mean": float(cfg.num_edges / cfg.num_nodes),
                          "p99": int(torch.quantile(deg[:: max(1, cfg.num_nodes // 1_000_000)].double(), 0.99))}
        del deg
        # host CSR for the oracle (parity, replay, cpu baseline): private at world 1, one shared
        # copy at world > 1 (rank 0 writes it; "topological data ... shared")
        self._csr_shm = []
        if need_host_csr and world == 1:
            self.host_indptr, self.host_indices = indptr.cpu().numpy(), indices.cpu().numpy()
        elif need_host_csr:
            a = SharedArray((cfg.num_nodes + 1,), np.int64, f"{cfg.name}_indptr", rank, world)
            b = SharedArray((cfg.num_edges,), np.int32, f"{cfg.name}_indices", rank, world)
            if rank == 0:
                a.array[:] = indptr.cpu().numpy()
                step = 1 << 28
                for s0 in range(0, cfg.num_edges, step):
                    b.array[s0:s0 + step] = indices[s0:s0 + step].cpu().numpy()
            barrier()
            self._csr_shm = [a, b]
            self.host_indptr, self.host_indices = a.array, b.array
        else:
            self.host_indptr = self.host_indices = None
        self.indptr, self.indices = indptr, indices
        t0 = time.time()
        if world == 1 and os.environ.get("GD_COMPACT_MEMORY", "1") == "1":
            # the table asks for transparent huge pages: compact host memory first so the fill's
            # page faults find free 2 MB pages (a reused box's memory may be fragmented)
            try:
                with open("/proc/sys/vm/compact_memory", "w") as f:
                    f.write("1")
            except OSError:
                pass
        self.thp_before = anon_huge_gb()
        self.table = HostTable(cfg.host_rows, cfg.row_bytes, cfg.name, rank, world)
        # page-lock + map once here, so FeatureBuffer re-inits (parity / preload) skip it.
        # Multi-rank: rank 0 registers (faulting the shared pages in) and fills first; the
        # others register afterwards, one at a time (concurrent first-touch pinning of the
        # same tmpfs pages by several processes fails).
        self.rank, self.world, self.device = rank, world, device
        self._barrier = barrier if world > 1 else (lambda: None)   # world 1: also under torchrun (reference arm)
        self.registered = False
        if rank == 0 and device.type == "cuda":
            self.interleaved = world > 1 and set_interleave(True)   # the pages fault in here
            try:
                self._register()
            finally:
                if self.interleaved:
                    set_interleave(False)
        self.t_table_alloc = time.time() - t0
        train, nb = train_batches(cfg, device)
        self.train, self.num_batches = train, nb
        self._orders = {}

    def _register(self):
        n = self.cfg.host_rows * self.cfg.row_bytes
        rc = torch.cuda.cudart().cudaHostRegister(self.table.tensor.data_ptr(), n, 3)
        if int(rc) != 0:
            raise RuntimeError(f"cudaHostRegister(host table, {n} bytes) failed: code {int(rc)}")
        self.registered = True

    def fill_table(self, numeric: bool = False):
        """Rank 0 writes the feature rows (generated on the GPU) into the host table; then
        the other ranks register the (now resident) shared pages one after another.
        numeric: finite fp32 features for the train stage (f4) instead of random bits."""
        t0 = time.time()
        if self.table.owner:
            cfg = self.cfg
            chunk = max(1, (256 << 20) // cfg.row_bytes)
            for s in range(0, cfg.host_rows, chunk):
                e = min(cfg.host_rows, s + chunk)
                rows = (synth.numeric_feature_rows(s, e, cfg.feat_dim, device=self.device).view(torch.uint8) if numeric
                        else synth.feature_rows(s, e, cfg.row_bytes, device=self.device))
                self.table.tensor[s:e].copy_(rows)
        if self.device.type == "cuda":
            torch.cuda.synchronize(self.device)
        self.thp_table_gb = (round(anon_huge_gb() - self.thp_before, 2)
                             if self.thp_before is not None and anon_huge_gb() is not None else None)
        self._barrier()
        for r in range(1, self.world):
            if self.rank == r:
                self._register()
            self._barrier()
        self.t_fill = time.time() - t0

    def close(self):
        if self.registered:
            torch.cuda.cudart().cudaHostUnregister(self.table.tensor.data_ptr())
        self.table.close()
        self.host_indptr = self.host_indices = None
        for a in self._csr_shm:
            a.close()

    def seeds(self, b, epoch):
        if epoch not in self._orders:
            self._orders[epoch] = synth.epoch_order(self.train, epoch)
        o = self._orders[epoch]
        B = self.cfg.batch_size
        return o[b * B:(b + 1) * B]


# ----------------------------------------------------------------------------- our arm

def config_from_args(args):
    import dataclasses
    cfg = synth.CONFIGS[args.config]
    over = {}
    if args.batch_size:
        over["batch_size"] = args.batch_size
    if args.feat_dim:
        over["feat_dim"] = args.feat_dim
    if args.buffer_frac is not None:
        over["buffer_frac"] = args.buffer_frac
        over["preload"] = False
    if args.table_rows:
        over["table_rows"] = min(args.table_rows, cfg.num_nodes)
    return dataclasses.replace(cfg, **over) if over else cfg


def run_ours(args, rank, world, local_rank):
    import paper_conf_icpp_jiangj024_b200 as gd

    cfg = config_from_args(args)
    dev = torch.device("cuda", local_rank)
    torch.cuda.set_device(dev)
    # NUMA: each rank (and the host-gather pool / CUDA callback threads it creates later) on the
    # CPUs of its GPU's socket, so its pinned staging is first-touched there; at N = 1
    # only with GD_NUMA_BIND=1 (one rank may use every core)
    if os.environ.get("GD_NUMA_BIND", "1" if world > 1 else "0") == "1":
        numa = bind_to_gpu_socket(local_rank)
    else:
        numa = {"bound": False, "cpus": len(os.sched_getaffinity(0))}
    want_cpu = (not args.no_cpu_baseline) and rank == 0 and world == 1 and not args.train
    want_replay = not args.no_replay
    need_host_csr = want_cpu or want_replay or args.parity_batches != 0
    W, K = args.warmup, args.steps
    t_setup = time.time()
    wl = Workload(cfg, rank, world, dev, need_host_csr)
    g = gd.Graph(wl.indptr, wl.indices, device=local_rank, validate=False)
    del wl.indptr, wl.indices
    torch.cuda.empty_cache()
    fan = list(cfg.fanouts)
    nm, em = g.bounds(cfg.batch_size, fan)
    n_max = nm[-1]
    S = capacity_for(cfg, n_max)
    if args.train:
        assert cfg.elem_bytes == 4, "--train needs fp32 features (papers100m, products, friendster, tiny)"
    wl.fill_table(numeric=args.train)
    t0 = time.time()
    buf = gd.FeatureBuffer(wl.table.tensor, S, Q, n_max, preload=cfg.preload, device=local_rank,
                           num_nodes=cfg.num_nodes)
    t_register = time.time() - t0
    # host-gather threads: the cores this rank may use, shared with the other ranks on them (after
    # a NUMA bind the mask is the socket's, shared by world / sockets ranks), minus ~3 for the
    # driver, CUDA callback and clock threads
    sharing = max(1, world // max(1, numa.get("numa_nodes", 1))) if numa.get("bound") else world
    host_threads = max(1, min(13, len(os.sched_getaffinity(0)) // sharing - 3))
    if "GD_HOST_THREADS" not in os.environ and not cfg.preload:
        buf.config(host_threads)
    log(f"setup: graph {wl.t_graph:.1f}s table alloc {wl.t_table_alloc:.1f}s register {t_register:.1f}s "
        f"fill {wl.t_fill:.1f}s; N={cfg.num_nodes} E={cfg.num_edges} S={S} n_max={n_max} deg={wl.deg_stats}")

    sweep_cfgs = [tuple(float(x) for x in c.split(":")) for c in args.miss_sweep.split(",") if c]
    PRE = 0 if cfg.preload else args.prewarm_max
    n_pipe = len([x for x in args.pipeline_sweep.split(",") if x])
    leg = world > 1 and not args.peer and not args.no_peer_leg and not cfg.preload
    TL = 16 if args.timeline else 0
    KI = 0 if os.environ.get("GD_KERNEL_TIMING", "0") == "1" else K      # instrumented region
    total = PRE + W + K + (0 if args.no_e2e else W + K) + (len(sweep_cfgs) + n_pipe + int(leg)) * (W + K) + TL + KI
    sched = batch_schedule(wl.num_batches, rank, world, total)
    seeds_dev = torch.stack([wl.seeds(b, ep) for b, ep in sched]).to(dev).contiguous()   # HBM-resident inputs
    seeds_host = seeds_dev.cpu().pin_memory()
    batch_ids = [ep * wl.num_batches + b for b, ep in sched]

    # per-batch buffers in flight: Q unreleased batches + the one being extracted + `--sample-ahead`
    # batches sampled ahead of extraction (the sampler -> extractor queue: sampling of batch j
    # waits for the release of batch j - RING, issued after extract(j - RING + Q); with RING = Q + 1
    # that chained every sampling to the previous batch's bookkeeping)
    RING = Q + 1 + sample_ahead(args, cfg)
    outs = [g.alloc_out(cfg.batch_size, fan) for _ in range(RING)]
    feats = [buf.alloc_out(n_max) for _ in range(RING)]
    aliases = [torch.empty(n_max, dtype=torch.int32, device=dev) for _ in range(RING)]
    dones = [torch.cuda.Event() for _ in range(RING)]
    for e in dones:
        e.record(torch.cuda.current_stream(dev))     # create the events (torch creates lazily)
    stats = torch.zeros((total, 4), dtype=torch.int64, device=dev)
    sizes_log = torch.zeros((total, 2 * len(fan) + 1), dtype=torch.int64, device=dev)
    main = torch.cuda.current_stream(dev)
    NS = max(1, args.samplers)
    samp_streams = [main] if NS == 1 else [torch.cuda.Stream(dev) for _ in range(NS)]
    samp_ws = [None] if NS == 1 else [g.workspace() for _ in range(NS)]
    ev_samp = [torch.cuda.Event() for _ in range(RING)]
    # slot s's previous batch has been released (its release reads outs[s].n_id): a sampler on
    # its own stream must not overwrite that n_id before (on the caller's stream the release's
    # event wait orders it)
    ev_relslot = [torch.cuda.Event() for _ in range(RING)]
    relslot_live = [False] * RING

    def samplers_after(ev):       # timed regions: no sampling work before their start event
        if NS > 1:
            for ss in samp_streams:
                ss.wait_event(ev)
    pending = []
    # releases on their own stream (GD_RELEASE_STREAM=0: on main); release(j - Q) is ordered after extract(j)'s bookkeeping
    # and before extract(j + 1)'s (the sequential order of Alg. 1, so the buffer state is the
    # oracle's), and overlaps sample(j + 1), which does not touch the buffer
    rel_stream = torch.cuda.Stream(dev) if os.environ.get("GD_RELEASE_STREAM", "1") == "1" else main
    ev_bk = torch.cuda.Event()      # extract(j)'s bookkeeping enqueued on main
    ev_rel = torch.cuda.Event()     # release(j - Q) done
    rel_live = [False]

    # ---- f4: the train stage on its own stream (GraphSAGE 3 x 256; DDP all-reduce)
    model = None
    if args.train:
        from paper_conf_icpp_jiangj024_b200.train import SageModel
        n_cls = NUM_CLASSES.get(cfg.name, 64)
        dims = [cfg.feat_dim] + [256] * (len(fan) - 1) + [n_cls]   # L = #hops layers, hidden 256
        model = SageModel(dims, synth.sage_init(dims), nm, device=local_rank)
        labels_dev = synth.labels(seeds_dev.reshape(-1), n_cls).reshape(seeds_dev.shape)
        tstream = torch.cuda.Stream(dev)
        tdones = [torch.cuda.Event() for _ in range(RING)]
        for e in tdones:
            e.record(main)
        loss_log = torch.zeros(total, dtype=torch.float32, device=dev)
        t_events = []
    train_timing = [False]

    dbg = os.environ.get("GD_DEBUG_SYNC") == "1"

    def dsync(what, j):
        if dbg:
            torch.cuda.synchronize(dev)
            log(f"  step {j}: {what} ok")

    last_o = [None]
    host_wait = [0.0]     # seconds the host loop spent waiting for the bounded queue (not enqueueing)
    HOST_BOUND = os.environ.get("GD_HOST_BOUND", "1") == "1"   # GD_HOST_BOUND=0: unbounded host lookahead

    def step(j, host_inputs=False, host_out=None):
        s = j % RING
        o = outs[s]
        last_o[0] = o
        if HOST_BOUND:
            t_w = time.perf_counter()
            dones[s].synchronize()         # the host, too, stays at most RING batches ahead (bounded queue)
            host_wait[0] += time.perf_counter() - t_w
        ss = samp_streams[j % NS]
        ss.wait_event(dones[s])            # batch j - RING is complete: its buffers are free
        if relslot_live[s] and ss is not main:
            ss.wait_event(ev_relslot[s])   # ... and released
        if model is not None:
            ss.wait_event(tdones[s])       # ... and trained (the trainer reads outs[s], feats[s])
        sd = seeds_host[j] if host_inputs else seeds_dev[j]
        g.sample(sd, fan, synth.RNG_SEED, batch_ids[j], out=o, stream=ss, workspace=samp_ws[j % NS])
        if ss is not main:
            ev_samp[s].record(ss)
            main.wait_event(ev_samp[s])
        dsync("sample", j)
        if rel_live[0]:
            main.wait_event(ev_rel)        # the previous step's release precedes this lookup
        buf.extract(o.n_id, o.num_nodes_dev, o.max_nodes, out=feats[s], alias=aliases[s], stats=stats[j],
                    stream=main, done=dones[s])
        dsync("extract", j)
        if model is not None:              # f4 on stream T: train on batch j once its rows are in
            tstream.wait_event(dones[s])
            with torch.cuda.stream(tstream):
                if train_timing[0]:
                    a, z = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    a.record(tstream)
                model.step(o, feats[s], labels_dev[j], stream=tstream)
                scale = model.allreduce_grads()           # NCCL sum over ranks (no-op at N=1)
                model.apply_sgd(args.lr, scale, stream=tstream)
                loss_log[j].copy_(model.loss[0])
                if train_timing[0]:
                    z.record(tstream)
                    t_events.append((a, z))
            tdones[s].record(tstream)
        pending.append((o, s))
        if len(pending) == Q:
            r, rs = pending.pop(0)
            if rel_stream is not main:
                ev_bk.record(main)
                rel_stream.wait_event(ev_bk)
            buf.release(r.n_id, r.num_nodes_dev, r.max_nodes, stream=rel_stream)
            ev_relslot[rs].record(rel_stream)
            relslot_live[rs] = True
            if rel_stream is not main:
                ev_rel.record(rel_stream)
                rel_live[0] = True
            dsync("release", j)
        sizes_log[j].copy_(o.sizes, non_blocking=True)
        if host_out is not None:               # e2e: this step's result -> pinned host memory (D2H on the
            hs, hst, hev, seen = host_out      # stream), read by the host Q steps later (the paper's queue
            k = j % len(hev)                   # depth between stages), so the host keeps the
            if seen[0] >= 0 and j - len(hev) >= seen[2]:   # same lead over the device as a pipelined loader
                hev[k].synchronize()                       # the result of step j - len(hev)
                seen[1] += int(hs[k][len(fan)]) + int(hst[k][0]) + int(hst[k][1])
            hs[k].copy_(o.sizes, non_blocking=True)
            hst[k].copy_(stats[j], non_blocking=True)
            hev[k].record(main)
            if seen[0] < 0:
                seen[2] = j
            seen[0] = j

    # ---- full-size sampled parity vs the oracle (untimed; first batches of this rank)
    parity = None
    n_par = args.parity_batches if args.parity_batches is not None else default_parity_batches(
        cfg, world, len(synth.segment(wl.num_batches, rank, world)))
    if n_par > 0:
        log(f"parity check ({n_par} batches per rank) ...")
        parity = check_parity(n_par, cfg, g, buf, wl, sched, batch_ids, fan, n_max, S, dev, world)
        buf.close()
        buf = gd.FeatureBuffer(wl.table.tensor, S, Q, n_max, preload=cfg.preload, device=local_rank,
                               num_nodes=cfg.num_nodes)
        if "GD_HOST_THREADS" not in os.environ and not cfg.preload:
            buf.config(host_threads)
    barrier()
    if args.peer and world > 1:
        import torch.distributed as dist
        blobs = [None] * world
        dist.all_gather_object(blobs, buf.peer_export_ipc())
        buf.peer_attach_ipc([bl for r, bl in enumerate(blobs) if r != rank][:7])
        barrier()
        log(f"peer buffers attached: {min(world - 1, 7)} per rank")

    # ---- buffer pre-warm (untimed): the feature buffer reaches steady state once the
    # cumulative misses exceed its capacity; stats are read every 8 batches
    log(f"parity {parity}; pre-warm ...")
    jp = 0
    while jp < PRE:
        for _ in range(8):
            if jp < PRE:
                step(jp)
                jp += 1
        if int(stats[:jp, 1].sum().item()) >= S:
            break
    prewarm_batches = jp
    torch.cuda.synchronize(dev)
    off = jp              # schedule offset: everything below uses batches after the pre-warm
    log(f"pre-warm: {prewarm_batches} batches; warm-up ...")
    for j in range(off, off + W):
        step(j)
    torch.cuda.synchronize(dev)
    barrier()
    torch.cuda.synchronize(dev)

    # ---- timed region (device events on the launching stream)
    clock_sampler = ClockSampler(local_rank)     # NVML initialised here, outside the region
    import gc
    gc.collect()
    gc.disable()                                  # no collector pause in the host loop of the region
    torch.cuda.synchronize(dev)
    log("timed region ...")
    # Per-kernel event pairs (g / buf timing) cost the pipeline ~18% (200-step papers100m on one box:
    # 436-445 batches/s with them, 527-535 without; timing-enabled events recorded between the
    # chained kernels and copies), so the timed region runs without them and the live per-kernel
    # figures come from an instrumented region of K more steps after it (GD_KERNEL_TIMING=1: the
    # old way, pairs inside the timed region).
    KT = os.environ.get("GD_KERNEL_TIMING", "0") == "1"
    g.timing(KT)
    buf.timing(KT)
    train_timing[0] = True
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    with clock_sampler as clk:
        ev0.record(main)
        samplers_after(ev0)
        win_ev = []
        host_wait[0] = 0.0
        t_host0 = time.perf_counter()
        for j in range(off + W, off + W + K):
            step(j)
            if args.window and (j - off - W + 1) % args.window == 0:
                e_ = torch.cuda.Event(enable_timing=True)
                e_.record(main)
                win_ev.append(e_)
        t_host1 = time.perf_counter()
        main.wait_event(dones[(off + W + K - 1) % RING])  # the last batch's rows are all in `out`
        if rel_live[0]:
            main.wait_event(ev_rel)                          # ... and the last release is done
        if model is not None:
            main.wait_event(tdones[(off + W + K - 1) % RING])   # ... and it is trained
        ev1.record(main)
        ev1.synchronize()
    host_loop = {"enqueue_ms_per_step": round((t_host1 - t_host0) * 1e3 / K, 4),
                 "busy_ms_per_step": round((t_host1 - t_host0 - host_wait[0]) * 1e3 / K, 4),
                 "def": "host wall time of the timed loop per step, and the same minus the bounded-queue waits "
                        "(the host thread's own enqueue work: Python, ctypes, the library's API calls)"}
    torch.cuda.synchronize(dev)
    g.timing(False)
    buf.timing(False)
    train_timing[0] = False
    gc.enable()
    ms = ev0.elapsed_time(ev1)
    ms_max = max_over_ranks(ms, dev)
    windows = None
    if win_ev:   # caller-stream progress per window (the miss stream trails it by < Q batches)
        marks = [ev0] + win_ev
        windows = [round(args.window / (a_.elapsed_time(b_) / 1e3), 1) for a_, b_ in zip(marks, marks[1:])]
    tg = g.timing_read() if KT else None
    tb = buf.timing_read() if KT else None
    policy = buf.policy_read() if not cfg.preload else None
    st = stats[off + W:off + W + K].sum(0).cpu().tolist()
    sz = sizes_log[off + W:off + W + K].double().mean(0).cpu().tolist()
    hits, misses, miss_zc, miss_staged = (int(x) for x in st)
    barrier()

    # ---- the timed configuration's output rows, checked by their closed form (P5):
    # out[i] == table row (n_id[i] mod P) for the last Q + 1 batches of the timed region
    # (extracted back to back, no host sync between them)
    # (and, when the host CSR is at hand, their sampled node lists against the oracle's)
    rows_check = {"batches": 0, "rows": 0, "ok": True, "n_id_vs_oracle": None}
    torch.cuda.synchronize(dev)
    for j in range(max(off + W, off + W + K - RING), off + W + K):
        s_ = j % RING
        dones[s_].synchronize()
        n_j = int(sizes_log[j][len(fan)].item())
        n_id_j = outs[s_].n_id[:n_j].cpu()
        ids = n_id_j.long() % cfg.host_rows
        want = wl.table.tensor.index_select(0, ids)
        got = feats[s_][:n_j].view(torch.uint8).reshape(n_j, cfg.row_bytes).cpu()
        rows_check["ok"] &= bool(torch.equal(got, want))
        if wl.host_indptr is not None:
            from oracle import oracle as O
            b_, ep_ = sched[j % len(sched)]
            ref = O.sample(wl.host_indptr, wl.host_indices, wl.seeds(b_, ep_).cpu().numpy(), fan, synth.RNG_SEED,
                           batch_ids[j])
            same = bool(np.array_equal(n_id_j.numpy(), ref.n_id))
            rows_check["n_id_vs_oracle"] = same if rows_check["n_id_vs_oracle"] is None else (
                rows_check["n_id_vs_oracle"] and same)
        rows_check["batches"] += 1
        rows_check["rows"] += n_j
    log(f"pipelined rows check: {rows_check}")

    # ---- e2e through the public API with host inputs / host-read results
    log(f"timed: {ms:.2f} ms for {K} steps; e2e ...")
    e2e = None
    if not args.no_e2e:
        LAG = int(os.environ.get("GD_E2E_LAG", Q))
        h_sizes = [torch.zeros(2 * len(fan) + 1, dtype=torch.int64).pin_memory() for _ in range(LAG)]
        h_stats = [torch.zeros(4, dtype=torch.int64).pin_memory() for _ in range(LAG)]
        h_ev = [torch.cuda.Event() for _ in range(LAG)]
        seen = [-1, 0, 0]                  # last step copied, running sum of what the host read, first step
        torch.cuda.synchronize(dev)
        # W untimed warm-up steps through the same public-API path, as before the device-timed region
        # (the host checks above leave the pipeline drained and the host threads cold; without them
        # the e2e region of the default run came out 10-15% below the device-timed one on papers100m)
        for j in range(off + W + K, off + 2 * W + K):
            step(j, host_inputs=True, host_out=(h_sizes, h_stats, h_ev, seen))
        torch.cuda.synchronize(dev)
        seen[0], seen[1], seen[2] = -1, 0, 0
        barrier()
        gc.collect()
        gc.disable()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(main)
        samplers_after(e0)
        j_end = off + 2 * W + 2 * K
        e2e_win = []
        for j in range(off + 2 * W + K, j_end):
            step(j, host_inputs=True, host_out=(h_sizes, h_stats, h_ev, seen))
            if args.window and (j - off - 2 * W - K + 1) % args.window == 0:
                e_ = torch.cuda.Event(enable_timing=True)
                e_.record(main)
                e2e_win.append(e_)
        for j in range(max(off + 2 * W + K, j_end - LAG), j_end):   # the last LAG results, inside the timed region
            k = j % LAG
            h_ev[k].synchronize()
            seen[1] += int(h_sizes[k][len(fan)]) + int(h_stats[k][0]) + int(h_stats[k][1])
        main.wait_event(dones[(j_end - 1) % RING])
        if rel_live[0]:
            main.wait_event(ev_rel)
        if model is not None:
            main.wait_event(tdones[(j_end - 1) % RING])
        e1.record(main)
        e1.synchronize()
        gc.enable()
        e2e_ms = max_over_ranks(e0.elapsed_time(e1), dev)
        e2e_windows = None
        if e2e_win:
            marks = [e0] + e2e_win
            e2e_windows = [round(args.window / (a_.elapsed_time(b_) / 1e3), 1) for a_, b_ in zip(marks, marks[1:])]
        e2e = {"value": round(world * K / (e2e_ms / 1e3), 2), "unit": "batches/s", "windows": e2e_windows,
               "warmup_steps": W,
               "h2d_bytes_per_step": cfg.batch_size * 4,
               "d2h_bytes_per_step": (2 * len(fan) + 1) * 8 + 32,
               "read_back": f"each step's sizes + hit/miss stats copied D2H into pinned memory on the stream and "
                            f"read by the host {Q} steps later (queue depth Q, P:177; the last {Q} inside the timed "
                            f"region)"}
    # ---- capture for the steady-state replay: this rank's buffer has run steps
    # [0, j_win) (pre-warm, warm-up, timed, e2e); keep their per-batch sizes and hit/miss
    # counts, the last RING batches' n_id + alias and the whole buffer state for the oracle
    j_win = off + W + K + (0 if args.no_e2e else W + K)
    replay_cap = None
    if want_replay:
        torch.cuda.synchronize(dev)
        stats_h = stats[:j_win].cpu().numpy()
        sizes_h = sizes_log[:j_win].cpu().numpy()
        tail = {}
        for j in range(max(0, j_win - RING), j_win):
            s_ = j % RING
            n_j = int(sizes_h[j][len(fan)])
            tail[j] = (outs[s_].n_id[:n_j].cpu().numpy(), aliases[s_][:n_j].cpu().numpy())
        replay_cap = (j_win, stats_h, sizes_h, tail, buf.snapshot())
    # ---- f2 leg at N > 1 (after the main measurement and its replay window): every rank attaches
    # the other ranks' buffers as NVLink peers (CUDA IPC, "reuse feature data loaded by other
    # subprocesses") and runs W + K more steps; reports its rate and the share of misses peers served
    peer_leg = None
    if leg:
        import torch.distributed as dist
        torch.cuda.synchronize(dev)
        s0, p0 = buf.peer_stats()
        blobs = [None] * world
        dist.all_gather_object(blobs, buf.peer_export_ipc())
        buf.peer_attach_ipc([bl for r, bl in enumerate(blobs) if r != rank][:7])
        barrier()
        jl = j_win
        for j in range(jl, jl + W):
            step(j)
        torch.cuda.synchronize(dev)
        barrier()
        pa_, pz_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        pa_.record(main)
        samplers_after(pa_)
        for j in range(jl + W, jl + W + K):
            step(j)
        main.wait_event(dones[(jl + W + K - 1) % RING])
        if rel_live[0]:
            main.wait_event(ev_rel)
        pz_.record(main)
        pz_.synchronize()
        pl_ms = max_over_ranks(pa_.elapsed_time(pz_), dev)
        s1, p1 = buf.peer_stats()
        served, probed = sum_over_ranks(s1 - s0, dev), sum_over_ranks(p1 - p0, dev)
        barrier()
        buf.peer_attach_ipc([])
        barrier()
        peer_leg = {"value": round(world * K / (pl_ms / 1e3), 2), "unit": "batches/s", "steps": K,
                    "served_rows": int(served), "probed_misses": int(probed),
                    "served_share": round(served / max(1, probed), 4), "peers_per_rank": min(world - 1, 7),
                    "same_device": os.environ.get("GD_BENCH_SAME_DEVICE") == "1",
                    "def": "f2: W + K further steps with every other rank's buffer attached as a peer (misses probe the "
                           "peers' maps and copy served rows over NVLink before the host paths); max-over-ranks time"}
        log(f"f2 peer leg: {peer_leg}")
        j_win_after = jl + W + K
    else:
        j_win_after = j_win
    # ---- timeline (VERDICT r1 missing #7): TL more steps under the CUPTI activity tracer
    timeline = None
    if TL:
        import tempfile
        from torch.profiler import ProfilerActivity, profile
        from tools.timeline import summarise
        torch.cuda.synchronize(dev)
        with profile(activities=[ProfilerActivity.CUDA]) as prof:
            for j in range(j_win_after, j_win_after + TL):
                step(j)
            torch.cuda.synchronize(dev)
        with tempfile.NamedTemporaryFile(suffix=".json", delete=False) as tf:
            path = tf.name
        prof.export_chrome_trace(path)
        if rank == 0:
            timeline = summarise(path, args.timeline, TL, f"Timeline — {cfg.name}, {TL} steps (bench.py --timeline)")
            log(f"timeline: {timeline}")
        os.unlink(path)
        j_win_after += TL
    # ---- instrumented region: K more steps with per-kernel event pairs on the streams the kernels run
    # on (the live per-kernel figures: sampling, bookkeeping, hit gather, each miss path); its own
    # hit / miss counts go with its timings
    inst = {"hits": hits, "misses": misses, "miss_zc": miss_zc, "miss_staged": miss_staged,
            "region": "the timed region (GD_KERNEL_TIMING=1)"}
    if not KT:
        torch.cuda.synchronize(dev)
        g.timing(True)
        buf.timing(True)
        ji = j_win_after
        for j in range(ji, ji + KI):
            step(j)
        main.wait_event(dones[(ji + KI - 1) % RING])
        torch.cuda.synchronize(dev)
        g.timing(False)
        buf.timing(False)
        tg = g.timing_read()
        tb = buf.timing_read()
        sti = [int(x) for x in stats[ji:ji + KI].sum(0).cpu().tolist()]
        inst = {"hits": sti[0], "misses": sti[1], "miss_zc": sti[2], "miss_staged": sti[3],
                "region": f"{KI} steps after the timed region, per-kernel event pairs on (they slow the pipeline, "
                          f"so the timed region runs without them)"}
        j_win_after += KI
    # ---- optional in-process sweep of the miss-stream configuration (tuning only)
    sweep = []
    j0 = j_win_after
    for (thr, share, zcb, plb) in sweep_cfgs:
        torch.cuda.synchronize(dev)
        buf.config(int(thr), share, int(zcb), int(plb))
        for j in range(j0, j0 + W):
            step(j)
        torch.cuda.synchronize(dev)
        buf.timing(True)
        a = torch.cuda.Event(enable_timing=True)
        z = torch.cuda.Event(enable_timing=True)
        a.record(main)
        for j in range(j0 + W, j0 + W + K):
            step(j)
        main.wait_event(dones[(j0 + W + K - 1) % RING])
        if model is not None:
            main.wait_event(tdones[(j0 + W + K - 1) % RING])
        z.record(main)
        z.synchronize()
        buf.timing(False)
        t = buf.timing_read()
        sst = stats[j0 + W:j0 + W + K].sum(0).cpu().tolist()
        el = a.elapsed_time(z)
        rec = {"host_threads": int(thr), "share": share, "zc_blocks": int(zcb), "pull_blocks": int(plb),
               "batches_per_s": round(K / (el / 1e3), 1),
               "link_GBps": round(cfg.row_bytes * sst[1] / (el / 1e3) / 1e9, 2),
               "ms": {k: round(v / max(1, t["batches"]), 3) for k, v in t.items() if k.endswith("_ms")},
               "zero_copy_share_final": round(t["zero_copy_share"], 3)}
        log("sweep", rec)
        sweep.append(rec)
        j0 += W + K
    # ---- f1: the SET pipeline with S concurrent samplers (optionally out-of-order extraction)
    pipe_res = []
    if args.pipeline_sweep:
        from paper_conf_icpp_jiangj024_b200.pipeline import SETPipeline
        torch.cuda.synchronize(dev)
        while pending:                              # hand the buffer over with nothing in flight
            r, _ = pending.pop(0)
            buf.release(r.n_id, r.num_nodes_dev, r.max_nodes, stream=main)
        torch.cuda.synchronize(dev)
        for spec in args.pipeline_sweep.split(","):
            S_, ro = spec.split(":")
            pipe = SETPipeline(g, buf, fan, cfg.batch_size, synth.RNG_SEED, samplers=int(S_), release_lag=Q,
                               reorder=bool(int(ro)), device=local_rank)
            nrun = W + K
            base_j = j0
            sd = [seeds_dev[(base_j + j) % len(seeds_dev)] for j in range(nrun)]
            bi = [batch_ids[(base_j + j) % len(batch_ids)] for j in range(nrun)]
            pipe.run(sd[:W], bi[:W])
            torch.cuda.synchronize(dev)
            t0 = time.perf_counter()
            order, pst = pipe.run(sd[W:], bi[W:])
            torch.cuda.synchronize(dev)
            el = time.perf_counter() - t0
            inversions = sum(1 for a_, b_ in zip(order, order[1:]) if b_ < a_)
            rec = {"samplers": int(S_), "reorder": bool(int(ro)), "batches_per_s": round(K / el, 1),
                   "out_of_order_extractions": inversions}
            log("pipeline", rec)
            pipe_res.append(rec)
            j0 += nrun
    # ---- the hit gather alone, after the timed regions: once every batch is released the last
    # sampled batch is re-extracted, so all its rows are hits (no miss stream, no sampling
    # beside it), with L2 flushed before each of 5 repetitions.  The live figure is the same
    # kernel sharing the GPU with the next batches' sampling and the miss stream.
    iso = None
    if last_o[0] is not None:
        torch.cuda.synchronize(dev)
        while pending:
            r, _ = pending.pop(0)
            buf.release(r.n_id, r.num_nodes_dev, r.max_nodes, stream=main)
        torch.cuda.synchronize(dev)
        lo = last_o[0]
        flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
        iso_stats = torch.zeros(4, dtype=torch.int64, device=dev)
        iso_done = torch.cuda.Event()
        hits_iso = 0
        buf.timing(True)
        for _ in range(5):
            flush.fill_(1)                      # 256 MB > L2: the gather starts cold
            iso_stats.zero_()
            buf.extract(lo.n_id, lo.num_nodes_dev, lo.max_nodes, out=feats[0], alias=aliases[0], stats=iso_stats,
                        stream=main, done=iso_done)
            main.wait_event(iso_done)
            buf.release(lo.n_id, lo.num_nodes_dev, lo.max_nodes, stream=main)
            torch.cuda.synchronize(dev)
            hits_iso += int(iso_stats[0].item())
        buf.timing(False)
        ti = buf.timing_read()
        del flush
        if ti["gather_ms"] > 0 and hits_iso:
            n_iso = int(lo.num_nodes_dev.item()) * 5
            byts = 2 * cfg.row_bytes * hits_iso + 5 * n_iso
            gbs = byts / (ti["gather_ms"] * 1e6)
            iso = {"achieved": round(gbs, 1), "ms_per_launch": round(ti["gather_ms"] / 5, 4),
                   "rows_per_launch": hits_iso // 5,
                   "def": "k_gather_rows alone on an all-hit re-extraction of the last batch (L2 flushed, "
                          "5 launches, CUDA events on its stream); algorithmic bytes 2R per hit + 5 per node"}
    status_g = g.check()
    status_b = buf.check()

    # ---- reference measurements for the roofline
    hbm_peak = measured_peaks().get("hbm_gbs")
    hbm_src = "MEASURED_PEAKS.json hbm_gbs (measured copy)"
    if not hbm_peak:   # B200_PROFILING.md: fallback only when the driver-written file is absent
        hbm_peak, hbm_src = 6650.0, "of fallback: B200_PROFILING.md 6.65 TB/s (MEASURED_PEAKS.json absent)"
    link_peaks = h2d_peaks(dev, rank, world)
    link_peak = link_peaks["concurrent"]          # the denominator at G GPUs
    R = cfg.row_bytes
    region_s = ms / 1e3
    nb = max(1, tb["batches"])
    ih, im, izc, ist = inst["hits"], inst["misses"], inst["miss_zc"], inst["miss_staged"]
    gather_bytes = 2 * R * ih + 5 * (ih + im)              # read slot + write out, alias+flag reads
    gather_gbs = gather_bytes / (tb["gather_ms"] * 1e6) if tb["gather_ms"] > 0 else None
    zc_gbs = R * izc / (tb["miss_zero_copy_ms"] * 1e6) if tb["miss_zero_copy_ms"] > 0 and izc else None
    pull_gbs = R * ist / (tb["miss_staged_ms"] * 1e6) if tb["miss_staged_ms"] > 0 and ist else None
    host_gbs = R * ist / (tb["host_gather_ms"] * 1e6) if tb["host_gather_ms"] > 0 and ist else None
    ce_gbs = R * ist / (tb["staged_copy_ms"] * 1e6) if tb["staged_copy_ms"] > 0 and ist else None
    link_gbs = R * misses / region_s / 1e9 if misses else None   # both miss paths, over the timed region
    kern = {"sample_ms_per_batch": tg["sample_ms"] / max(1, tg["calls"]),
            "bookkeeping_ms_per_batch": tb["bookkeeping_ms"] / nb,
            "gather_ms_per_batch": tb["gather_ms"] / nb,
            "miss_zero_copy_ms_per_batch": tb["miss_zero_copy_ms"] / nb,
            "miss_staged_pull_ms_per_batch": tb["miss_staged_ms"] / nb,
            "host_gather_ms_per_batch": tb["host_gather_ms"] / nb,
            "staged_copy_engine_ms_per_batch": tb["staged_copy_ms"] / nb,
            "zero_copy_share_final": tb["zero_copy_share"]}
    rnd = lambda x, k=2: round(x, k) if x is not None else None  # noqa: E731
    roof_gather = {"bound": "hbm", "achieved": rnd(gather_gbs, 1), "peak": hbm_peak, "unit": "GB/s",
                   "frac": rnd(gather_gbs / hbm_peak, 4) if gather_gbs and hbm_peak else None, "traffic": None,
                   "kernel": "k_gather_rows", "peak_source": hbm_src,
                   "achieved_def": "live: algorithmic bytes of the hit gathers / their summed launch durations (events "
                                   "on the gather stream, concurrent with the next batches' sampling and the miss "
                                   "stream), over " + inst["region"]}
    if iso:
        iso["frac"] = rnd(iso["achieved"] / hbm_peak, 4) if hbm_peak else None
        roof_gather["isolated"] = iso
    roof_miss = {"bound": "host_link", "achieved": rnd(link_gbs), "peak": round(link_peak, 2), "unit": "GB/s",
                 "frac": rnd(link_gbs / link_peak, 4) if link_gbs else None, "traffic": None,
                 "kernel": ("k_miss_copy (zero-copy share) + host gather -> cudaMemcpyAsync H2D (copy engine) -> "
                            "k_miss_copy<staged> scatter" if os.environ.get("GD_STAGE_COPY_ENGINE", "1") != "0" else
                            "k_miss_copy (zero-copy share) + k_miss_copy<staged> (pull of the host-gathered share)"),
                 "achieved_def": "row bytes of all misses / timed region (the two miss paths run concurrently "
                                 "and are the critical path)",
                 "per_path_GBps": {"zero_copy_kernel": rnd(zc_gbs), "staged_pull_or_scatter_kernel": rnd(pull_gbs),
                                   "staged_copy_engine_h2d": rnd(ce_gbs), "host_gather_phase1": rnd(host_gbs),
                                   "measured_over": inst["region"]},
                 "misses_zero_copy": miss_zc, "misses_staged": miss_staged,
                 "peak_source": "in-run pinned 1 GiB H2D cudaMemcpyAsync, best of 10" + (
                     ", all ranks copying at once (barrier per repetition)" if world > 1 else "")}
    if world > 1:   # the whole job: every rank's misses over the slowest rank's region, vs the summed concurrent peaks
        tot_bytes = sum_over_ranks(R * misses, dev)
        tot_peak = sum_over_ranks(link_peak, dev)
        roof_miss["rank0"] = {"achieved": roof_miss["achieved"], "peak": roof_miss["peak"], "frac": roof_miss["frac"]}
        roof_miss["achieved"] = rnd(tot_bytes / (ms_max / 1e3) / 1e9)
        roof_miss["peak"] = round(tot_peak, 2)
        roof_miss["frac"] = rnd(roof_miss["achieved"] / tot_peak, 4) if tot_bytes else None
        roof_miss["achieved_def"] = ("row bytes of all ranks' misses / the slowest rank's timed region, against the "
                                     "sum of the per-rank concurrent H2D peaks")
    miss_busy = max(kern["miss_zero_copy_ms_per_batch"], kern["miss_staged_pull_ms_per_batch"],
                    kern["staged_copy_engine_ms_per_batch"])
    dominant = roof_miss if misses > 0 and miss_busy >= kern["gather_ms_per_batch"] else roof_gather
    traffic = load_traffic(cfg.name)
    if traffic:                            # per-launch DRAM bytes of the committed ncu launch list
        for kname, tv in traffic.items():
            base = kname.replace("gd::", "").split("<")[0]
            if base == roof_gather["kernel"] and isinstance(tv, (int, float)):
                roof_gather["traffic"] = tv
                roof_gather["traffic_source"] = f"profiles/traffic.json[{cfg.name}][{kname}] (ncu, per launch)"
    roof_miss["traffic_note"] = ("host-link bound: the bytes that bound it cross PCIe (R per miss); DRAM traffic of "
                                 "the miss kernels is in profiles/r01_<config>_launches.md")

    train_info = None
    if model is not None:
        t_ms = sum(a.elapsed_time(z) for a, z in t_events) / max(1, len(t_events))
        L = model.L
        flop = 0
        for j in range(L):
            nd, din, dout = sz[L - 1 - j], model.dims[j], model.dims[j + 1]   # mean actual dst rows
            flop += 2 * nd * 2 * din * dout * (2 if j == 0 else 3)   # fwd + dW (+ dA above layer 0)
        ll = loss_log[off + W:off + W + K].cpu().tolist()
        train_info = {"model": f"GraphSAGE mean, widths {model.dims} (P:173)", "lr": args.lr,
                      "train_ms_per_batch": round(t_ms, 4),
                      "gemm": "hand-written tcgen05 (gd_umma.cuh) over the device-resident row counts",
                      "gemm_gflop_per_batch": round(flop / 1e9, 2),
                      "gemm_tflops_if_train_ms_were_gemm": round(flop / (t_ms * 1e9), 1) if t_ms > 0 else None,
                      "loss_first": round(ll[0], 4), "loss_last": round(ll[-1], 4),
                      "allreduce": "NCCL all_reduce of the flat fp32 gradients (P:140)" if world > 1 else "none (N=1)"}
    peer_info = None
    if args.peer and world > 1:
        served, probed = buf.peer_stats()
        served_all, probed_all = sum_over_ranks(served, dev), sum_over_ranks(probed, dev)
        peer_info = {"served_rows": int(served_all), "probed_misses": int(probed_all),
                     "served_share": round(served_all / max(1, probed_all), 4), "peers_per_rank": min(world - 1, 7)}
    # ---- steady-state parity: the oracle replays this rank's whole schedule (CPU only)
    replay, single = None, None
    if replay_cap is not None:
        log(f"oracle replay of {replay_cap[0]} batches ...")
        thr = max(2, (os.cpu_count() or 2) // world)
        keep = want_cpu and S * R <= 48e9
        replay, single = oracle_replay(cfg, wl, seeds_host, batch_ids, fan, S, *replay_cap, threads=thr,
                                       keep_rows=keep, t_single=0.5 * args.cpu_seconds if want_cpu else 0.0)
        log(f"replay: {replay}")
    first_all = gather_objects(parity, world)
    replay_all = gather_objects(replay, world)
    parity_out = {"first": first_all[0] if world == 1 else first_all,
                  "steady_state": replay_all[0] if world == 1 else replay_all,
                  "bit_exact": all(x is None or x["bit_exact"] for x in first_all + replay_all)}
    cpu = None
    log("cpu baseline ...")
    if want_cpu:
        cpu = cpu_variant_baseline(cfg, wl.table.array, wl.host_indptr, wl.host_indices, seeds_host, batch_ids, fan,
                                   args.cpu_seconds, len(os.sched_getaffinity(0)))
        cpu["single_thread_full_oracle"] = single
        cpu["host_cpu"] = host_cpu_info()
    total_batches = sum_over_ranks(K, dev)
    value = total_batches / (ms_max / 1e3)
    line = {
        "metric": "SET (sampled+extracted+trained) mini-batches/s" if model is not None else "sampled+extracted mini-batches/s",
        "value": round(value, 2), "unit": "batches/s", "n_gpus": world, "steps": K, "warmup": W,
        "ms_per_step": round(ms_max / K, 4), "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "int32", "data": "synthetic (Chung-Lu power law, seeded; synth/)",
        "config": config_dict(cfg, S, world, prewarm_batches, NS, RING),
        "e2e": e2e,
        # per step: seed intake + K x (sample, relabel) + col resolve + hash clear | lookup, pop/assign, hit gather
        # [+ zero-copy miss copy unless preload] [+ staged scatter when the host path is on] [+ peer-tag
        # publish with peers attached: not in the timed region] | compact, release [| train: L x (agg, FWD GEMM,
        # DW GEMM, 2 colsum) + xent + loss + (L-1) x (DA GEMM, scatter init, scatter, relu') + SGD + L bf16 casts]
        "gpu_launches": K * ((2 * len(fan) + 3) + 3 + (0 if cfg.preload else 1) + (3 if args.peer and world > 1 else 0)
                             + (1 if (miss_staged > 0 or tb["miss_staged_ms"] > 1e-3) and not cfg.preload else 0) + 2
                             + (0 if model is None else 5 * model.L + 2 + 4 * (model.L - 1) + 1 + model.L)),
        "roofline": dominant,
        "roofline_gather": roof_gather,
        "roofline_miss": roof_miss,
        "cpu_baseline": cpu,
        "clocks": clk.summary(),
        "per_batch": {"n_nodes": round(sz[len(fan)], 1), "edges": [round(x, 1) for x in sz[len(fan) + 1:]],
                      "hits": hits / K, "misses": misses / K,
                      "hit_rate": round(hits / max(1, hits + misses), 4), **{k: round(v, 4) for k, v in kern.items()},
                      "kernel_ms_measured_over": inst["region"]},
        "miss_policy": {k: (round(v, 3) if isinstance(v, float) else v) for k, v in policy.items()} if policy else None,
        "parity": parity_out,
        "rows_check": rows_check,
        "host_link_peaks_GBps": {k: round(v, 2) for k, v in link_peaks.items()},
        "host_table": {"GB": round(cfg.host_rows * R / 1e9, 2), "thp_requested": bool(getattr(wl.table, "thp", False)),
                       "huge_pages_GB_after_fill": wl.thp_table_gb},
        "numa": numa,
        "windows": windows,
        "host_loop": host_loop,
        "sweep": sweep or None,
        "pipeline": pipe_res or None,
        "device_status": {"graph": status_g, "buffer": status_b},
        "peer": peer_info,
        "peer_leg": peer_leg,
        "timeline": timeline,
        "train": train_info,
        "setup_s": round(time.time() - t_setup, 1),
    }
    if rank == 0:
        s = json.dumps(line)
        print(s, flush=True)
        if args.out:
            with open(args.out, "w") as f:
                f.write(s + "\n")
    if model is not None:
        model.close()
    buf.close()
    g.close()
    wl.close()


def load_traffic(config_name):
    """dram bytes per launch from the committed ncu --set full summary, if any."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        return json.load(open(p)).get(config_name)
    except Exception:  # noqa: BLE001
        return None


def check_parity(n_par, cfg, g, buf, wl, sched, batch_ids, fan, n_max, S, dev, world):
    """Full-size cold parity: this rank's first `n_par` batches in the bench's launch
    configuration, bit-exact against the oracle: sampling outputs (sizes, n_id, rowptr, col,
    eid), alias, hits/misses, and the out rows (the oracle's slot rows at world 1; the closed
    form table[n_id mod P] (P5) at world > 1, where each rank's replay buffer keeps no rows)."""
    from oracle import oracle as O
    t0 = time.time()
    keep = world == 1
    ob = O.Buffer(wl.table.array, S, preload=cfg.preload, num_nodes=cfg.num_nodes, keep_rows=keep)
    log(f"  oracle buffer ready {time.time() - t0:.1f}s")
    res_ok = True
    checked = 0
    pend = []
    for j in range(min(n_par, len(sched))):
        b, ep = sched[j]
        seeds = wl.seeds(b, ep)
        o = g.sample(seeds.to(dev), fan, synth.RNG_SEED, batch_ids[j], with_eid=True)
        alias = torch.empty(n_max, dtype=torch.int32, device=dev)
        st = torch.zeros(4, dtype=torch.int64, device=dev)
        out, _, done = buf.extract(o.n_id, o.num_nodes_dev, o.max_nodes, alias=alias, stats=st)
        done.synchronize()
        h = o.to_host()
        ref = O.sample(wl.host_indptr, wl.host_indices, seeds.cpu().numpy(), fan, synth.RNG_SEED, batch_ids[j])
        ok = np.array_equal(h["sizes"], ref.sizes) and np.array_equal(h["n_id"], ref.n_id)
        for k in range(len(fan)):
            ok &= np.array_equal(h["rowptr"][k], ref.rowptr[k]) and np.array_equal(h["col"][k], ref.col[k])
            ok &= np.array_equal(h["eid"][k], ref.eid[k])
        o_out, o_alias, o_st = ob.extract(ref.n_id)
        n = len(ref.n_id)
        ok &= tuple(st.cpu().tolist()[:2]) == o_st
        ok &= np.array_equal(alias[:n].cpu().numpy(), o_alias)
        got = out[:n].cpu().numpy()
        ok &= np.array_equal(got, o_out if keep else wl.table.array[ref.n_id.astype(np.int64) % cfg.host_rows])
        pend.append((o, ref.n_id))           # release with lag Q, as the timed loop does
        if len(pend) == Q:
            o0, n0 = pend.pop(0)
            buf.release(o0.n_id, o0.num_nodes_dev, o0.max_nodes)
            ob.release(n0)
        res_ok &= bool(ok)
        checked += 1
        log(f"  batch {j}: ok={ok} ({time.time() - t0:.1f}s)")
    torch.cuda.synchronize(dev)
    return {"batches": checked, "bit_exact": res_ok, "seconds": round(time.time() - t0, 1),
            "rows_vs": "oracle slot rows" if keep else "closed form table[n_id mod P]"}


def oracle_replay(cfg, wl, seeds_host, batch_ids, fan, S, j_end, stats_h, sizes_h, tail, gpu_state, threads,
                  keep_rows, t_single=0.0):
    """Steady-state parity: the oracle's Alg. 1 replayed over this
    rank's WHOLE schedule [0, j_end) -- pre-warm, warm-up, timed and e2e batches, with the same
    release lag Q -- from its own sampling (never the GPU's n_id).  Compared per batch: the 2K+1
    block sizes and (hits, misses); for the last batches still in the bench's ring: n_id and
    alias; at the end: the whole buffer state (map slot / refcount / valid bit, reverse map,
    standby list in LRU order) against the GPU's snapshot.  Sampling runs `threads`-wide
    ahead (independent per batch); Alg. 1 itself is sequential, as the paper's.
    t_single > 0 (world 1): afterwards, the full oracle (sample + extract with rows + release)
    on one thread from this warm state for about t_single seconds: the single-thread figure."""
    from concurrent.futures import ThreadPoolExecutor
    from oracle import oracle as O
    t0 = time.time()
    ob = O.Buffer(wl.table.array, S, preload=cfg.preload, num_nodes=cfg.num_nodes, keep_rows=keep_rows)
    t_buf = time.time() - t0
    K = len(fan)

    def samp(j):
        return O.sample(wl.host_indptr, wl.host_indices, seeds_host[j].numpy(), fan, synth.RNG_SEED, batch_ids[j])

    bad_sizes, bad_stats, bad_tail = [], [], []
    pend = []
    hits = misses = 0
    with ThreadPoolExecutor(max(1, threads)) as ex:
        futs, nxt = {}, 0
        for j in range(j_end):
            while nxt < min(j_end, j + 2 * max(1, threads)):
                futs[nxt] = ex.submit(samp, nxt)
                nxt += 1
            ref = futs.pop(j).result()
            if not np.array_equal(ref.sizes, sizes_h[j]):
                bad_sizes.append(j)
            _, alias, st = ob.extract(ref.n_id, want_out=False)
            hits += st[0]
            misses += st[1]
            if st != (int(stats_h[j][0]), int(stats_h[j][1])):
                bad_stats.append(j)
            if j in tail:
                g_nid, g_alias = tail[j]
                if not (np.array_equal(g_nid, ref.n_id) and np.array_equal(g_alias, alias)):
                    bad_tail.append(j)
            pend.append(ref.n_id)
            if len(pend) == Q:
                ob.release(pend.pop(0))
    t_replay = time.time() - t0
    st_ok = None
    if gpu_state is not None:
        o = ob.state()
        st_ok = all(np.array_equal(gpu_state[k], o[k]) for k in ("slot", "rc", "valid", "reverse", "standby"))
    res = {"batches": j_end, "hits": int(hits), "misses": int(misses), "sizes_equal": not bad_sizes,
           "hits_misses_equal": not bad_stats, "tail_batches_n_id_alias": len(tail), "tail_equal": not bad_tail,
           "final_state_equal": st_ok,
           "bit_exact": not bad_sizes and not bad_stats and not bad_tail and st_ok is not False,
           "first_mismatch": min(bad_sizes + bad_stats + bad_tail) if (bad_sizes or bad_stats or bad_tail) else None,
           "seconds": round(t_replay, 1), "oracle_buffer_s": round(t_buf, 1), "sampler_threads": threads}
    single = None
    if t_single > 0 and keep_rows:
        n, t1 = 0, time.perf_counter()
        while True:
            j = j_end + n
            ref = samp(j % len(batch_ids))
            ob.extract(ref.n_id, want_out=True)
            pend.append(ref.n_id)
            if len(pend) == Q:
                ob.release(pend.pop(0))
            n += 1
            el = time.perf_counter() - t1
            if el >= t_single or n >= 10_000:
                break
        single = {"value": round(n / el, 3), "unit": "batches/s", "cores": 1, "kind": "oracle",
                  "sample": f"{n} full mini-batches (sample + Alg. 1 extract with rows + release, Q={Q}) continuing "
                            f"from the replayed steady-state buffer, {el:.1f} s on 1 host thread"}
    return res, single


def cpu_variant_baseline(cfg, table, indptr, indices, seeds_host, batch_ids, fan, budget_s, threads, n_target=None):
    """SURVEY 8(d) CPU baseline: the oracle's sample + relabel on `threads` host threads, one
    independent batch stream per thread (the paper's per-subprocess model), rows gathered
    straight from the host table (every row host-resident: the CPU variant's data path, P:152,
    without an SSD).  Runs until budget_s (or n_target batches in total); value = batches
    finished / wall time of the slowest thread."""
    from concurrent.futures import ThreadPoolExecutor
    from oracle import oracle as O
    R = table.shape[1]
    CH = max(1, (16 << 20) // R)                     # gather in 16 MB chunks per thread
    nb = len(batch_ids)
    t0 = time.perf_counter()
    stop = t0 + budget_s

    def work(t):
        out = np.empty((CH, R), dtype=np.uint8)
        done, j, rows = 0, t, 0
        while True:
            if n_target is not None and j >= n_target:
                break
            if n_target is None and time.perf_counter() >= stop:
                break
            ref = O.sample(indptr, indices, seeds_host[j % nb].numpy(), fan, synth.RNG_SEED, batch_ids[j % nb])
            for s0 in range(0, len(ref.n_id), CH):
                ids = ref.n_id[s0:s0 + CH]
                O.gather_rows(table, ids, out[:len(ids)])
            rows += len(ref.n_id)
            done += 1
            j += threads
        return done, rows, time.perf_counter()

    with ThreadPoolExecutor(threads) as ex:
        res = list(ex.map(work, range(threads)))
    n = sum(r[0] for r in res)
    el = max(r[2] for r in res) - t0
    return {"value": round(n / el, 3), "unit": "batches/s", "cores": threads, "kind": "oracle",
            "sample": f"{n} mini-batches of {cfg.name} (oracle sample + relabel, rows gathered from the host table: "
                      f"{sum(r[1] for r in res) * R / 2**30:.1f} GiB), one batch stream per thread on {threads} "
                      f"threads (every core of the affinity mask), {el:.1f} s",
            "seconds": round(el, 2)}


def host_cpu_info():
    import subprocess
    info = {"affinity_cores": len(os.sched_getaffinity(0))}
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            k, _, v = line.partition(":")
            if k.strip() in ("Model name", "Socket(s)", "Core(s) per socket", "Thread(s) per core", "NUMA node(s)", "CPU(s)"):
                info[k.strip()] = v.strip()
    except Exception:  # noqa: BLE001
        pass
    return info


def sample_ahead(args, cfg):
    """Batches sampled ahead of extraction.  Measured on one box each (profiles/r02_ab): products
    (all resident, sampling-bound) 4697 -> 5260 batches/s with 3; papers100m (host-link bound)
    the same rate with 0 or 3 (505-521) but the hit gather's live share of HBM 29-32% with 0 vs
    22% with 3 (the extra sampling in flight holds the SM slots the gather waits for)."""
    if args.sample_ahead is not None:
        return max(0, args.sample_ahead)
    return 3 if cfg.preload else 0


def config_dict(cfg, S, world, prewarm, samplers, ring):
    """The `config` object of the JSON line; identical for both arms."""
    R = cfg.row_bytes
    return {"workload": cfg.name, "num_nodes": cfg.num_nodes, "num_edges": cfg.num_edges,
            "feat_dim": cfg.feat_dim, "feat_bytes": R, "batch_size": cfg.batch_size, "fanouts": list(cfg.fanouts),
            "buffer_slots": S, "buffer_frac": round(S / cfg.num_nodes, 4), "release_lag": Q,
            "buffer_prewarm_batches": prewarm,
            "parallelism": f"dp{world} (batch segments, no collective)", "sampler_streams": samplers,
            "batches_in_flight": ring,
            "l2": "inputs larger than L2 (topology %.1f GB, slots %.1f GB, host table %.1f GB)" % (
                (cfg.num_nodes + 1) * 8e-9 + cfg.num_edges * 4e-9, S * R * 1e-9, cfg.host_rows * R * 1e-9),
            "host_table_rows": cfg.host_rows}


# ----------------------------------------------------------------------- reference arm

def run_reference(args, rank, world, local_rank):
    """The oracle (oracle/) as the reference arm, on the host cores; rank 0 only (the other
    ranks exit without work).  Never loads the product package (libgd.so).
      value: W warm-up then K timed mini-batches of the CPU variant (sample + relabel + rows
             from the host table) spread over every core of the affinity mask (cpu_variant_baseline);
      single_thread_full_oracle: the full oracle (Alg. 1 buffer with rows) on one thread, after
             the GPU arm's pre-warm rule (cumulative misses >= S, checked every 8 batches)."""
    if rank != 0:
        return
    from oracle import oracle as O
    cfg = config_from_args(args)
    dev = torch.device("cuda", local_rank) if torch.cuda.is_available() else torch.device("cpu")
    wl = Workload(cfg, 0, 1, dev, True)
    del wl.indptr, wl.indices
    wl.fill_table()
    fan = list(cfg.fanouts)
    nm = O.sample_bounds(cfg.batch_size, fan, cfg.num_nodes, cfg.num_edges)[0]
    S = capacity_for(cfg, nm[-1])
    W, K = args.warmup, args.steps
    PRE = 0 if cfg.preload else args.prewarm_max
    threads = len(os.sched_getaffinity(0))
    n_all = W + -(-K // threads) * threads + PRE + 64
    sched = batch_schedule(wl.num_batches, 0, 1, n_all)
    bids = [ep * wl.num_batches + b for b, ep in sched]
    seeds_host = torch.stack([wl.seeds(b, ep) for b, ep in sched]).cpu()
    # (1) multi-core CPU variant: W warm-up batches, then K timed batches over `threads` threads
    cpu_variant_baseline(cfg, wl.table.array, wl.host_indptr, wl.host_indices, seeds_host, bids, fan, 0, threads,
                         n_target=W)
    # K timed batches, rounded up to whole rounds of the thread pool so that every thread is busy
    # for the whole timed span (a rate over a partly idle pool would understate the host)
    n_timed = -(-K // threads) * threads
    cv = cpu_variant_baseline(cfg, wl.table.array, wl.host_indptr, wl.host_indices, seeds_host[W:], bids[W:], fan, 0,
                              threads, n_target=n_timed)
    v = cv["value"]
    # (2) the full single-thread oracle from a pre-warmed buffer (the GPU arm's rule)
    keep = S * cfg.row_bytes <= 48e9
    ob = O.Buffer(wl.table.array, S, preload=cfg.preload, num_nodes=cfg.num_nodes, keep_rows=keep)
    pend, jp, cum_miss = [], 0, 0

    def full_step(j, want_out):
        nonlocal cum_miss
        ref = O.sample(wl.host_indptr, wl.host_indices, seeds_host[j].numpy(), fan, synth.RNG_SEED, bids[j])
        _, _, st = ob.extract(ref.n_id, want_out=want_out)
        cum_miss += st[1]
        pend.append(ref.n_id)
        if len(pend) == Q:
            ob.release(pend.pop(0))

    while jp < PRE:
        for _ in range(8):
            if jp < PRE:
                full_step(jp, False)
                jp += 1
        if cum_miss >= S:
            break
    t1 = time.perf_counter()
    n1 = 0
    while n1 < 8 or time.perf_counter() - t1 < 6.0:
        full_step(jp + n1, keep)
        n1 += 1
        if jp + n1 >= len(bids) - 1:
            break
    el1 = time.perf_counter() - t1
    single = {"value": round(n1 / el1, 3), "unit": "batches/s", "cores": 1, "kind": "oracle",
              "sample": f"{n1} full mini-batches (sample + Alg. 1 extract{' with rows' if keep else ''} + release, "
                        f"Q={Q}) after a {jp}-batch pre-warm, {el1:.1f} s on 1 host thread"}
    line = {"impl": "reference", "metric": "sampled+extracted mini-batches/s", "value": v,
            "unit": "batches/s", "n_gpus": world, "steps": K, "warmup": W,
            "ms_per_step": round(1e3 / v, 3) if v else None, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "int32", "data": "synthetic (Chung-Lu power law, seeded; synth/)",
            "config": config_dict(cfg, S, world, jp, max(1, args.samplers), Q + 1 + sample_ahead(args, cfg)),
            "cpu_baseline": cv, "single_thread_full_oracle": single, "host_cpu": host_cpu_info(),
            "e2e": {"value": v, "unit": "batches/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "native_libs_loaded": loaded_native_libs()}
    print(json.dumps(line), flush=True)
    wl.close()


def main():
    import faulthandler
    faulthandler.dump_traceback_later(float(os.environ.get("GD_BENCH_WATCHDOG", "240")), repeat=True)
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        import torch.distributed as dist
        if os.environ.get("GD_BENCH_SAME_DEVICE") == "1" or not torch.cuda.is_available():
            # test modes: every rank on cuda:0 (1-GPU boxes; NCCL refuses shared GPUs) or CPU-only
            # (the reference arm's multi-rank launch), both over gloo
            local_rank = 0
            if torch.cuda.is_available():
                torch.cuda.set_device(0)
            dist.init_process_group("gloo")
        else:
            torch.cuda.set_device(local_rank)
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    try:
        if args.impl == "reference":
            run_reference(args, rank, world, local_rank)
        else:
            run_ours(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
