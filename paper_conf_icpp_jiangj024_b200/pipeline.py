"""Pipelined sample -> extract -> (train) -> release driver.

GNNDrive runs "a pool of threads as samplers" feeding an extracting queue, extractors
feeding a training queue, and a releaser (Fig. 4; 4 samplers, queue capacities
6/4).  "Samplers concurrently deal with multiple mini-batches ... the order of
enqueuing mini-batches into the extracting queue may differ from the initial order"
(mini-batch reordering).

On the GPU: S sampler streams, each with its own gd_workspace, sample batches
concurrently; one extraction stream runs gd_extract in *completion* order (reorder=True:
the driver polls the samplers' events and extracts whichever batch finished first, the
paper's out-of-order extracting queue) or in submission order (reorder=False); the batch
extracted Q steps earlier is released after each extraction (training-queue depth Q).
The extraction order is recorded, so the sequential oracle can replay it bit-exactly.
This module is orchestration only: every step runs in libgd's kernels.
"""
from __future__ import annotations

import collections
import time

import torch

from . import FeatureBuffer, Graph


class SETPipeline:
    def __init__(self, graph: Graph, buf: FeatureBuffer, fanouts, batch_size: int, rng_seed: int,
                 samplers: int = 2, release_lag: int = 4, reorder: bool = True, device: int = 0,
                 max_wait_s: float = 0.002):
        assert samplers >= 1 and release_lag >= 1
        assert buf.max_inflight >= release_lag
        self.g, self.buf = graph, buf
        self.fanouts = list(fanouts)
        self.rng_seed = rng_seed
        self.S, self.Q, self.reorder = samplers, release_lag, reorder
        self.max_wait_s = max_wait_s
        self.dev = torch.device("cuda", device)
        self.n_max = graph.bounds(batch_size, self.fanouts)[0][-1]
        assert self.n_max <= buf.max_nodes_per_batch
        self.streams = [torch.cuda.Stream(self.dev) for _ in range(samplers)]
        self.workspaces = [graph.workspace() for _ in range(samplers)]
        self.xstream = torch.cuda.Stream(self.dev)               # extraction / release stream
        # per-batch buffers: S sampling + Q extracted-unreleased + 1 being extracted
        self.R = samplers + release_lag + 1
        self.outs = [graph.alloc_out(batch_size, self.fanouts) for _ in range(self.R)]
        self.feats = [buf.alloc_out(self.n_max) for _ in range(self.R)]
        self.alias = [torch.empty(self.n_max, dtype=torch.int32, device=self.dev) for _ in range(self.R)]
        self.stats = None
        self.free_ev = [torch.cuda.Event() for _ in range(self.R)]    # slot reusable once recorded
        for e in self.free_ev:
            e.record(self.xstream)
        self.order = []            # batch ids in extraction order

    def run(self, seeds, batch_ids, consumer=None):
        """Run every batch through sample -> extract -> release.  `seeds[k]` (device int32)
        and `batch_ids[k]` define batch k.  `consumer(k, out_rows, alias, done_event)` is the
        training-stage stand-in, called in extraction order.  Returns the extraction order
        (indices k) and per-batch stats [n, 4] (hits, misses, zero-copy, staged)."""
        n = len(seeds)
        self.stats = torch.zeros((n, 4), dtype=torch.int64, device=self.dev)
        slot_of = {}
        sampled = collections.OrderedDict()         # k -> (slot, event), sampled but not extracted
        extracted = collections.deque()             # (k, slot) extracted, not released
        free = collections.deque(range(self.R))
        nxt = 0
        order = []
        while len(order) < n:
            # keep up to S batches sampling
            while nxt < n and len(sampled) < self.S and free:
                slot = free.popleft()
                st = self.streams[nxt % self.S]
                st.wait_event(self.free_ev[slot])
                self.g.sample(seeds[nxt], self.fanouts, self.rng_seed, batch_ids[nxt], out=self.outs[slot],
                              stream=st, workspace=self.workspaces[nxt % self.S])
                ev = torch.cuda.Event()
                ev.record(st)
                sampled[nxt] = (slot, ev)
                slot_of[nxt] = slot
                nxt += 1
            # pick the batch to extract: the first finished sampler (reorder: poll the sampler
            # events for up to max_wait_s, like an extractor dequeuing whatever the samplers
            # finished first) or the oldest (in order: a device-side wait, no host poll)
            k = next(iter(sampled))
            if self.reorder:
                t0 = time.perf_counter()
                while True:
                    done = [kk for kk, (_, e) in sampled.items() if e.query()]
                    if done or time.perf_counter() - t0 > self.max_wait_s:
                        break
                    time.sleep(0)
                if done:
                    k = done[0]
            slot, ev = sampled.pop(k)
            self.xstream.wait_event(ev)
            o = self.outs[slot]
            done_ev = torch.cuda.Event()
            self.buf.extract(o.n_id, o.num_nodes_dev, o.max_nodes, out=self.feats[slot], alias=self.alias[slot],
                             stats=self.stats[k], stream=self.xstream, done=done_ev)
            order.append(k)
            if consumer is not None:
                consumer(k, self.feats[slot], self.alias[slot], done_ev)
            extracted.append((k, slot, done_ev))
            if len(extracted) == self.Q:
                k0, s0, d0 = extracted.popleft()
                o0 = self.outs[s0]
                self.buf.release(o0.n_id, o0.num_nodes_dev, o0.max_nodes, stream=self.xstream)
                self.xstream.wait_event(d0)              # its rows were consumed (done) before reuse
                self.free_ev[s0].record(self.xstream)
                free.append(s0)
        while extracted:                                  # drain: release the rest
            k0, s0, d0 = extracted.popleft()
            o0 = self.outs[s0]
            self.buf.release(o0.n_id, o0.num_nodes_dev, o0.max_nodes, stream=self.xstream)
            self.xstream.wait_event(d0)
            self.free_ev[s0].record(self.xstream)
            free.append(s0)
        self.order = order
        return order, self.stats
