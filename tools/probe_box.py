"""Probe the GPU box: host RAM, CPU, PCIe host-link bandwidth (pinned H2D/D2H), GPU facts.

Writes gpurun_out/probe.json. Not part of the product path; used to size the workloads.
"""
import json
import os
import subprocess
import time

import torch


def sh(cmd):
    try:
        return subprocess.run(cmd, shell=True, capture_output=True, text=True, timeout=60).stdout
    except Exception as e:  # noqa: BLE001
        return f"ERR {e}"


def bw(src, dst, iters=10):
    s = torch.cuda.Stream()
    best = 0.0
    with torch.cuda.stream(s):
        for _ in range(iters):
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record(s)
            dst.copy_(src, non_blocking=True)
            b.record(s)
            b.synchronize()
            ms = a.elapsed_time(b)
            best = max(best, src.numel() * src.element_size() / ms / 1e6)
    return best


def main():
    os.makedirs("gpurun_out", exist_ok=True)
    out = {}
    out["nproc"] = os.cpu_count()
    out["affinity"] = len(os.sched_getaffinity(0))
    out["free"] = sh("free -g")
    out["lscpu"] = sh("lscpu | head -30")
    out["numa"] = sh("numactl -H 2>/dev/null | head -20")
    out["shm"] = sh("df -h /dev/shm")
    out["ulimit_l"] = sh("ulimit -l")
    out["smi"] = sh("nvidia-smi --query-gpu=index,name,memory.total,clocks.sm,clocks.max.sm,pcie.link.gen.current,pcie.link.width.current --format=csv")
    out["topo"] = sh("nvidia-smi topo -m")
    p = torch.cuda.get_device_properties(0)
    out["props"] = {"name": p.name, "sms": p.multi_processor_count, "mem": p.total_memory,
                    "l2": getattr(p, "L2_cache_size", None)}
    n = 1 << 30
    t0 = time.time()
    h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    out["pin_1GiB_s"] = time.time() - t0
    h.fill_(1)
    d = torch.empty(n, dtype=torch.uint8, device="cuda")
    out["h2d_GBps"] = bw(h, d)
    out["d2h_GBps"] = bw(d, h)
    # big pinned alloc timing (8 GiB)
    t0 = time.time()
    try:
        big = torch.empty(8 << 30, dtype=torch.uint8, pin_memory=True)
        out["pin_8GiB_s"] = time.time() - t0
        del big
    except Exception as e:  # noqa: BLE001
        out["pin_8GiB_err"] = str(e)
    json.dump(out, open("gpurun_out/probe.json", "w"), indent=1)
    print(json.dumps({k: v for k, v in out.items() if not isinstance(v, str)}, indent=1))
    print(out["free"], out["smi"], out["lscpu"])


if __name__ == "__main__":
    main()
