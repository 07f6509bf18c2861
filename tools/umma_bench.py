"""Stand-alone timing of the train stage's tcgen05 GEMM (gd_debug_umma_gemm) at the f4 layer
shapes, for ncu source-level profiling: python tools/umma_bench.py [reps]."""
import ctypes
import os
import sys


import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icpp_jiangj024_b200 import _lib

SHAPES = [  # (name, mode, rows, K, N)
    ("fwd_l0", 0, 120_000, 200, 256), ("fwd_l1", 0, 11_000, 512, 256), ("fwd_top", 0, 1024, 512, 47),
    ("dw_l0", 2, 120_000, 200, 256), ("da_l1", 1, 11_000, 256, 512)]


def vp(t):
    return ctypes.c_void_p(t.data_ptr())


def main(reps):
    st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    for name, mode, rows, K, N in SHAPES:
        Np = (N + 15) // 16 * 16
        rows_dev = torch.tensor([rows], dtype=torch.int64, device="cuda")
        if mode == 0:
            A = torch.randn(rows, K, device="cuda").bfloat16()
            B = torch.randn(K, Np, device="cuda").bfloat16()
            C = torch.empty(rows, Np, device="cuda", dtype=torch.bfloat16)
            args = (0, vp(A), K, vp(B), Np, vp(C), Np, 1, 1, None, vp(rows_dev), rows, 0, K, Np, N, 1, st)
            byts = rows * K * 2 + rows * N * 2
        elif mode == 1:
            A = torch.randn(rows, K, device="cuda").bfloat16()
            B = torch.randn(N, K, device="cuda").bfloat16()
            C = torch.empty(rows, N, device="cuda")
            args = (1, vp(A), K, vp(B), K, vp(C), N, 0, 0, None, vp(rows_dev), rows, 0, K, N, N, 1, st)
            byts = rows * K * 2 + rows * N * 4
        else:
            A = torch.randn(rows, K, device="cuda").bfloat16()
            B = torch.randn(rows, Np, device="cuda").bfloat16()
            C = torch.zeros(K, N, device="cuda")
            args = (2, vp(A), K, vp(B), Np, vp(C), N, 0, 0, None, vp(rows_dev), rows, K, 0, Np, N, 148 // ((K + 127) // 128), st)
            byts = rows * K * 2 + rows * Np * 2
        for _ in range(3):
            _lib.check(_lib.lib.gd_debug_umma_gemm(*args))
        torch.cuda.synchronize()
        # capture the launches in a CUDA graph so the host-side argument setup of the test
        # entry (tensor maps, counter) does not leave the GPU idle between launches
        gs = torch.cuda.Stream()
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph, stream=gs):
            a2 = list(args)
            a2[-1] = ctypes.c_void_p(gs.cuda_stream)
            for _ in range(reps):
                _lib.check(_lib.lib.gd_debug_umma_gemm(*a2))
        graph.replay()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        graph.replay()
        e1.record()
        torch.cuda.synchronize()
        us = e0.elapsed_time(e1) / reps * 1e3
        print(f"{name:8} rows {rows:7d} K {K:4d} N {N:4d}: {us:8.1f} us  {byts / us / 1e3:7.1f} GB/s  "
              f"{2 * rows * K * N / us / 1e6:7.1f} TFLOP/s")


if __name__ == "__main__":
    main(int(sys.argv[1]) if len(sys.argv) > 1 else 20)
