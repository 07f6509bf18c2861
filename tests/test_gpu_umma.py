"""The train stage's hand-written tcgen05 GEMM (csrc/gd_umma.cuh) against a plain PyTorch
fp32 matmul of the same bf16 operands, through the C ABI (gd_debug_umma_gemm).

Both sides multiply the same bf16 values exactly (a bf16 x bf16 product is exact in fp32)
and accumulate in fp32 in different orders, so |C_gpu - C_ref| <= K 2^-23 (|A| |B|) + tiny;
the test uses 2^-14 (|A| |B|) for K <= 2^9 per CTA (DW: the split partials add via fp32
red.add, a few more roundings).  Shapes cover ragged device row counts (tiles past the
device count must not be touched), K not a multiple of the 64-wide stage, N = 47 (padded to
48 in B), N = 512 (two N tiles), several split-K CTAs, and an empty row count."""
import ctypes

import pytest
import torch

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def lib():
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_icpp_jiangj024_b200 import _lib
    return _lib


def vp(t):
    return ctypes.c_void_p(t.data_ptr() if t is not None else 0)


def run(lib, mode, A, lda, B, ldb, C, ldc, rows, rows_max, m_valid, k_valid, n_valid, n_store, splits=1,
        relu=0, bias=None):
    rows_dev = torch.tensor([rows], dtype=torch.int64, device="cuda")
    c_bf16 = int(C.dtype == torch.bfloat16)
    lib.check(lib.lib.gd_debug_umma_gemm(mode, vp(A), lda, vp(B), ldb, vp(C), ldc, c_bf16, relu, vp(bias),
                                         vp(rows_dev), rows_max, m_valid, k_valid, n_valid, n_store, splits,
                                         ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)))
    torch.cuda.synchronize()


def bf(shape, g):
    return (torch.randn(shape, generator=g) * 2).to(torch.bfloat16).cuda()


def close(got, ref, mag, tol=2.0 ** -14):
    err = (got - ref).abs()
    assert bool((err <= tol * mag + 1e-6).all()), float((err / (mag + 1e-6)).max())


@pytest.mark.parametrize("rows,rows_max,K,N", [(1000, 1300, 200, 256), (129, 512, 256, 47), (128, 128, 512, 256),
                                               (77, 300, 64, 16), (0, 256, 96, 32), (5000, 5000, 128, 208)])
def test_fwd(lib, rows, rows_max, K, N):
    g = torch.Generator().manual_seed(rows + K + N)
    Np = (N + 15) // 16 * 16
    A = bf((rows_max, K), g)
    W = torch.zeros(K, Np, dtype=torch.bfloat16, device="cuda")
    W[:, :N] = bf((K, N), g)
    bias = torch.randn(N, generator=g).cuda()
    C = torch.full((rows_max, Np), 7.0, device="cuda")
    H = torch.full((rows_max, Np), 7.0, device="cuda", dtype=torch.bfloat16)
    run(lib, 0, A, K, W, Np, C, Np, rows, rows_max, 0, K, Np, N, bias=bias)
    run(lib, 0, A, K, W, Np, H, Np, rows, rows_max, 0, K, Np, N, relu=1, bias=bias)
    Af, Wf = A[:rows].float(), W[:, :N].float()
    ref = Af @ Wf + bias
    mag = Af.abs() @ Wf.abs() + bias.abs()
    close(C[:rows, :N], ref, mag)
    # bf16 output: one more rounding of the result (unit roundoff 2^-8 relative)
    close(H[:rows, :N].float(), ref.clamp_min(0), mag + 2.0 ** 6 * ref.abs(), tol=2.0 ** -14)
    assert bool((C[rows:] == 7.0).all()) and bool((C[:, N:] == 7.0).all())   # nothing past the device count / n_store
    assert bool((H[rows:].float() == 7.0).all())


@pytest.mark.parametrize("rows,rows_max,K,N", [(1000, 1100, 256, 512), (300, 300, 48, 200), (129, 256, 256, 256)])
def test_da(lib, rows, rows_max, K, N):
    g = torch.Generator().manual_seed(3 * rows + K + N)
    dZ = bf((rows_max, K), g)
    W = bf((N, K), g)            # [2 din x dp] row-major: B[n, k]
    C = torch.full((rows_max, N), 7.0, device="cuda")
    run(lib, 1, dZ, K, W, K, C, N, rows, rows_max, 0, K, N, N)
    ref = dZ[:rows].float() @ W.float().T
    close(C[:rows], ref, dZ[:rows].float().abs() @ W.float().abs().T)
    assert bool((C[rows:] == 7.0).all())


@pytest.mark.parametrize("rows,Mv,N,splits", [(1000, 256, 256, 8), (70, 200, 48, 3), (4097, 512, 256, 37), (0, 256, 256, 4),
                                              (130, 128, 47, 1)])
def test_dw(lib, rows, Mv, N, splits):
    g = torch.Generator().manual_seed(5 * rows + Mv + N)
    Np = (N + 15) // 16 * 16
    A = bf((max(rows, 1) + 64, Mv), g)            # [rows x 2 din]
    B = torch.zeros(max(rows, 1) + 64, Np, dtype=torch.bfloat16, device="cuda")
    B[:, :N] = bf((max(rows, 1) + 64, N), g)
    pad = (rows + 63) // 64 * 64                  # the DW contract: rows [rows, round_up(rows, 64)) are zero
    A[rows:pad] = 0
    B[rows:pad] = 0
    A[pad:] = float("nan")                        # rows past that are never read
    B[pad:] = float("nan")
    C = torch.zeros(Mv, N, device="cuda")
    run(lib, 2, A, Mv, B, Np, C, N, rows, A.shape[0], Mv, 0, Np, N, splits=splits)
    Af, Bf = A[:rows].float(), B[:rows, :N].float()
    ref = Af.T @ Bf
    close(C, ref, Af.abs().T @ Bf.abs(), tol=2.0 ** -12)
