"""The dense kernels alone (tcgen05 tensor-core path and SIMT path) against
torch matmul in float64 of the same bf16 operands (test hook betty_test_gemm).
Shapes span several 128-row tiles, ragged M / K / N tails and N up to 256."""
import pytest
import torch

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def B():
    import paper_conf_asplos_yangzd023_b200 as B
    return B


@pytest.fixture(scope="module")
def ctx(B):
    return B.betty_ctx_create(0)


SHAPES = [(1, 16, 16), (127, 64, 48), (128, 100, 47), (300, 209, 256), (5000, 257, 96), (4099, 513, 208),
          (700, 40, 256), (2000, 513, 256), (1000, 257, 256),   # these three stream B (too big to stay resident)
          (777, 200, 513)]                                       # 256-column blocks (the pool layers' dXA)


def rel(a, b):
    return (torch.linalg.norm(a.double() - b) / torch.linalg.norm(b)).item()


@pytest.mark.parametrize("use_tc", [True, False])
@pytest.mark.parametrize("M,K,N", SHAPES)
def test_row_gemm(B, ctx, M, K, N, use_tc):
    g = torch.Generator(device="cuda").manual_seed(M + K + N)
    ld = (K + 7) // 8 * 8
    A = torch.randn((M, ld), device="cuda", generator=g).to(torch.bfloat16)
    W = torch.randn((N, ld), device="cuda", generator=g).to(torch.bfloat16)
    C = B.betty_test_gemm(ctx, 0, A, W, K, N, use_tc)
    ref = A[:, :K].double() @ W[:, :K].double().T
    assert rel(C, ref) < 1e-5


@pytest.mark.parametrize("use_tc", [True, False])
@pytest.mark.parametrize("M,K,N", SHAPES)
def test_red_gemm(B, ctx, M, K, N, use_tc):
    g = torch.Generator(device="cuda").manual_seed(7 * M + K + N)
    lda, ldb = (K + 7) // 8 * 8, (N + 7) // 8 * 8
    A = torch.randn((M, lda), device="cuda", generator=g).to(torch.bfloat16)
    Bm = torch.randn((M, ldb), device="cuda", generator=g).to(torch.bfloat16)
    C = B.betty_test_gemm(ctx, 1, A, Bm, K, N, use_tc)
    ref = A[:, :K].double().T @ Bm[:, :N].double()
    assert rel(C, ref) < 1e-5


def test_red_gemm_ignores_rows_past_M(B, ctx):
    """Garbage (NaN) past the last valid row must not leak into the reduction."""
    M, K, N = 1000, 64, 64
    A = torch.randn((1100, K), device="cuda").to(torch.bfloat16)
    Bm = torch.randn((1100, N), device="cuda").to(torch.bfloat16)
    A[M:] = float("nan")
    Bm[M:] = float("nan")
    for tc in (True, False):
        C = B.betty_test_gemm(ctx, 1, A, Bm, K, N, tc, M=M)
        ref = A[:M].double().T @ Bm[:M].double()
        assert torch.isfinite(C).all()
        assert rel(C, ref) < 1e-5


# ------------------------------------------------ FP32 mode: 3xTF32 on tcgen05 (vs SIMT FFMA)
@pytest.mark.parametrize("use_tc", [True, False])
@pytest.mark.parametrize("M,K,N", SHAPES)
def test_row_gemm_fp32(B, ctx, M, K, N, use_tc):
    """fp32 operands: the 3xTF32 split (hi*hi + lo*hi + hi*lo) is accurate to ~1e-6 relative (the
    dropped lo*lo term and the tf32 truncation of lo are ~2^-21), like SIMT FFMA; plain TF32 would be
    ~1e-3 and fails this bound."""
    g = torch.Generator(device="cuda").manual_seed(M + K + N)
    ld = (K + 3) // 4 * 4
    A = torch.randn((M, ld), device="cuda", generator=g)
    W = torch.randn((N, ld), device="cuda", generator=g)
    C = B.betty_test_gemm(ctx, 0, A, W, K, N, use_tc)
    ref = A[:, :K].double() @ W[:, :K].double().T
    assert rel(C, ref) < 3e-6


@pytest.mark.parametrize("use_tc", [True, False])
@pytest.mark.parametrize("M,K,N", SHAPES)
def test_red_gemm_fp32(B, ctx, M, K, N, use_tc):
    g = torch.Generator(device="cuda").manual_seed(7 * M + K + N)
    lda, ldb = (K + 3) // 4 * 4, (N + 3) // 4 * 4
    A = torch.randn((M, lda), device="cuda", generator=g)
    Bm = torch.randn((M, ldb), device="cuda", generator=g)
    C = B.betty_test_gemm(ctx, 1, A, Bm, K, N, use_tc)
    ref = A[:, :K].double().T @ Bm[:, :N].double()
    assert rel(C, ref) < 3e-6


def test_red_gemm_fp32_ignores_rows_past_M(B, ctx):
    M, K, N = 1000, 64, 64
    A = torch.randn((1100, K), device="cuda")
    Bm = torch.randn((1100, N), device="cuda")
    A[M:] = float("nan")
    Bm[M:] = float("nan")
    for tc in (True, False):
        C = B.betty_test_gemm(ctx, 1, A, Bm, K, N, tc, M=M)
        ref = A[:M].double().T @ Bm[:M].double()
        assert torch.isfinite(C).all()
        assert rel(C, ref) < 3e-6
