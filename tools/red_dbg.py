import torch, sys
sys.path.insert(0, '.')
import paper_conf_asplos_yangzd023_b200 as B
ctx = B.betty_ctx_create(0)
for (M, K, N) in [(64, 32, 32), (100, 41, 32), (1000, 64, 64), (300, 209, 256), (200000, 216, 256), (2000000, 216, 256)]:
    A = torch.randn((M, (K + 3) // 4 * 4), device="cuda")
    Bm = torch.randn((M, (N + 3) // 4 * 4), device="cuda")
    for tc in (True, False):
        C = B.betty_test_gemm(ctx, 1, A, Bm, K, N, tc)
        ref = A[:, :K].double().T @ Bm[:, :N].double()
        print(M, K, N, tc, "norm C", C.norm().item(), "ref", ref.norm().item(), "rel", ((C.double() - ref).norm() / ref.norm()).item(), flush=True)
