"""Practical HBM ceiling for row gathers: torch index_select of random rows of a
bf16 table (no reuse, table >> L2) for several row widths; prints GB/s of
(rows read + rows written)."""
import torch
torch.manual_seed(0)
N = 20_000_000
for cols in (104, 128, 96, 64):
    X = torch.randn(N, cols, device="cuda").to(torch.bfloat16)
    for order in ("random", "sorted"):
        idx = torch.randint(0, N, (25_000_000,), device="cuda")
        if order == "sorted":
            idx, _ = idx.sort()
        out = torch.empty(len(idx), cols, device="cuda", dtype=torch.bfloat16)
        for _ in range(3):
            torch.index_select(X, 0, idx, out=out)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(5):
            torch.index_select(X, 0, idx, out=out)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 5
        by = len(idx) * cols * 2 * 2 + len(idx) * 8
        print(f"cols {cols} ({cols*2} B rows) {order}: {ms:.3f} ms  {by / ms / 1e6:.0f} GB/s")
    del X, out, idx
    torch.cuda.empty_cache()
