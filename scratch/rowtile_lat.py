"""Latency of the tcgen05 row-tile projection vs M (run under ncu for per-launch times)."""
import sys, numpy as np, torch
sys.path.insert(0, '/root/repo')
import paper_conf_ppopp_mal0c0wlc25_b200.apt as A
ctx = A.Ctx(0, 1, 0)
for (N, K) in ((256, 256), (256, 104), (48, 256)):
    for M in (128, 1024, 6800, 49500):
        Kp = (K + 1 + 7) // 8 * 8
        Z = torch.zeros(M, Kp, dtype=torch.bfloat16, device='cuda').normal_()
        W = torch.randn(N, K, device='cuda')
        b = torch.zeros(N, device='cuda')
        Y = torch.empty(M, (N + 3) // 4 * 4, device='cuda')
        for _ in range(3):
            ctx.project(Z, Kp, A.BF16, W, b, M, N, K, 1, Y, Y.shape[1])
        print(N, K, M, flush=True)
