import numpy as np, torch, sys
sys.path.insert(0, '/root/repo')
import paper_conf_ppopp_mal0c0wlc25_b200.apt as A
np.set_printoptions(linewidth=200, precision=3, suppress=True)
ctx = A.Ctx(0, 1, 0)
def run(Z, W, relu=0):
    M, K = Z.shape; N = W.shape[0]
    kp = (K + 7) // 8 * 8
    Zb = np.zeros((M, kp), np.uint16)
    Zb[:, :K] = (Z.astype(np.float32).view(np.uint32) >> 16).astype(np.uint16)
    yp = (N + 3) // 4 * 4
    Y = torch.full((M, yp), -7.0, dtype=torch.float32, device="cuda")
    ctx.project(torch.as_tensor(Zb.view(np.int16)).cuda(), kp, A.BF16, torch.as_tensor(W.astype(np.float32)).cuda(),
                torch.zeros(N, device='cuda'), M, N, K, relu, Y, yp)
    return Y.cpu().numpy()[:, :N]
M, N, K = 128, 16, 64
print("ones", run(np.ones((M, K)), np.ones((N, K)))[:3])
Z = np.zeros((M, K)); Z[np.arange(M), np.arange(M) % K] = 1
W = np.arange(N * K).reshape(N, K) / 64.0
print("Z=e_{m%64}, W[n,k]=(n*64+k)/64 -> Y[m,n] = n + (m%64)/64")
y = run(Z, W)
print(y[:4]); print(y[64:66]); print(y[120:128:3])
Z = np.ones((M, K)); W = np.zeros((N, K)); W[:, 0] = np.arange(N)
print("W col0 = n", run(Z, W)[:2])
Z = np.zeros((M, K)); Z[:, 0] = np.arange(M); W = np.zeros((N, K)); W[:, 0] = 1
print("Z col0 = m", run(Z, W)[:, 0][:40])
