import sys, ctypes, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm
dev = torch.device('cuda:0')
ctx = rdm.Context(device=0)
lib = rdm._lib
lib.rdm_debug_disable_tc.argtypes = [ctypes.c_int]
def pad(A):
    r, c = A.shape; ld = (c + 3) // 4 * 4
    t = torch.zeros((r, ld), device=dev); t[:, :c] = torch.from_numpy(A).to(dev); return t
for rows, k, m in [(6000, 100, 256), (6000, 256, 256), (6000, 256, 47), (4097, 256, 256), (300, 100, 256), (20000, 602, 128), (20000, 128, 41)]:
    rng = np.random.default_rng(1)
    X = rng.standard_normal((rows, k)).astype(np.float32)
    W = rng.standard_normal((k, m)).astype(np.float32)
    G = rng.standard_normal((rows, m)).astype(np.float32)
    for tc in (1, 0):
        lib.rdm_debug_disable_tc(1 - tc)
        Xd, Gd, Wd = pad(X), pad(G), torch.from_numpy(W).to(dev)
        C = torch.zeros((rows, (m+3)//4*4), device=dev); ctx.gemm(rdm.GEMM_NN, Xd, Wd, C, rows, k, m)
        D = torch.zeros((rows, (k+3)//4*4), device=dev); ctx.gemm(rdm.GEMM_NT, Gd, Wd, D, rows, k, m)
        Y = torch.zeros((k, m), device=dev); ctx.gemm(rdm.GEMM_TN, Xd, Gd, Y, rows, k, m)
        ctx.sync()
        X64, W64, G64 = X.astype(np.float64), W.astype(np.float64), G.astype(np.float64)
        e = lambda a, r: float(np.abs(a - r).max() / np.abs(r).max())
        print(f"{'tc  ' if tc else 'simt'} {rows:6d} {k:4d} {m:4d}  NN {e(C[:, :m].cpu().numpy(), X64 @ W64):.2e}  NT {e(D[:, :k].cpu().numpy(), G64 @ W64.T):.2e}  TN {e(Y.cpu().numpy(), X64.T @ G64):.2e}")
