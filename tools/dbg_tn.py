import sys, ctypes, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm
dev = torch.device('cuda:0')
ctx = rdm.Context(device=0)
for rows, k, m in [(64, 128, 128), (256, 128, 128), (1000, 7, 128), (1000, 128, 41), (5000, 602, 128)]:
    rng = np.random.default_rng(0)
    X = rng.standard_normal((rows, k)).astype(np.float32)
    U = rng.standard_normal((rows, m)).astype(np.float32)
    ldx = (k + 3) // 4 * 4; ldu = (m + 3) // 4 * 4
    Xd = torch.zeros((rows, ldx), device=dev); Xd[:, :k] = torch.from_numpy(X).to(dev)
    Ud = torch.zeros((rows, ldu), device=dev); Ud[:, :m] = torch.from_numpy(U).to(dev)
    Y = torch.zeros((k, m), device=dev)
    ctx.gemm(rdm.GEMM_TN, Xd, Ud, Y, rows, k, m)
    ctx.sync()
    ref = X.astype(np.float64).T @ U
    y = Y.cpu().numpy()
    print(rows, k, m, 'maxabs', np.abs(y).max(), 'err', np.abs(y - ref).max() / np.abs(ref).max())
    print(' y[0,:6]', y[0, :6]); print(' r[0,:6]', ref[0, :6])
    if k > 1: print(' y[1,:6]', y[1, :6]); print(' r[1,:6]', ref[1, :6])
