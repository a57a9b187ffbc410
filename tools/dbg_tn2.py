import os, sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm
dev = torch.device('cuda:0')
ctx = rdm.Context(device=0)
rows, k, m = 64, 128, 128
X = (np.arange(rows * k).reshape(rows, k) % 97).astype(np.float32) + 1
U = (np.arange(rows * m).reshape(rows, m) % 89).astype(np.float32) + 1
Xd = torch.from_numpy(X).to(dev); Ud = torch.from_numpy(U).to(dev)
ref = X.astype(np.float64).T @ U
for dbg in [0, 1, 2, 4]:
    os.environ['RDM_TC_DBG'] = str(dbg)
    Y = torch.zeros((k, m), device=dev)
    ctx.gemm(rdm.GEMM_TN, Xd, Ud, Y, rows, k, m); ctx.sync()
    y = Y.cpu().numpy()
    print('dbg', dbg, 'maxabs', np.abs(y).max(), 'relerr', np.abs(y - ref).max() / np.abs(ref).max())
    print('  y[0,:8]', y[0, :8]); print('  y[1,:8]', y[1, :8])
print('ref[0,:8]', ref[0, :8])
print('X[:2,:8]', X[:2, :8])
os.environ['RDM_TC_DBG'] = '0'
W = np.ones((k, m), np.float32); Wd = torch.from_numpy(W).to(dev)
C = torch.zeros((rows, m), device=dev); ctx.gemm(rdm.GEMM_NN, Xd, Wd, C, rows, k, m); ctx.sync()
print('NN err', np.abs(C.cpu().numpy() - X.astype(np.float64) @ W).max())
