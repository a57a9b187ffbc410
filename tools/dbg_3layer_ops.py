import sys, ctypes, numpy as np
sys.path.insert(0, '.'); sys.path.insert(0, 'tests')
import paper_conf_ipps_kurtysps23_b200 as rdm
from oracle import gcn as og
from test_gpu_gcn import _problem, _run
rdm._lib.rdm_debug_disable_tc.argtypes = [ctypes.c_int]
f = (100, 256, 256, 47)
g, H0, Ws, y, m = _problem(n=6000, E=60000, f=f, seed=4)
for tc in (1, 0):
    rdm._lib.rdm_debug_disable_tc(1 - tc)
    loss, dW, model, ctx, _ = _run(rdm, g, H0, Ws, y, m, 0, P=1)
    T = lambda w, l: model.tensor_torch(w, l).cpu().numpy().astype(np.float64)
    H1, H2, G3, G2, G1 = T(rdm.T_H, 1), T(rdm.T_H, 2), T(rdm.T_G, 3), T(rdm.T_G, 2), T(rdm.T_G, 1)
    W = [w.astype(np.float64) for w in Ws]
    U3 = og.spmm(g, G3); G2r = (U3 @ W[2].T) * (H2 > 0)
    U2 = og.spmm(g, G2); G1r = (U2 @ W[1].T) * (H1 > 0)
    print('tc' if tc else 'simt', 'G2', og.max_rel_err(G2, G2r), 'G1', og.max_rel_err(G1, G1r),
          'Y3', og.max_rel_err(dW[2], H2.T @ U3), 'Y2', og.max_rel_err(dW[1], H1.T @ U2),
          'Y1', og.max_rel_err(dW[0], H0.astype(np.float64).T @ og.spmm(g, G1)))
    print('  |Y2| max', np.abs(H1.T @ U2).max(), 'sum|terms| max', (np.abs(H1).T @ np.abs(U2)).max())
