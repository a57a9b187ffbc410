import sys, ctypes, numpy as np
sys.path.insert(0, '.'); sys.path.insert(0, 'tests')
import paper_conf_ipps_kurtysps23_b200 as rdm
import synth
from oracle import gcn as og, cost_model as ocm
from test_gpu_gcn import _problem, _run
rdm._lib.rdm_debug_disable_tc.argtypes = [ctypes.c_int]
f = (100, 256, 256, 47)
g, H0, Ws, y, m = _problem(n=6000, E=60000, f=f, seed=4)
ref = og.epoch(g, H0, Ws, y, m)
for tc in (1, 0):
    rdm._lib.rdm_debug_disable_tc(1 - tc)
    for cfg in ocm.pareto_front(f) + [0, 63]:
        for P in (1, 4):
            loss, dW, model, ctx, _ = _run(rdm, g, H0, Ws, y, m, cfg, P=P)
            errs = [og.max_rel_err(dW[l], ref.Y[l + 1]) for l in range(3)]
            print('tc' if tc else 'simt', cfg, P, f"loss {abs(loss-ref.loss)/abs(ref.loss):.1e}", ' '.join(f"{e:.1e}" for e in errs))
# conditioning: |Y1| entries
print('max|Y1|', np.abs(ref.Y[1]).max(), 'median', np.median(np.abs(ref.Y[1])))
