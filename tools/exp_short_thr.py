"""SpMM per call vs the short-row degree threshold (RDM_SPMM_SHORT) with the
up-front (col, val) short-row kernel; outputs bitwise equal across thresholds."""
import os, sys, torch, numpy as np
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
for wlname, widths in [('reddit', [128, 41]), ('products', [256, 100, 47])]:
    wl = synth.WORKLOADS[wlname]; g = synth.make_graph(wl)
    ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    def timeit(fn, it=10):
        fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
    for w in widths:
        X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev); res = []; ref = None
        for thr in ['32', '40', '48', '64']:
            os.environ['RDM_SPMM_SHORT'] = thr
            O = torch.zeros_like(X)
            ms = timeit(lambda: ctx.spmm(0, X, O, w))
            if ref is None: ref = O.clone(); eq = True
            else: eq = bool(torch.equal(O.view(torch.int32), ref.view(torch.int32)))
            res.append(f"{thr}: {ms:.3f}" + ("" if eq else " DIFF"))
        os.environ.pop('RDM_SPMM_SHORT')
        print(wlname, f"w{w}", ' | '.join(res), flush=True)
        del X
    del ctx
