"""Short-row SpMM: entries in flight per row (RDM_SPMM_SHORT_U 1 / 2 / 4) per
call at the workload widths; outputs bitwise equal (same entry order)."""
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
for wlname, widths in [('products', [256, 100, 47]), ('reddit', [128, 41])]:
    wl = synth.WORKLOADS[wlname]; g = synth.make_graph(wl)
    ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    def timeit(fn, it=10):
        fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
    for w in widths:
        X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev); res = []; ref = None
        for u in ['2', '4', '1', '2', '4']:
            os.environ['RDM_SPMM_SHORT_U'] = u
            O = torch.zeros_like(X)
            ms = timeit(lambda: ctx.spmm(0, X, O, w))
            if ref is None: ref = O.clone(); eq = True
            else: eq = bool(torch.equal(O.view(torch.int32), ref.view(torch.int32)))
            res.append(f"U{u}: {ms:.3f}" + ("" if eq else " DIFF"))
        os.environ.pop('RDM_SPMM_SHORT_U')
        print(wlname, f"w{w}", ' | '.join(res), flush=True)
        del X
    del ctx
