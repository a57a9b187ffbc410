"""SpMM per call with the short-row kernel on the auxiliary stream beside the
long-row kernel (RDM_SPMM_CONC=1, default) vs one stream (0); bit-identical."""
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
for wlname, widths in [('reddit', [128, 41, 16]), ('products', [256, 100, 47])]:
    wl = synth.WORKLOADS[wlname]; g = synth.make_graph(wl)
    ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    def timeit(fn, it=10):
        fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
    for w in widths:
        X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev)
        res = []; ref = None
        for c in ['0', '1', '0', '1']:
            os.environ['RDM_SPMM_CONC'] = c
            O = torch.zeros_like(X)
            ms = timeit(lambda: ctx.spmm(0, X, O, w))
            if ref is None: ref = O.clone(); same = True
            else: same = bool(torch.equal(O.view(torch.int32), ref.view(torch.int32)))
            res.append(f"conc={c}: {ms:.3f} ms{'' if same else ' DIFF'}")
        print(wlname, f"w{w}", ' | '.join(res), flush=True)
        del X
    del ctx
