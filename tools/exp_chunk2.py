import os, sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
for wname, widths in (('products', [256]), ('reddit', [602, 256])):
    wl = synth.WORKLOADS[wname]; g = synth.make_graph(wl)
    ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val)
    def t(fn, it=3):
        fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
    for w in widths:
        ld = (w + 3) // 4 * 4
        X = torch.randn(g.n, ld, device=dev); O = torch.zeros_like(X)
        res = []
        for c4 in [32, 64]:
            os.environ['RDM_SPMM_CHUNK4'] = str(c4)
            res.append(f"c{c4*4}: {t(lambda: ctx.spmm(0, X, O, w)):.3f}")
        print(wname, w, ' | '.join(res), flush=True)
        del X, O
    del ctx
