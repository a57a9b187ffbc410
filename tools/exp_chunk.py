import os, sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wname = sys.argv[1]
wl = synth.WORKLOADS[wname]; g = synth.make_graph(wl)
ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val)
print(wname, ctx.graph_info(), flush=True)
def t(fn, it=3):
    fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
widths = [128, 44, 16] if wname == 'reddit' else [256, 100, 48]
for w in widths:
    X = torch.randn(g.n, w, device=dev); O = torch.zeros_like(X)
    res = []
    for c4 in [32, 16, 8, 4, 2]:
        os.environ['RDM_SPMM_CHUNK4'] = str(c4)
        res.append(f"c{c4*4}: {t(lambda: ctx.spmm(0, X, O, w)):.3f}")
    print(w, ' | '.join(res), flush=True)
    del X, O
