"""Experiment: residual-CSR SpMM time per call vs the lane mapping (G lanes per
nnz, V 128-bit gathers per lane, U nnz in flight per group) for both
precisions, on the Reddit-/products-shaped graph with the production hub tiles.
Usage: python tools/exp_gvu.py <workload> <widths> <prec> <G,V,U;G,V,U;...|auto>"""
import os, sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wl = synth.WORKLOADS[sys.argv[1]]
g = synth.make_graph(wl)
widths = [int(x) for x in sys.argv[2].split(',')]
prec = sys.argv[3]
combos = sys.argv[4].split(';')
ctx = rdm.Context(device=0)
ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
ctx.set_precision(prec)
def timeit(fn, it=5):
    fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
for w in widths:
    torch.manual_seed(w)
    X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev)
    ref = None
    out = []
    for cb in combos:
        for k in ('RDM_SPMM_GV', 'RDM_SPMM_U'):
            os.environ.pop(k, None)
        if cb != 'auto':
            G, V, U = cb.split(',')
            os.environ['RDM_SPMM_GV'] = f'{G},{V}'
            os.environ['RDM_SPMM_U'] = U
        O = torch.full_like(X, float('nan'))   # columns a mapping does not cover stay NaN
        try:
            ms = timeit(lambda: ctx.spmm(0, X, O, w))
        except Exception as ex:
            out.append(f"{cb}: ERR"); continue
        if ref is None:
            ref = O.clone()
        err = float((O[:, :w] - ref[:, :w]).abs().max() / ref[:, :w].abs().max())
        bad = bool(torch.isnan(O[:, :w]).any()) or not (err < 1e-6)
        out.append(f"{cb}: {ms:.3f}" + (" INVALID" if bad else ""))
    print(f"{sys.argv[1]} {prec} w{w}: " + " | ".join(out), flush=True)
