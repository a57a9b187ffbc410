"""Experiment: the hot-row panel of the residual SpMM on DRAM-resident slices
(spmm.cu Hot): time per call with the panel off (RDM_NO_HOT=1 at set_graph),
on with / without the L2 persisting window, at several panel budgets.
Usage: python tools/exp_hot.py <workload> <widths>"""
import os, sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wl = synth.WORKLOADS[sys.argv[1]]
g = synth.make_graph(wl)
widths = [int(x) for x in sys.argv[2].split(',')]
def timeit(fn, it=5):
    fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
Xs = {w: torch.randn(g.n, (w + 3) // 4 * 4, device=dev, generator=torch.Generator(device=dev).manual_seed(w)) for w in widths}
ref = {}
for mode in ['nohot', 'persist', 'nopersist']:
    os.environ.pop('RDM_NO_HOT', None); os.environ.pop('RDM_HOT_PERSIST', None)
    if mode == 'nohot':
        os.environ['RDM_NO_HOT'] = '1'
    if mode == 'nopersist':
        os.environ['RDM_HOT_PERSIST'] = '0'
    ctx = rdm.Context(device=0)
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=synth.symmetric_values(wl))
    for mb in (['64'] if mode == 'nohot' else ['32', '64', '96']):
        os.environ['RDM_HOT_MB'] = mb
        line = [f"{mode:>9} {mb:>3} MB"]
        for w in widths:
            O = torch.zeros_like(Xs[w])
            ms = timeit(lambda: ctx.spmm(0, Xs[w], O, w))
            if w not in ref:
                ref[w] = O.clone(); err = 0.0
            else:
                err = float((O[:, :w] - ref[w][:, :w]).abs().max() / ref[w][:, :w].abs().max())
            line.append(f"w{w}: {ms:.3f} ms (diff {err:.1e})")
        print(' | '.join(line), flush=True)
    del ctx
    torch.cuda.empty_cache()
