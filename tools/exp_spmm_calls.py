"""Per-call SpMM times at the workload widths (for A/B of library builds:
RDM_LIB_VARIANT=<name> loads lib/librdm_<name>.so)."""
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
tag = os.environ.get('RDM_LIB_VARIANT', 'default')
for wlname, widths in [('reddit', [128, 41, 16]), ('products', [256, 100, 47])]:
    wl = synth.WORKLOADS[wlname]; g = synth.make_graph(wl)
    ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    def timeit(fn, it=10):
        fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
    res = []
    for w in widths:
        X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev); O = torch.zeros_like(X)
        res.append(f"w{w}: {timeit(lambda: ctx.spmm(0, X, O, w)):.3f} ms")
        del X, O
    print(tag, wlname, ' | '.join(res), flush=True)
    del ctx
