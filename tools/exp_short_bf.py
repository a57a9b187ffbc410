"""Fast-variant SpMM per call with the bf16 short-row kernel on the auxiliary
stream (RDM_SPMM_SHORT_BF=1, default) vs warp-per-row for every light row (0)."""
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
for wlname, widths in [('reddit', [128, 41, 16]), ('products', [256, 100, 47])]:
    wl = synth.WORKLOADS[wlname]; g = synth.make_graph(wl)
    ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True); ctx.set_precision('fast')
    def timeit(fn, it=10):
        fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
    for w in widths:
        X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev); res = []; ref = None
        for v in ['0', '1', '0', '1']:
            os.environ['RDM_SPMM_SHORT_BF'] = v
            O = torch.zeros_like(X)
            ms = timeit(lambda: ctx.spmm(0, X, O, w))
            if ref is None: ref = O.clone(); d = 0.0
            else: d = float((O[:, :w] - ref[:, :w]).abs().max() / ref[:, :w].abs().max())
            res.append(f"short_bf={v}: {ms:.3f} (rel {d:.1e})")
        print(wlname, f"w{w}", ' | '.join(res), flush=True)
        del X
    del ctx
