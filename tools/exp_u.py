"""Residual-CSR SpMM per call vs nnz in flight per lane group (RDM_SPMM_U) at the
Reddit-shaped widths (the long-row kernel is latency-bound: long-scoreboard
stalls ≈ 10.7 per issue, 47 % warps active)."""
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wl = synth.WORKLOADS['reddit']; g = synth.make_graph(wl)
ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
def timeit(fn, it=10):
    fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
for prec in (sys.argv[1].split(',') if len(sys.argv) > 1 else ['fp32', 'fast']):
    ctx.set_precision(prec)
    for w, gvs in ([(128, ['16,2', '32,1', '8,4'])] if len(sys.argv) > 2 else [(128, ['8,4', '16,2', '4,8']), (41, ['8,2', '4,3', '16,1']), (16, ['4,1', '2,2', '8,1'])]):
        X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev); O = torch.zeros_like(X)
        res = []; ref = None
        for gv in ['auto'] + gvs:
            for u in ['1', '2', '4']:
                os.environ.pop('RDM_SPMM_GV', None)
                if gv != 'auto': os.environ['RDM_SPMM_GV'] = gv
                os.environ['RDM_SPMM_U'] = u
                try:
                    ms = timeit(lambda: ctx.spmm(0, X, O, w))
                except Exception as ex:
                    res.append(f"{gv}/{u}: ERR"); continue
                if ref is None: ref = O[:, :w].clone(); d = 0.0
                else: d = float((O[:, :w] - ref).abs().max() / ref.abs().max())
                res.append(f"{gv}/{u}: {ms:.3f}" + ("" if d < 1e-5 else f" BAD {d:.1e}"))
        os.environ.pop('RDM_SPMM_GV', None); os.environ.pop('RDM_SPMM_U', None)
        print(prec, f"w{w}", ' | '.join(res), flush=True)
