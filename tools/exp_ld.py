"""SpMM per-call time vs the row pitch (ld) of the dense operand: are narrow
slices (w = 41 → ld 44, 176-byte rows straddling 128-byte lines) faster with
64-byte-aligned rows (ld 48) or 128-byte rows (ld 64)?"""
import sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
for wlname, widths in [('reddit', [41, 16, 128]), ('products', [47, 100])]:
    wl = synth.WORKLOADS[wlname]; g = synth.make_graph(wl)
    ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    def timeit(fn, it=10):
        fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
    for w in widths:
        res = []; ref = None
        for ld in sorted({(w + 3) // 4 * 4, (w + 7) // 8 * 8, (w + 15) // 16 * 16, (w + 31) // 32 * 32}):
            X = torch.zeros(g.n, ld, device=dev); X[:, :w] = torch.randn(g.n, w, device=dev, generator=torch.Generator(device=dev).manual_seed(w))
            O = torch.zeros_like(X)
            ms = timeit(lambda: ctx.spmm(0, X, O, w))
            if ref is None: ref = O[:, :w].clone(); d = 0.0
            else: d = float((O[:, :w] - ref).abs().max())
            res.append(f"ld{ld}: {ms:.3f} ms (diff {d:.1e})")
            del X, O
        print(wlname, f"w{w}", ' | '.join(res), flush=True)
    del ctx
