"""Experiment: the short-row kernel (row per lane group) threshold — SpMM time
per call for RDM_SPMM_SHORT in {0 (off), 8, 16, 32, 64, 127}.
Usage: python tools/exp_short.py <workload> <widths> [P (emulated rank 0 of P)] [precision]"""
import os, sys, time, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wl = synth.WORKLOADS[sys.argv[1]]
t0 = time.time(); g = synth.make_graph(wl); print(f"gen {time.time() - t0:.1f}s", flush=True)
widths = [int(x) for x in sys.argv[2].split(',')]
P = int(sys.argv[3]) if len(sys.argv) > 3 else 1
ctx = rdm.Context(rank=0, world=P, device=0, emulate=True) if P > 1 else rdm.Context(device=0)
if len(sys.argv) > 4:
    ctx.set_precision(sys.argv[4])
ctx.set_graph(g.rowptr, g.col, g.val, symmetric=synth.symmetric_values(wl))
n = g.n
del g
def timeit(fn, it=3):
    fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
for w in widths:
    X = torch.randn(n, (w + 3) // 4 * 4, device=dev, generator=torch.Generator(device=dev).manual_seed(w))
    ref = None
    line = [f"w{w}"]
    for t in ('0', '8', '16', '32', '64', '127'):
        os.environ['RDM_SPMM_SHORT'] = t
        O = torch.zeros_like(X)
        ms = timeit(lambda: ctx.spmm(0, X, O, w))
        if ref is None:
            ref = O.clone(); err = 0.0
        else:
            err = float((O[:, :w] - ref[:, :w]).abs().max() / ref[:, :w].abs().max())
        line.append(f"short<={t}: {ms:.3f}" + ("" if err < 1e-6 else f" BAD {err:.1e}"))
    print(" | ".join(line), flush=True)
    del X
    torch.cuda.empty_cache()
