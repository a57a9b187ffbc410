import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wl = synth.WORKLOADS['reddit']; g = synth.make_graph(wl)
ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val)
print(ctx.graph_info())
def t(fn, it=5):
    fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
for w, ld in [(41, 44), (41, 48), (41, 64), (44, 44), (48, 48), (128, 128), (16, 16), (76, 76), (76, 80)]:
    X = torch.zeros(g.n, ld, device=dev); X[:, :w] = torch.randn(g.n, w, device=dev); O = torch.zeros_like(X)
    print(w, ld, f'{t(lambda: ctx.spmm(0, X, O, w)):.3f} ms', flush=True)
