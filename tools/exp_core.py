"""Experiment: how much SpMM time does removing a dense hub core save, and what
does the core cost as a tcgen05 GEMM?"""
import sys, time, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wl = synth.WORKLOADS['reddit']; g = synth.make_graph(wl)
deg = np.diff(g.rowptr); order = np.argsort(-deg, kind='stable'); rank = np.empty(g.n, np.int64); rank[order] = np.arange(g.n)
rows = np.repeat(np.arange(g.n), deg)
def timeit(fn, it=5):
    fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
ctx = rdm.Context(device=0)
res = {}
for K in [0, 4096, 8192, 16384, 24576]:
    keep = ~((rank[rows] < K) & (rank[g.col] < K)) if K else np.ones(g.nnz, bool)
    r2 = rows[keep]; c2 = g.col[keep]; v2 = g.val[keep]
    rp = np.zeros(g.n + 1, np.int64); np.add.at(rp, r2 + 1, 1); rp = np.cumsum(rp)
    ctx.set_graph(rp, c2.astype(np.int32), v2, symmetric=True)
    line = [f"K={K:6d} nnz={keep.sum()/g.nnz:.3f}"]
    for w in (128, 44, 16):
        X = torch.randn(g.n, w, device=dev); O = torch.zeros_like(X)
        line.append(f"w{w}: {timeit(lambda: ctx.spmm(0, X, O, w)):.3f} ms")
    if K:
        A = torch.randn(K, K, device=dev)
        for w in (128, 48, 16):
            B = torch.randn(K, w, device=dev); C = torch.zeros(K, w, device=dev)
            line.append(f"core{w}: {timeit(lambda: ctx.gemm(rdm.GEMM_NN, A, B, C, K, K, w)):.3f} ms")
    print(' | '.join(line), flush=True)
