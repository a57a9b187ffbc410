import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm
import os
dev = torch.device('cuda:0'); ctx = rdm.Context(device=0)
ctx.set_precision(os.environ.get('RDM_PREC', 'fp32'))
rows = 232965
def t(fn, it=10):
    fn(); ctx.sync(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it * 1e3
for (op, k, m, epi) in [(rdm.GEMM_NT, 128, 41, 0), (rdm.GEMM_NT, 128, 41, rdm.EPI_MASK), (rdm.GEMM_NT, 128, 44, 0), (rdm.GEMM_NT, 128, 48, 0),
                        (rdm.GEMM_NT, 128, 64, 0), (rdm.GEMM_NN, 128, 41, 0), (rdm.GEMM_NN, 602, 128, 0), (rdm.GEMM_NT, 602, 128, 0), (rdm.GEMM_TN, 602, 128, 0), (rdm.GEMM_TN, 128, 41, 0)]:
    ldk, ldm = (k + 3) // 4 * 4, (m + 3) // 4 * 4
    if op == rdm.GEMM_NN:
        X = torch.randn(rows, ldk, device=dev); C = torch.zeros(rows, ldm, device=dev); W = torch.randn(k, m, device=dev); M = None
        f = lambda: ctx.gemm(op, X, W, C, rows, k, m, epi)
    elif op == rdm.GEMM_NT:
        X = torch.randn(rows, ldm, device=dev); C = torch.zeros(rows, ldk, device=dev); W = torch.randn(k, m, device=dev); Mk = torch.randn(rows, ldk, device=dev)
        f = lambda: ctx.gemm(op, X, W, C, rows, k, m, epi, mask=Mk if epi else None)
    else:
        X = torch.randn(rows, ldk, device=dev); U = torch.randn(rows, ldm, device=dev); C = torch.zeros(k, m, device=dev)
        f = lambda: ctx.gemm(op, X, U, C, rows, k, m)
    print(['NN','NT','TN'][op], k, m, 'epi', epi, f'{t(f):.1f} us')
# hub-core shaped GEMMs: K x K dense times K x w
for K in ():
    for w in (16, 48, 128):
        A = torch.randn(K, K, device=dev); B = torch.randn(K, w, device=dev); C = torch.zeros(K, w, device=dev)
        print('core', K, w, f'{t(lambda: ctx.gemm(rdm.GEMM_NN, A, B, C, K, K, w), 5):.1f} us')
# products-shaped
rows = 2449029
for (op, k, m) in [(rdm.GEMM_NN, 256, 256), (rdm.GEMM_NT, 256, 256), (rdm.GEMM_TN, 256, 256), (rdm.GEMM_NN, 100, 256), (rdm.GEMM_TN, 100, 256)]:
    ldk, ldm = (k + 3) // 4 * 4, (m + 3) // 4 * 4
    if op == rdm.GEMM_NN:
        X = torch.randn(rows, ldk, device=dev); C = torch.zeros(rows, ldm, device=dev); W = torch.randn(k, m, device=dev)
        f = lambda: ctx.gemm(op, X, W, C, rows, k, m)
    elif op == rdm.GEMM_NT:
        X = torch.randn(rows, ldm, device=dev); C = torch.zeros(rows, ldk, device=dev); W = torch.randn(k, m, device=dev)
        f = lambda: ctx.gemm(op, X, W, C, rows, k, m)
    else:
        X = torch.randn(rows, ldk, device=dev); U = torch.randn(rows, ldm, device=dev); C = torch.zeros(k, m, device=dev)
        f = lambda: ctx.gemm(op, X, U, C, rows, k, m)
    print('products', ['NN','NT','TN'][op], k, m, f'{t(f, 5):.1f} us')
    del X, C
