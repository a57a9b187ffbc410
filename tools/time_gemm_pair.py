"""CTA-pair GEMM diagnosis: per-call time of the Reddit-shaped 602-wide NN / NT
products, single CTA vs pair, with parts of the pipeline switched off
(RDM_TC_DBG: 1 = skip the split/convert, 2 = skip the MMAs, 4 = skip stores)."""
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm
dev = torch.device('cuda:0'); ctx = rdm.Context(device=0)
rows = 232965
def t(fn, it=10):
    fn(); ctx.sync(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it * 1e3
X = torch.randn(rows, 604, device=dev); C = torch.zeros(rows, 128, device=dev); W = torch.randn(602, 128, device=dev)
G = torch.randn(rows, 128, device=dev); D = torch.zeros(rows, 604, device=dev)
for dbg in ['0', '1', '2', '3', '4', '7']:
    res = []
    for pair in ['0', '1']:
        os.environ['RDM_PAIR'] = pair; os.environ['RDM_TC_DBG'] = dbg
        res.append(f"NN pair={pair} {t(lambda: ctx.gemm(rdm.GEMM_NN, X, W, C, rows, 602, 128)):.1f} us")
        res.append(f"NT pair={pair} {t(lambda: ctx.gemm(rdm.GEMM_NT, G, W, D, rows, 602, 128)):.1f} us")
    print('dbg', dbg, ' | '.join(res), flush=True)
