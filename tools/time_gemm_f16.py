"""Fast-variant GEMM per-call times, kind::f16 (bf16) vs 1xTF32, over K for the
products-shaped rows (the NN 100 -> 256 call regressed with bf16)."""
import os, sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm
dev = torch.device('cuda:0'); ctx = rdm.Context(device=0); ctx.set_precision('fast')
def t(fn, it=5):
    fn(); ctx.sync(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it * 1e3
rows = 2449029
for (k, m) in [(32, 256), (64, 256), (100, 256), (128, 256), (256, 256), (100, 128), (256, 100), (256, 47)]:
    X = torch.randn(rows, (k + 3) // 4 * 4, device=dev); C = torch.zeros(rows, (m + 3) // 4 * 4, device=dev); W = torch.randn(k, m, device=dev)
    res = []
    for f in ['0', '1']:
        os.environ['RDM_F16_GEMM'] = f
        res.append(f"f16={f} {t(lambda: ctx.gemm(rdm.GEMM_NN, X, W, C, rows, k, m)):.1f} us")
    print(f"NN k={k} m={m}", ' | '.join(res), flush=True)
    del X, C
