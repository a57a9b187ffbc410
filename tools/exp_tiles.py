"""Experiment: binary hub tiles (hubtiles.cu) vs the fp32 dense hub core vs
plain CSR on the Reddit-/products-shaped graph: SpMM time per call at several
widths and tile-selection thresholds (CUDA events, 5 calls after 1 warm-up)."""
import os, sys, time, json, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wl = synth.WORKLOADS[sys.argv[1] if len(sys.argv) > 1 else 'reddit']
g = synth.make_graph(wl)
widths = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else '128,48,16').split(',')]
settings = sys.argv[3].split(',') if len(sys.argv) > 3 else ['csr', 'dense', '200', '400', '800', '1600']
def timeit(fn, it=5):
    fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
ref = {}
for st in settings:
    for k in ('RDM_NO_TILES', 'RDM_NO_CORE', 'RDM_TILE_MIN_NNZ'):
        os.environ.pop(k, None)
    if st == 'csr':
        os.environ['RDM_NO_CORE'] = '1'
    elif st == 'dense':
        os.environ['RDM_NO_TILES'] = '1'
    elif st != 'auto':
        os.environ['RDM_TILE_MIN_NNZ'] = st
    ctx = rdm.Context(device=0)
    t0 = time.time(); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True); tset = time.time() - t0
    gi = ctx.graph_info()
    line = [f"{st:>6}: set {tset:5.1f}s tiles {gi['n_tiles']:6d} items {gi['n_tile_items']:5d} ranks {gi['tile_ranks']:7d} "
            f"moved {gi['core_nnz']/g.nnz:.3f} K {gi['core_K']}"]
    for w in widths:
        torch.manual_seed(w)
        X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev); O = torch.zeros_like(X)
        ms = timeit(lambda: ctx.spmm(0, X, O, w))
        if w not in ref:
            ref[w] = O.clone()
            err = 0.0
        else:
            err = float((O[:, :w] - ref[w][:, :w]).abs().max() / ref[w][:, :w].abs().max())
        line.append(f"w{w}: {ms:.3f} ms (diff {err:.1e})")
    print(' | '.join(line), flush=True)
    del ctx
    torch.cuda.empty_cache()
