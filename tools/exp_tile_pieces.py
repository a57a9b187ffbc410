"""Experiment: SpMM time per call (hub tiles + residual CSR) for the tile
piece forms — int8 digits on kind::i8 (8), fp16 pair (2), bf16 triple (3) —
at several tile-selection thresholds, with the error against the CSR-only
product.  Usage: python tools/exp_tile_pieces.py <workload> <widths> <pieces,..> <thresholds,..|auto>"""
import os, sys, time, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wl = synth.WORKLOADS[sys.argv[1]]
g = synth.make_graph(wl)
widths = [int(x) for x in sys.argv[2].split(',')]
pieces = sys.argv[3].split(',')
thr = sys.argv[4].split(',')
def timeit(fn, it=5):
    fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
Xs = {w: torch.randn(g.n, (w + 3) // 4 * 4, device=dev, generator=torch.Generator(device=dev).manual_seed(w)) for w in widths}
os.environ['RDM_NO_CORE'] = '1'
ctx = rdm.Context(device=0)
ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
ref = {}
for w in widths:
    O = torch.zeros_like(Xs[w]); ms = timeit(lambda: ctx.spmm(0, Xs[w], O, w)); ref[w] = O.clone()
    print(f"csr-only w{w}: {ms:.3f} ms", flush=True)
del ctx
os.environ.pop('RDM_NO_CORE')
for t in thr:
    if t == 'auto':
        os.environ.pop('RDM_TILE_MIN_NNZ', None)
    else:
        os.environ['RDM_TILE_MIN_NNZ'] = t
    ctx = rdm.Context(device=0)
    t0 = time.time(); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True); ts = time.time() - t0
    gi = ctx.graph_info()
    for p in pieces:
        os.environ['RDM_TILE_PIECES'] = p
        line = [f"thr {t:>5} pieces {p}: set {ts:.1f}s tiles {gi['n_tiles']} moved {gi['core_nnz'] / g.nnz:.3f}"]
        for w in widths:
            O = torch.zeros_like(Xs[w])
            ms = timeit(lambda: ctx.spmm(0, Xs[w], O, w))
            err = float((O[:, :w] - ref[w][:, :w]).abs().max() / ref[w][:, :w].abs().max())
            line.append(f"w{w}: {ms:.3f} ms (err {err:.1e})")
        print(' | '.join(line), flush=True)
    del ctx
    torch.cuda.empty_cache()
