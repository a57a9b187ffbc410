"""Experiment: column relabelling of DRAM-resident SpMM slices (spmm.cu Hot /
rank_panel) — per-call time with the relabelled column stream (input gathered
into rank order) vs the plain one (RDM_RELABEL=0), for several lane mappings.
Usage: python tools/exp_relabel.py <workload> <widths> <G,V,U;...|auto> [P]
P > 1: an emulated rank 0 of P (rdm_init_emulated) — the column slice width is
the given width (one rank's share)."""
import os, sys, time, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wl = synth.WORKLOADS[sys.argv[1]]
t0 = time.time(); g = synth.make_graph(wl); print(f"gen {time.time() - t0:.1f}s", flush=True)
widths = [int(x) for x in sys.argv[2].split(',')]
combos = sys.argv[3].split(';')
P = int(sys.argv[4]) if len(sys.argv) > 4 else 1
ctx = rdm.Context(rank=0, world=P, device=0, emulate=True) if P > 1 else rdm.Context(device=0)
t0 = time.time(); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=synth.symmetric_values(wl))
print(f"set_graph {time.time() - t0:.1f}s", ctx.graph_info(), flush=True)
n = g.n
del g
def timeit(fn, it=3):
    fn(); torch.cuda.synchronize(); s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); [fn() for _ in range(it)]; e.record(); torch.cuda.synchronize(); return s.elapsed_time(e) / it
for w in widths:
    X = torch.randn(n, (w + 3) // 4 * 4, device=dev, generator=torch.Generator(device=dev).manual_seed(w))
    ref = None
    for rl in ('0', '1'):
        os.environ['RDM_RELABEL'] = rl
        line = [f"w{w} relabel {rl}"]
        for cb in combos:
            for k in ('RDM_SPMM_GV', 'RDM_SPMM_U'):
                os.environ.pop(k, None)
            if cb != 'auto':
                G, V, U = cb.split(',')
                os.environ['RDM_SPMM_GV'] = f'{G},{V}'
                os.environ['RDM_SPMM_U'] = U
            O = torch.zeros_like(X)
            try:
                ms = timeit(lambda: ctx.spmm(0, X, O, w))
            except Exception as ex:
                line.append(f"{cb}: ERR"); continue
            if ref is None:
                ref = O.clone(); err = 0.0
            else:
                err = float((O[:, :w] - ref[:, :w]).abs().max() / ref[:, :w].abs().max())
            line.append(f"{cb}: {ms:.3f}" + ("" if err < 1e-6 else f" BAD {err:.1e}"))
        print(" | ".join(line), flush=True)
    del X
    torch.cuda.empty_cache()
