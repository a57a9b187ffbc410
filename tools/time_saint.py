"""GraphSAINT-RDM step timing on the Reddit-shaped graph (BASELINE config 4:
2-layer, hidden 256, ~8k-root random-walk subgraphs).  Step = sample +
induced-subgraph build + input gather + forward + backward + Adam."""
import json, sys, time
import numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth

dev = torch.device('cuda:0')
wl = synth.WORKLOADS['reddit']
f = [wl.f[0], 256, wl.f[-1]]
g = synth.make_graph(wl)
H0 = torch.from_numpy(synth.features(wl.n, f[0])).to(dev)
y = torch.from_numpy(synth.labels(wl.n, f[-1])).to(dev)
m = torch.from_numpy(synth.train_mask(wl.n).astype(np.uint8)).to(dev)
Ws = [torch.from_numpy(w).to(dev) for w in synth.weights(f)]
res = {}
for P in [int(x) for x in (sys.argv[1:] or ['1'])]:
    ctx = rdm.Context(device=0) if P == 1 else rdm.Context(rank=rdm.ALL_RANKS, world=P, device=0)
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    s = rdm.Saint(ctx, 8000, walk_len=4, seed=1)
    n0, nnz0 = s.sample(0)
    _, cfg, *_ = rdm.select_config(f, n0, nnz0, P)
    model = s.gcn(f, cfg)
    dW = [torch.zeros_like(w) for w in Ws]; mo = [torch.zeros_like(w) for w in Ws]; ve = [torch.zeros_like(w) for w in Ws]
    loss = torch.zeros(1, dtype=torch.float64, device=dev)
    sizes = []
    def step(it):
        n, nnz = s.sample(it); sizes.append((n, nnz))
        model.saint_input(H0, y, m)
        model.forward(Ws, loss); model.backward(Ws, dW)
        ctx.adam_step(Ws, dW, mo, ve, it + 1)
    for it in range(3):
        step(it)
    ctx.sync(); torch.cuda.synchronize()
    K = 40
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter(); e0.record()
    for it in range(3, 3 + K):
        step(it)
    e1.record(); torch.cuda.synchronize(); wall = (time.perf_counter() - t0) * 1e3 / K
    dev_ms = e0.elapsed_time(e1) / K
    ctx.set_timing(True); ctx.reset_phase_times()
    for it in range(100, 105):
        step(it)
    ph = {k: round(v / 5, 3) for k, v in ctx.phase_times()[0].items() if v > 0}
    ctx.set_timing(False)
    # per-call wall time with a device sync after each call (host-side gaps)
    per = {"sample": 0.0, "input": 0.0, "fwd": 0.0, "bwd": 0.0, "adam": 0.0}
    for it in range(200, 205):
        for k, fn in (("sample", lambda: s.sample(it)), ("input", lambda: model.saint_input(H0, y, m)),
                      ("fwd", lambda: model.forward(Ws, loss)), ("bwd", lambda: model.backward(Ws, dW)),
                      ("adam", lambda: ctx.adam_step(Ws, dW, mo, ve, it + 1))):
            torch.cuda.synchronize(); t = time.perf_counter(); fn(); ctx.sync(); per[k] += (time.perf_counter() - t) * 200
    ns = np.array(sizes[3:])
    r = {"P": P, "cfg": cfg, "ms_per_subgraph_event": round(dev_ms, 3), "ms_per_subgraph_wall": round(wall, 3),
         "n_sub_mean": float(ns[:, 0].mean()), "nnz_sub_mean": float(ns[:, 1].mean()),
         "subgraphs_per_epoch": float(wl.n / ns[:, 0].mean()), "phases": ph, "per_call_sync_ms": {k: round(v, 3) for k, v in per.items()}, "loss": float(loss.item())}
    print(json.dumps(r), flush=True)
    res[P] = r
    model.close(); s.close(); ctx.close()
json.dump(res, open('gpurun_out/saint_time.json', 'w'), indent=1)
