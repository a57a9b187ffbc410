"""Diagnose GraphSAINT step-time variance: host time of each sample() call and
of each step (training enqueue + next sample), 40 steps, no clock sampler."""
import sys, time, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wl = synth.WORKLOADS['reddit']
g = synth.make_graph(wl)
f = [wl.f[0], 256, wl.f[-1]]
H0 = synth.features(wl.n, f[0]); y = synth.labels(wl.n, f[-1]); msk = synth.train_mask(wl.n)
stream = torch.cuda.Stream(device=dev); torch.cuda.set_stream(stream)
ctx = rdm.Context(device=0, stream=stream)
ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
Hd = torch.from_numpy(H0).to(dev); yd = torch.from_numpy(y).to(dev); md = torch.from_numpy(msk.astype(np.uint8)).to(dev)
Wd = [torch.from_numpy(w).to(dev) for w in synth.weights(f)]
dW = [torch.zeros_like(w) for w in Wd]; mo = [torch.zeros_like(w) for w in Wd]; ve = [torch.zeros_like(w) for w in Wd]
loss = torch.zeros(1, dtype=torch.float64, device=dev)
sam = rdm.Saint(ctx, 8000, walk_len=4, seed=1)
n0, nnz0 = sam.sample(0)
_, cfg, *_ = rdm.select_config(f, n0, nnz0, 1)
model = sam.gcn(f, cfg)
it = 0
rows = []
ctx.set_timing(len(sys.argv) > 1)
for step in range(60):
    t0 = time.perf_counter()
    model.saint_input(Hd, yd, md); model.forward(Wd, loss); model.backward(Wd, dW)
    it += 1
    ctx.adam_step(Wd, dW, mo, ve, it, lr=0.01)
    t1 = time.perf_counter()
    n, nnz = sam.sample(it)
    t2 = time.perf_counter()
    rows.append((step, (t1 - t0) * 1e3, (t2 - t1) * 1e3, n, nnz))
torch.cuda.synchronize()
for r in rows:
    print("step %2d enqueue %.2f ms  sample %.2f ms  n %d nnz %d" % r)
