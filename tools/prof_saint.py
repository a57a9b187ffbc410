"""A few GraphSAINT steps (Reddit-shaped, config 4) for an ncu launch list."""
import sys
import numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth
dev = torch.device('cuda:0')
wl = synth.WORKLOADS['reddit']; f = [wl.f[0], 256, wl.f[-1]]
g = synth.make_graph(wl)
H0 = torch.from_numpy(synth.features(wl.n, f[0])).to(dev); y = torch.from_numpy(synth.labels(wl.n, f[-1])).to(dev)
Ws = [torch.from_numpy(w).to(dev) for w in synth.weights(f)]
ctx = rdm.Context(device=0); ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
s = rdm.Saint(ctx, 8000, walk_len=4, seed=1); model = s.gcn(f, 3)
dW = [torch.zeros_like(w) for w in Ws]; loss = torch.zeros(1, dtype=torch.float64, device=dev)
for it in range(int(sys.argv[1]) if len(sys.argv) > 1 else 3):
    s.sample(it); model.saint_input(H0, y); model.forward(Ws, loss); model.backward(Ws, dW)
ctx.sync()
