"""Small invocations of every kernel family for compute-sanitizer (memcheck,
racecheck, synccheck): SpMM with int8 / fp16 hub tiles and the dense core,
the tcgen05 GEMM in NN / NT / TN, pack / unpack in a virtual group, loss,
Adam, and one GraphSAINT sample.  Usage:
  compute-sanitizer --tool racecheck python tools/sanitize_small.py"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_kurtysps23_b200 as rdm  # noqa: E402
import synth  # noqa: E402

dev = torch.device("cuda:0")
os.environ["RDM_TILE_MIN_NNZ"] = "1"
g = synth.rmat(4096, 40000, seed=3)
for pieces in ("8", "2"):
    os.environ["RDM_TILE_PIECES"] = pieces
    ctx = rdm.Context(device=0)
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    for w in (41, 128):
        X = torch.randn(g.n, (w + 3) // 4 * 4, device=dev)
        O = torch.zeros_like(X)
        ctx.spmm(0, X, O, w)
    ctx.sync()
    ctx.close()
    print("spmm tiles", pieces, "ok", flush=True)
os.environ.pop("RDM_TILE_MIN_NNZ")
ctx = rdm.Context(device=0)
ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
for (r, k, m) in ((1000, 64, 128), (1000, 128, 41), (700, 256, 256)):
    X = torch.randn(r, k, device=dev)
    W = torch.randn(k, m, device=dev)
    C = torch.zeros(r, (m + 3) // 4 * 4, device=dev)[:, :m]
    ctx.gemm(rdm.GEMM_NN, X, W, C, r, k, m)
    Ct = torch.zeros(r, k, device=dev)
    ctx.gemm(rdm.GEMM_NT, C, W, Ct, r, k, m)
    Y = torch.zeros(k, m, device=dev)
    ctx.gemm(rdm.GEMM_TN, X, C, Y, r, k, m)
ctx.sync()
print("gemm ok", flush=True)
# round-2 kernels: CTA-pair GEMMs (A in TMEM / smem, 256-wide), TN on pairs,
# the fast variant's kind::f16 GEMMs
for env in ({"RDM_PAIR": "1", "RDM_PAIR_ASMEM": "0"}, {"RDM_PAIR": "1", "RDM_PAIR_ASMEM": "1"},
            {"RDM_TN_PAIR": "1"}):
    os.environ.update(env)
    for (r, k, m) in ((1000, 64, 128), (1000, 128, 41), (700, 256, 256), (600, 128, 602)):
        X = torch.randn(r, k, device=dev)
        W = torch.randn(k, m, device=dev)
        C = torch.zeros(r, (m + 3) // 4 * 4, device=dev)
        ctx.gemm(rdm.GEMM_NN, X, W, C, r, k, m)
        Ct = torch.zeros(r, k, device=dev)
        ctx.gemm(rdm.GEMM_NT, C, W, Ct, r, k, m)
        Y = torch.zeros(k, m, device=dev)
        ctx.gemm(rdm.GEMM_TN, X, C, Y, r, k, m)
    ctx.sync()
    for key in env:
        os.environ.pop(key)
    print("gemm", env, "ok", flush=True)
ctx.set_precision("fast")
for (r, k, m) in ((1000, 64, 128), (1000, 128, 41), (700, 100, 256)):
    X = torch.randn(r, k + (-k) % 4, device=dev)
    W = torch.randn(k, m, device=dev)
    C = torch.zeros(r, (m + 3) // 4 * 4, device=dev)
    ctx.gemm(rdm.GEMM_NN, X, W, C, r, k, m)
    Ct = torch.zeros(r, (k + 3) // 4 * 4, device=dev)
    ctx.gemm(rdm.GEMM_NT, C, W, Ct, r, k, m)
ctx.sync()
ctx.set_precision("fp32")
print("gemm f16 ok", flush=True)
f = [70, 32, 7]
vg = rdm.Context(rank=rdm.ALL_RANKS, world=2, device=0)
vg.set_graph(g.rowptr, g.col, g.val, symmetric=True)
model = rdm.GCN(vg, f, 10)
H0 = synth.features(g.n, f[0])
y = synth.labels(g.n, f[-1])
parts = [rdm.partition(2, rdm.ROW, g.n, f[0], q) for q in range(2)]
model.set_input([torch.from_numpy(np.ascontiguousarray(H0[lo:hi])).to(dev) for lo, hi, _ in parts],
                [torch.from_numpy(y[lo:hi]).to(dev) for lo, hi, _ in parts])
Wd = [torch.from_numpy(w).to(dev) for w in synth.weights(f)]
dW = [torch.zeros_like(w) for w in Wd]
mo = [torch.zeros_like(w) for w in Wd]
ve = [torch.zeros_like(w) for w in Wd]
loss = torch.zeros(1, dtype=torch.float64, device=dev)
model.forward(Wd, loss)
model.backward(Wd, dW)
vg.adam_step(Wd, dW, mo, ve, 1)
vg.sync()
print("epoch ok", float(loss.item()), flush=True)
s = rdm.Saint(ctx, 200, walk_len=4, seed=1)
s.sample(0)
s.sample(1)
ctx.sync()
print("saint ok", flush=True)
