"""Virtual-group proxy for the fused (P2P) redistribution: Reddit-shaped epoch
on one GPU with P in-process ranks, transport NCCL-path (pack + copies +
unpack) vs P2P (scatter in the producer's epilogue).  Prints ms/epoch and the
per-phase split."""
import json, sys
import numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_ipps_kurtysps23_b200 as rdm, synth

dev = torch.device('cuda:0')
wl = synth.WORKLOADS[sys.argv[1] if len(sys.argv) > 1 else 'reddit']
g = synth.make_graph(wl)
H0 = synth.features(wl.n, wl.f[0]); y = synth.labels(wl.n, wl.f[-1]); msk = synth.train_mask(wl.n)
Ws = [torch.from_numpy(w).to(dev) for w in synth.weights(wl.f)]
res = []
for P in (2, 4, 8):
    _, chosen, *_ = rdm.select_config(list(wl.f), wl.n, wl.nnz, P)
    for cfg in sorted({chosen, 10}):
        for tr in ("nccl", "p2p"):
            ctx = rdm.Context(rank=rdm.ALL_RANKS, world=P, device=0)
            ctx.set_transport(tr)
            ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
            m = rdm.GCN(ctx, wl.f, cfg)
            Hs, ys, ms = [], [], []
            for p in range(P):
                lo, hi, _ = rdm.partition(P, rdm.ROW, wl.n, wl.f[0], p)
                Hs.append(torch.from_numpy(H0[lo:hi]).to(dev)); ys.append(torch.from_numpy(y[lo:hi]).to(dev))
                ms.append(torch.from_numpy(msk[lo:hi]).to(dev))
            m.set_input(Hs, ys, ms)
            dW = [torch.zeros_like(w) for w in Ws]
            loss = torch.zeros(1, dtype=torch.float64, device=dev)
            for _ in range(3):
                m.forward(Ws, loss); m.backward(Ws, dW)
            ctx.sync()
            s0 = torch.cuda.Event(enable_timing=True); s1 = torch.cuda.Event(enable_timing=True)
            s0.record()
            K = 10
            for _ in range(K):
                m.forward(Ws, loss); m.backward(Ws, dW)
            s1.record(); torch.cuda.synchronize()
            ms_ep = s0.elapsed_time(s1) / K
            ctx.set_timing(True); ctx.reset_phase_times()
            for _ in range(3):
                m.forward(Ws, loss); m.backward(Ws, dW)
            ph = {k: v / 3 for k, v in ctx.phase_times()[0].items()}
            ctx.set_timing(False)
            ctx.reset_counters()
            m.forward(Ws, loss); m.backward(Ws, dW); ctx.sync()
            c = ctx.counters()
            info = m.info()
            r = {"P": P, "cfg": cfg, "transport": tr, "ms": round(ms_ep, 3), "loss": float(loss.item()),
                 "phases": {k: round(v, 3) for k, v in ph.items() if v > 0},
                 "a2a_elems_per_epoch": c["a2a_elems_payload"], "model_comm_units": info["model_comm_units"],
                 "a2a_elems_over_NxUnits": c["a2a_elems_payload"] / (wl.n * max(1, info["model_comm_units"])),
                 "per_rank_elems": c["a2a_elems_payload"] / P}
            print(json.dumps(r), flush=True)
            res.append(r)
            m.close(); ctx.close()
json.dump(res, open('gpurun_out/p2p_virtual.json', 'w'), indent=1)
