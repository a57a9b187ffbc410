"""Worker of tests/test_gpu_multirank.py — one rank of a real NCCL job.

Launched by torchrun (one process per GPU).  Every rank:
  * creates an NCCL rdm context (rdm_init with the broadcast unique id) and
    checks the communicator (rdm_comm_info: P ranks, its own rank/device);
  * for each (configuration, transport) runs one epoch (forward, backward,
    all-reduce of Y) through grouped ncclSend/ncclRecv (NCCL transport) or the
    CUDA-IPC peer-store fusion (P2P transport) and ncclAllReduce;
  * runs the same epoch in a virtual group of P ranks on its own GPU and
    requires its own slot's tensors (H^l, logits, G^0 — all computed before
    any floating-point all-reduce) to be bit-identical, and dW / loss equal to
    the virtual group's up to the all-reduce's summation order;
  * compares dW and the loss with the fp64 oracle (1e-4 / 1e-5 gates).
Writes one JSON result per rank to $RDM_MGPU_OUT/rank<r>.json.
"""
import json
import os
import sys
import traceback

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_kurtysps23_b200 as rdm
    import synth
    from oracle import gcn as og

    rank = int(os.environ["RANK"])
    world = int(os.environ["WORLD_SIZE"])
    local = int(os.environ.get("LOCAL_RANK", rank))
    out_dir = os.environ["RDM_MGPU_OUT"]
    res = {"rank": rank, "world": world, "ok": False, "checks": []}
    try:
        torch.cuda.set_device(local)
        dev = torch.device("cuda", local)
        dist.init_process_group("nccl", device_id=dev)
        obj = [rdm.get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        n, E, f = 3000, 24000, (301, 64, 13)
        g = synth.rmat(n, E, seed=5)
        H0 = synth.features(n, f[0])
        Ws = synth.weights(f)
        y = synth.labels(n, f[-1])
        m = synth.train_mask(n, 0.7, seed=3)
        ref = og.epoch(g, H0, Ws, y, m)
        stream = torch.cuda.Stream(device=dev)
        torch.cuda.set_stream(stream)
        ctx = rdm.Context(rank=rank, world=world, device=local, stream=stream, unique_id=obj[0])
        ci = ctx.comm_info()
        assert ci["ranks"] == world and ci["rank"] == rank and ci["device"] == local, ci
        res["nccl"] = ci
        ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
        vg = rdm.Context(rank=rdm.ALL_RANKS, world=world, device=local, stream=stream)
        vg.set_graph(g.rowptr, g.col, g.val, symmetric=True)
        parts = [rdm.partition(world, rdm.ROW, n, f[0], q) for q in range(world)]
        Wd = [torch.from_numpy(w.copy()).to(dev) for w in Ws]

        def run(c, cfg, transport, slots):
            c.set_transport(transport)
            model = rdm.GCN(c, list(f), cfg)
            sl = [parts[q] for q in slots]
            model.set_input([torch.from_numpy(np.ascontiguousarray(H0[lo:hi])).to(dev) for lo, hi, _ in sl],
                            [torch.from_numpy(y[lo:hi]).to(dev) for lo, hi, _ in sl],
                            [torch.from_numpy(m[lo:hi]).to(dev) for lo, hi, _ in sl])
            loss = torch.zeros(1, dtype=torch.float64, device=dev)
            dW = [torch.zeros_like(w) for w in Wd]
            c.reset_counters()
            model.forward(Wd, loss)
            model.backward(Wd, dW)
            c.sync()
            return model, float(loss.item()), [d.cpu().numpy() for d in dW], c.counters()

        def mine(model, slot, which, layer):
            for lay in (rdm.ROW, rdm.COL):
                try:
                    return model.tensor_torch(which, layer, slot, lay).cpu().numpy(), lay
                except rdm.RdmError:
                    continue
            return None, None

        for cfg in (2, 3, 5, 10, 15):
            for transport in ("nccl", "p2p"):
                mr, lr, dr, cr = run(ctx, cfg, transport, [rank])
                mv, lv, dv, cv = run(vg, cfg, transport, list(range(world)))
                for which, layer in ((rdm.T_H, 1), (rdm.T_Z, 0), (rdm.T_G, 0)):
                    a, la = mine(mr, 0, which, layer)
                    b, lb = mine(mv, rank, which, layer)
                    assert la == lb and a is not None, (cfg, transport, which, la, lb)
                    assert np.array_equal(a, b), (cfg, transport, which, "not bit-identical")
                assert abs(lr - lv) <= 1e-12 * abs(lv), (cfg, transport, lr, lv)
                assert abs(lr - ref.loss) <= 1e-5 * abs(ref.loss), (cfg, transport, lr, ref.loss)
                for l in range(len(Ws)):
                    assert og.max_rel_err(dr[l], dv[l]) < 1e-6, (cfg, transport, l)
                    assert og.max_rel_err(dr[l], ref.Y[l + 1]) < 1e-4, (cfg, transport, l)
                # NCCL rank moved exactly its share of the virtual group's payload
                assert cr["a2a_width_units"] == cv["a2a_width_units"]
                res["checks"].append({"cfg": cfg, "transport": transport, "loss": lr,
                                      "a2a_bytes_wire": cr["a2a_bytes_wire"]})
                mr.close()
                mv.close()
        tot = torch.tensor([sum(c["a2a_bytes_wire"] for c in res["checks"])], dtype=torch.float64,
                           device=dev)
        dist.all_reduce(tot)
        res["a2a_bytes_all_ranks"] = float(tot.item())
        ctx.close()
        vg.close()
        dist.barrier()
        dist.destroy_process_group()
        res["ok"] = True
    except Exception:
        res["error"] = traceback.format_exc()
    with open(os.path.join(out_dir, f"rank{rank}.json"), "w") as fh:
        json.dump(res, fh)
    return 0 if res["ok"] else 1


if __name__ == "__main__":
    sys.exit(main())
