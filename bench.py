#!/usr/bin/env python
"""Benchmark: full-batch GCN epoch of the GNN-RDM hot path on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload reddit]
                    [--impl rdm|reference] [--config auto|ID]

One "step" = one full-batch epoch: forward (all layers) + loss + backward +
weight-gradient all-reduce + Adam, on a synthetic
graph shaped like BASELINE.json's configs[1] (Reddit-shaped, N = 232,965,
nnz = 114,848,857, f = 602/128/41) by default.  N > 1 runs one rank per GPU
under torchrun (NCCL), strong scaling (the graph is fixed).

Prints ONE JSON line on rank 0 (contract in the task statement): value =
epoch ms (max over ranks, CUDA events on the library's stream), plus e2e,
roofline (dominant kernel: SpMM), cpu_baseline (the fp64 oracle on a bounded
row sample, timed on this host), clocks, gpu_launches, per-phase split.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "full-batch GCN epoch ms at 1/2/4/8 B200; SpMM HBM GB/s; all-to-all bus GB/s"
DTYPES = {"fp32": "f32", "fast": "bf16 SpMM operand + bf16 (kind::f16) NN/NT GEMM, tf32 TN, f32 accumulate"}
GATES = {"fp32": 1e-4, "fast": 2e-2}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--workload", default="reddit")
    ap.add_argument("--impl", default="rdm", choices=["rdm", "reference"])
    ap.add_argument("--config", default="auto")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--emulate", type=int, default=0,
                    help="one-rank emulation of a P-rank job on one GPU (rdm_init_emulated); "
                         "default workload papers (BASELINE configs[4]) at P = 8")
    ap.add_argument("--emulate-rank", type=int, default=0)
    ap.add_argument("--emulate-check", type=int, default=1,
                    help="--emulate: per-op parity on 4,096 sampled rows against the fp64 oracle")
    ap.add_argument("--threads", type=int, default=0,
                    help="--impl reference: oracle threads (default nproc)")
    ap.add_argument("--ref-budget-s", type=float, default=150.0,
                    help="--impl reference: stop after this many seconds of whole epochs (>= 1 epoch)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--transport", default="nccl", choices=["nccl", "p2p"],
                    help="redistribution transport for N > 1 (rdm.h rdm_set_transport)")
    ap.add_argument("--precision", default="fp32", choices=["fp32", "fast"],
                    help="operator arithmetic (rdm.h rdm_set_precision): fp32 (1e-4 gate) or fast "
                         "(bf16 SpMM operand + 1xTF32 GEMM, 2e-2 gate)")
    ap.add_argument("--ra", type=int, default=0,
                    help="R_A < P partial replication (rdm.h rdm_set_graph_panels): replicas of A; "
                         "0 = full replication (R_A = P)")
    ap.add_argument("--no-variants", action="store_true",
                    help="skip the extra timing of the fast-precision variant")
    ap.add_argument("--saint", action="store_true",
                    help="GraphSAINT-RDM (BASELINE configs[3]): step = one sampled subgraph")
    ap.add_argument("--roots", type=int, default=8000)
    ap.add_argument("--walk-len", type=int, default=4)
    ap.add_argument("--hidden", type=int, default=0, help="override the hidden width (saint: 256)")
    ap.add_argument("--sweep", action="store_true",
                    help="also time every configuration (Table VIII analogue) into config.sweep_ms")
    return ap.parse_args()


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled DURING the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device = device
        self.proc = None
        self.lines = []

    def start(self):
        if os.environ.get("RDM_BENCH_NO_CLOCKS"):   # diagnosis only: no clock record
            return
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                 "-lms", "200", "-i", str(self.device)],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def ready(self):
        """True once nvidia-smi has produced its first sample (its start-up
        NVML initialisation stalls host-side CUDA calls for up to ~100 ms:
        it must not land inside the timed region)."""
        return self.proc is None or len(self.lines) > 0

    def stop(self):
        if not self.proc:
            return None
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx = max(mx, float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        if not sm:
            return None
        sm.sort()
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


# --------------------------------------------------------------- oracle leg
def graph_desc(wl):
    """The input recipe of a workload's graph."""
    g = "R-MAT (0.57,0.19,0.19,0.05)" if wl.graph == "rmat" else "uniform (Erdos-Renyi)"
    g += ", permuted" if wl.permute else ", un-permuted (R-MAT order)"
    v = {"sym": "D^-1/2 (A+I) D^-1/2", "row": "D^-1 (A+I) (not symmetric)",
         "noise": "D^-1/2 (A+I) D^-1/2 x (1 + u_ij/16), u symmetric (not a rank-1 scaling)"}[wl.values]
    return g + ", symmetric pattern, self loops, " + v


def host_cpu_info():
    """lscpu model / sockets / cores of the host the oracle runs on."""
    info = {"nproc": os.cpu_count()}
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            k, _, v = ln.partition(":")
            k, v = k.strip(), v.strip()
            if k == "Model name":
                info["model"] = v
            elif k == "Socket(s)":
                info["sockets"] = int(v)
            elif k == "Core(s) per socket":
                info["cores_per_socket"] = int(v)
            elif k == "Thread(s) per core":
                info["threads_per_core"] = int(v)
    except Exception:
        pass
    return info


def oracle_set_threads(n):
    """OpenMP threads of oracle/spmm.c and BLAS threads of numpy's fp64 matmul."""
    from oracle import lib as olib
    olib().oracle_set_threads(int(n))
    try:
        from threadpoolctl import threadpool_limits
        return threadpool_limits(limits=int(n))
    except Exception:
        return None


def oracle_full_epoch_ms(g, H0, Ws, y, msk):
    """ONE whole fp64 oracle epoch as it stands (oracle/gcn.py: forward of every
    layer, loss, backward with G^0, Adam on every W) — wall clock, not scaled."""
    import numpy as np
    from oracle import gcn as og
    t0 = time.perf_counter()
    r = og.epoch(g, H0, Ws, y, msk)
    for l in range(len(Ws)):
        og.adam(Ws[l], r.Y[l + 1], np.zeros_like(r.Y[l + 1]), np.zeros_like(r.Y[l + 1]), 1)
    return (time.perf_counter() - t0) * 1e3


def oracle_saint_step_ms(g, H0, y, msk, Ws, roots, walk_len, seed, it):
    """The oracle (oracle/saint.py + oracle/gcn.py, as they stand) on ONE whole
    GraphSAINT step: sample + induced subgraph + fp64 epoch on it."""
    from oracle import gcn as og
    from oracle import lib as olib
    from oracle import saint as osaint
    t0 = time.perf_counter()
    nodes, rp, cs, vs = osaint.sample(g, roots, walk_len, seed, it)
    import synth
    sub = synth.CSR(len(nodes), rp, cs, vs)
    og.epoch(sub, H0[nodes], Ws, y[nodes], msk[nodes])
    dt = time.perf_counter() - t0
    desc = (f"one whole subgraph step (iteration {it}: {len(nodes)} vertices, {len(cs)} entries): "
            f"oracle sampler + induced subgraph + fp64 epoch, {dt:.1f} s CPU wall")
    return dt * 1e3, desc, olib().oracle_num_threads()


def saint_main(a, world, rank, local_rank):
    """GraphSAINT-RDM (§III-F, §V-C; BASELINE configs[3]): every step
    samples one subgraph (same seed on every rank), builds it, gathers its input
    and runs forward + backward + all-reduce + Adam on it with RDM."""
    import numpy as np
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_kurtysps23_b200 as rdm
    import synth
    wl = synth.WORKLOADS[a.workload]
    f = [wl.f[0], a.hidden or 256] + [wl.f[-1]] if wl.L == 2 else list(wl.f)
    metric = "GraphSAINT-RDM ms per subgraph step (sample + build + fwd + bwd + Adam)"
    # BASELINE configs[3]: GraphSAINT on the Reddit-shaped graph, 2 layers, hidden 256
    saint_name = f"{wl.name.split(' ')[0]} GraphSAINT-RDM {len(f) - 1}L h{f[1]} (BASELINE configs[3])"
    g = synth.make_graph(wl)
    H0 = synth.features(wl.n, f[0])
    y = synth.labels(wl.n, f[-1])
    msk = synth.train_mask(wl.n)
    Ws_h = synth.weights(f)
    if a.impl == "reference":
        if rank != 0:
            return
        times, desc, cores = [], None, None
        for k in range(max(1, min(a.steps, 3))):
            ms, desc, cores = oracle_saint_step_ms(g, H0, y, msk, Ws_h, a.roots, a.walk_len, 1, k)
            times.append(ms)
        v = float(np.mean(times))
        print(json.dumps({"metric": metric, "value": v, "unit": "ms", "impl": "reference",
                          "n_gpus": a.gpus, "steps": len(times), "warmup": 0, "ms_per_step": v,
                          "higher_is_better": False, "scaling": "strong", "vs_baseline": None,
                          "dtype": "f64", "data": "synthetic",
                          "config": {"workload": saint_name, "f": f, "roots": a.roots,
                                     "walk_len": a.walk_len},
                          "cpu_baseline": {"value": v, "unit": "ms", "cores": cores, "kind": "oracle",
                                           "sample": desc},
                          "e2e": {"value": v, "unit": "ms", "h2d_bytes_per_step": 0,
                                  "d2h_bytes_per_step": 0}}), flush=True)
        return
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    uid = None
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
        obj = [rdm.get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]
    stream = torch.cuda.Stream(device=dev)
    torch.cuda.set_stream(stream)
    ctx = rdm.Context(rank=rank if world > 1 else 0, world=world, device=local_rank, stream=stream,
                      unique_id=uid)
    ctx.set_transport(a.transport)
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=True)
    Hd = torch.from_numpy(H0).to(dev)
    yd = torch.from_numpy(y).to(dev)
    md = torch.from_numpy(msk.astype(np.uint8)).to(dev)
    Wd = [torch.from_numpy(w).to(dev) for w in Ws_h]
    dW = [torch.zeros_like(w) for w in Wd]
    mo = [torch.zeros_like(w) for w in Wd]
    ve = [torch.zeros_like(w) for w in Wd]
    loss = torch.zeros(1, dtype=torch.float64, device=dev)
    sam = rdm.Saint(ctx, a.roots, walk_len=a.walk_len, seed=1)
    n0, nnz0 = sam.sample(0)
    pareto, cfg_id, *_ = rdm.select_config(f, n0, nnz0, world)
    model = sam.gcn(f, cfg_id)
    it = [0]
    sizes = []

    cur = [(n0, nnz0)]

    def step():
        # train on the sampled subgraph (enqueued, asynchronous), then build the
        # next one on the sampler's stream while the GPU trains (rdm_saint_sample
        # double-buffers its subgraphs)
        sizes.append(cur[0])
        model.saint_input(Hd, yd, md)
        model.forward(Wd, loss)
        model.backward(Wd, dW)
        it[0] += 1
        ctx.adam_step(Wd, dW, mo, ve, it[0], lr=0.01)
        cur[0] = sam.sample(it[0])

    # the clock sampler starts during the warm-up (no idle gap before the timed
    # steps: after an idle pause the first host-synchronised sampler steps ran
    # several times slower)
    clk = ClockSampler(local_rank)
    clk.start()
    for _ in range(max(3, a.warmup)):
        step()
    # keep warming up until the clock sampler is past its start-up (a one-off
    # 10-100 ms stall of the host-synchronised sampler steps otherwise hit the
    # 4th timed step)
    t_w = time.time()
    while not clk.ready() and time.time() - t_w < 5.0:
        step()
    ctx.sync()
    sizes.clear()
    ctx.reset_counters()
    ctx.reset_phase_times()
    ctx.set_timing(True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    if os.environ.get("RDM_WS_LOG"):
        print("[bench] timed region start", file=sys.stderr, flush=True)
    e0.record(stream)
    # per-step marks on the compute stream (no host sync): the step-time
    # distribution shows whether a slow run is a few slow steps or all of them
    marks = []
    for _ in range(a.steps):
        step()
        ev = torch.cuda.Event(enable_timing=True)
        ev.record(stream)
        marks.append(ev)
    sam.wait()   # the last step's subgraph build (sampler stream) inside the bracket
    e1.record(stream)
    torch.cuda.synchronize(dev)
    clocks = clk.stop()
    ms_total = e0.elapsed_time(e1)
    step_ms = [e0.elapsed_time(marks[0])] + [marks[i - 1].elapsed_time(marks[i]) for i in range(1, len(marks))]
    cnt = ctx.counters()
    ph_ms, _ = ctx.phase_times()
    ctx.set_timing(False)
    if world > 1:
        t = torch.tensor([ms_total], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_total = float(t.item())
    ms_step = ms_total / a.steps
    # e2e: the user's loop through the public API, wall clock, loss read back every step
    loss_host = torch.zeros(1, dtype=torch.float64).pin_memory()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    k2 = max(3, a.steps // 2)
    t0 = time.perf_counter()
    for _ in range(k2):
        step()
        loss_host.copy_(loss, non_blocking=True)
    torch.cuda.synchronize(dev)
    e_ms = (time.perf_counter() - t0) * 1e3 / k2
    if world > 1:
        t = torch.tensor([e_ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e_ms = float(t.item())
    # roofline of the dominant kernel (SpMM) over the timed steps
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0))
    calls_ps = cnt["spmm_calls"] / a.steps
    w_ps = cnt["spmm_width_units"] / a.steps / max(1, world)   # per-rank Σ w per step
    alg = sum(calls_ps * (8 * nz + 8 * (nv + 1)) + 8 * nv * w_ps for nv, nz in sizes[:a.steps])
    spmm_s = ph_ms["spmm"] / 1e3
    achieved = alg / spmm_s / 1e9 if spmm_s > 0 else 0.0
    ns = np.array(sizes[:a.steps], dtype=np.float64)
    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        ms, desc, cores = oracle_saint_step_ms(g, H0, y, msk, Ws_h, a.roots, a.walk_len, 1, 0)
        cpu = {"value": ms, "unit": "ms", "cores": cores, "kind": "oracle", "sample": desc}
    if rank == 0:
        print(json.dumps({
            "metric": metric, "value": ms_step, "unit": "ms", "n_gpus": world, "steps": a.steps,
            "warmup": max(3, a.warmup), "ms_per_step": ms_step, "higher_is_better": False,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": saint_name, "model": f"GCN 2L f={'/'.join(map(str, f))}",
                       "sampler": f"random walk, {a.roots} roots, length {a.walk_len} (readings R31-R34)",
                       "n_sub_mean": float(ns[:, 0].mean()), "nnz_sub_mean": float(ns[:, 1].mean()),
                       "config_id": cfg_id, "pareto": pareto, "transport": a.transport,
                       "parallelism": f"rdm{world} per subgraph, one Adam step per subgraph (L390)",
                       "l2": "CSR of the full graph streamed by the sampler each step (0.92 GB)"},
            "clocks": clocks,
            "step_ms": {"median": float(np.median(step_ms)), "min": float(np.min(step_ms)),
                        "max": float(np.max(step_ms)), "p90": float(np.percentile(step_ms, 90)),
                        "all": [round(float(x), 3) for x in step_ms]},
            "e2e": {"value": e_ms, "unit": "ms", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 8,
                    "note": "wall clock of the public-API loop; features resident on the device, "
                            "the per-step input is the sampler seed"},
            "gpu_launches": cnt["kernel_launches"],
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": hbm_peak, "unit": "GB/s",
                         "frac": achieved / hbm_peak, "traffic": None,
                         "kernel": "spmm on the subgraphs",
                         "spmm_share_of_step": ph_ms["spmm"] / max(1e-9, ms_total)},
            "cpu_baseline": cpu,
            "phases_ms_per_step": {k: v / a.steps for k, v in ph_ms.items()},
            "phases_note": "sample = subgraph build on the sampler stream, overlapped with the "
                           "previous subgraph's training: the phases add up to more than the step",
            "loss": float(loss.item())}), flush=True)
    ctx.sync()
    model.close()
    sam.close()
    ctx.close()
    if world > 1:
        dist.destroy_process_group()


def emulate_main(a):
    """One-rank emulation of a P-rank job on one GPU (rdm.h rdm_init_emulated):
    rank `--emulate-rank` of P = --emulate holds exactly its partitions and runs
    exactly its SpMMs, GEMMs, pack/unpack, loss and Adam at the P-rank shapes;
    exchanges and all-reduces are skipped (nothing crosses a link).  Default
    workload: BASELINE configs[4], papers100M-shaped 2L h128 at P = 8, with the
    liveness-based workspace (RDM_GCN_LOW_MEMORY).  The line reports the rank's
    compute epoch (device time), its per-phase split, the SpMM roofline, and the
    exchange volume a real rank would move with the time it would take at the
    NVLink peer bandwidth B200_PROFILING.md records for this pool (770 GB/s per
    direction; not measured by this build)."""
    import numpy as np
    import torch
    import paper_conf_ipps_kurtysps23_b200 as rdm
    import synth
    P, p = a.emulate, a.emulate_rank
    wl = synth.WORKLOADS[a.workload]
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    stream = torch.cuda.Stream(device=dev)
    torch.cuda.set_stream(stream)
    t0 = time.time()
    g = synth.make_graph(wl)
    t_gen = time.time() - t0
    lo, hi, _ = rdm.partition(P, rdm.ROW, wl.n, wl.f[0], p)
    H0 = torch.from_numpy(synth.features_rows(lo, hi, wl.f[0])).to(dev)
    y = torch.from_numpy(synth.labels_rows(lo, hi, wl.f[-1])).to(dev)
    m = torch.ones(hi - lo, dtype=torch.uint8, device=dev)
    Wd = [torch.from_numpy(w).to(dev) for w in synth.weights(wl.f)]
    dW = [torch.zeros_like(w) for w in Wd]
    mom = [torch.zeros_like(w) for w in Wd]
    vel = [torch.zeros_like(w) for w in Wd]
    loss = torch.zeros(1, dtype=torch.float64, device=dev)
    ctx = rdm.Context(rank=p, world=P, device=0, stream=stream, emulate=True)
    ctx.set_precision(a.precision)
    t0 = time.time()
    ctx.set_graph(g.rowptr, g.col, g.val, symmetric=synth.symmetric_values(wl))
    t_set = time.time() - t0
    ginfo = ctx.graph_info()
    pareto, chosen, _, _ = rdm.select_config(list(wl.f), wl.n, wl.nnz, P)
    cfg = chosen if a.config == "auto" else int(a.config)
    # per-op parity at these full sizes, in this launch configuration (SURVEY
    # §8(c) "per-op on sampled rows"): the rank's SpMM on a seeded column
    # slice of width w_p and its NN GEMM on its row slice, against the fp64
    # oracle on 4,096 sampled output rows
    parity = None
    if a.emulate_check:
        from oracle import gcn as og
        rng = np.random.default_rng(11)
        n_all = wl.n
        c0, c1, ldc = rdm.partition(P, rdm.COL, n_all, wl.f[1], p)
        wp = c1 - c0
        Xc = torch.zeros(n_all, ldc, device=dev)
        Xc[:, :wp] = torch.from_numpy(synth.features(n_all, wp, seed=12)).to(dev)
        Oc = torch.zeros_like(Xc)
        ctx.spmm(1, Xc, Oc, wp)
        ctx.sync()
        rows = np.sort(rng.choice(n_all, size=4096, replace=False))
        ref = og.spmm_rows(g, Xc[:, :wp].cpu().numpy(), rows)
        e_sp = og.max_rel_err(Oc[rows][:, :wp].cpu().numpy(), ref)
        del Xc, Oc
        Tr = torch.zeros(hi - lo, wl.f[1], device=dev)
        ctx.gemm(rdm.GEMM_NN, H0, Wd[0], Tr, hi - lo, wl.f[0], wl.f[1])
        ctx.sync()
        rr = np.sort(rng.choice(hi - lo, size=4096, replace=False))
        e_gm = og.max_rel_err(Tr[rr].cpu().numpy(),
                              H0[rr].cpu().numpy().astype(np.float64) @ Wd[0].cpu().numpy().astype(np.float64))
        del Tr
        parity = {"spmm_w": wp, "spmm_rows_checked": 4096, "spmm_max_rel_err": e_sp,
                  "gemm_nn_rows_checked": 4096, "gemm_nn_max_rel_err": e_gm, "gate": 1e-4,
                  "pass": bool(e_sp < 1e-4 and e_gm < 1e-4)}
    model = rdm.GCN(ctx, wl.f, cfg, low_memory=True)
    info = model.info()
    model.set_input([H0], [y], [m])
    del g
    step = [0]

    def epoch():
        model.forward(Wd, loss)
        model.backward(Wd, dW)
        step[0] += 1
        ctx.adam_step(Wd, dW, mom, vel, step[0], lr=0.01)

    for _ in range(max(3, a.warmup)):
        epoch()
    ctx.sync()
    ctx.reset_counters()
    ctx.reset_phase_times()
    ctx.set_timing(True)
    clk = ClockSampler(0)
    clk.start()
    time.sleep(0.3)
    t_w = time.time()
    while not clk.ready() and time.time() - t_w < 5.0:
        time.sleep(0.05)
    torch.cuda.synchronize(dev)
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(a.steps):
        epoch()
    e1.record(stream)
    torch.cuda.synchronize(dev)
    clocks = clk.stop()
    ms = e0.elapsed_time(e1) / a.steps
    cnt = ctx.counters()
    ph_ms, _ = ctx.phase_times()
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0))
    n, nnz = wl.n, wl.nnz
    calls = cnt["spmm_calls"]
    sum_w = cnt["spmm_nnz_cols"] / max(1, nnz)          # Σ w_p over the rank's SpMM calls
    alg = calls * (8 * nnz + 8 * (n + 1)) + 8 * n * sum_w
    spmm_s = ph_ms["spmm"] / 1e3
    achieved = alg / spmm_s / 1e9 if spmm_s > 0 else 0.0
    nvlink = 770.0
    a2a_ms = cnt["a2a_bytes_wire"] / a.steps / (nvlink * 1e9) * 1e3
    line = {
        "metric": METRIC, "impl": "rdm-emulated-rank", "value": ms, "unit": "ms",
        "n_gpus": 1, "emulated_world": P, "emulated_rank": p, "steps": a.steps,
        "warmup": max(3, a.warmup), "ms_per_step": ms, "higher_is_better": False,
        "scaling": "strong", "vs_baseline": None, "dtype": DTYPES[a.precision], "data": "synthetic",
        "config": {"workload": wl.name + f" (one-rank emulation of P = {P}, BASELINE configs[4])",
                   "model": f"GCN {wl.L}L f={'/'.join(map(str, wl.f))}", "n": n, "nnz": nnz,
                   "config_id": cfg, "config_name": rdm.config_name(model.cfg), "pareto": pareto,
                   "row_slice": [lo, hi], "low_memory": True,
                   "workspace_gb": info["workspace_bytes"] / 1e9,
                   "graph_gb": (8 * nnz + 8 * (n + 1)) / 1e9,
                   "device_mem_peak_gb": torch.cuda.max_memory_allocated(dev) / 1e9,
                   "device_mem_used_gb": (torch.cuda.mem_get_info(dev)[1] - torch.cuda.mem_get_info(dev)[0]) / 1e9,
                   "hub_tiles": ginfo.get("n_tiles", 0), "core_K": ginfo.get("core_K", 0),
                   "gen_s": round(t_gen, 1), "set_graph_s": round(t_set, 1),
                   "l2": "inputs larger than L2 (13.7 GB CSR streamed per SpMM)"},
        "what_is_timed": "this rank's compute only: SpMMs, GEMMs, pack/unpack, loss, Adam; no exchange",
        "clocks": clocks, "gpu_launches": cnt["kernel_launches"],
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": hbm_peak, "unit": "GB/s",
                     "frac": achieved / hbm_peak, "traffic": None,
                     "algorithmic_gb_per_call": alg / max(1, calls) / 1e9,
                     "avg_call_ms": ph_ms["spmm"] / a.steps / max(1, calls / a.steps),
                     "kernel": "spmm call on the rank's column slice (w = f/P)",
                     "peak_source": "MEASURED_PEAKS.json hbm_gbs (measured copy)"},
        "phases_ms_per_step": {k: v / a.steps for k, v in ph_ms.items()},
        "exchange": {"bytes_per_step": cnt["a2a_bytes_wire"] / a.steps,
                     "modelled_ms_at_770_gbs": a2a_ms,
                     "epoch_ms_compute_plus_modelled_exchange": ms + a2a_ms,
                     "note": "770 GB/s per direction = B200_PROFILING.md's measured peer copy on this "
                             "pool (not measured by this build); no overlap assumed"},
        "plan": {"model_comm_units": info["model_comm_units"],
                 "model_sparse_units": info["model_sparse_units"]},
        "parity": parity,
    }
    print(json.dumps(line), flush=True)
    model.close()
    ctx.close()


def cpu_baseline_full(a, wl, g, H0, Ws, y, msk):
    """cpu_baseline of the GPU line: ONE whole fp64 oracle epoch of this workload
    at nproc threads, timed live on this host.  The 1-thread
    figure of the same epoch is long (minutes), so it is read from the committed
    record of `bench.py --impl reference --threads 1` (profiles/r2_oracle_cpu.json)
    and labelled as such."""
    threads = os.cpu_count()
    lim = oracle_set_threads(threads)
    ms = oracle_full_epoch_ms(g, H0, Ws, y, msk)
    del lim
    cpu = {"value": ms, "unit": "ms", "cores": threads, "kind": "oracle",
           "sample": f"one whole fp64 oracle epoch of {wl.name} (forward, loss, backward incl. G^0, "
                     f"Adam) at {threads} threads, wall clock, not scaled",
           "host": host_cpu_info()}
    try:
        rec = json.load(open(os.path.join(ROOT, "profiles", "r2_oracle_cpu.json")))
        one = rec.get(wl.name, {}).get("1")
        if one:
            cpu["one_thread"] = {"value": one["value"], "unit": "ms", "host": one.get("host"),
                                 "source": "profiles/r2_oracle_cpu.json (committed; not this run)"}
    except Exception:
        pass
    return cpu


# ------------------------------------------------------------------- main
def main():
    a = parse()
    import numpy as np
    if a.emulate:
        if a.workload == "reddit" and "--workload" not in sys.argv:
            a.workload = "papers"
        return emulate_main(a)
    if a.saint:
        return saint_main(a, int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0")),
                          int(os.environ.get("LOCAL_RANK", "0")))

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    import synth
    wl = synth.WORKLOADS[a.workload]
    if a.workload == "papers" and world < 8:
        # BASELINE configs[4] is an 8-GPU stress case (≈13.7 GB CSR + ≈70 GB of
        # dense slices per GPU at P = 8); fewer GPUs do not hold it.  One rank of
        # it runs on one GPU with --emulate 8.
        if rank == 0:
            print(json.dumps({"metric": METRIC, "impl": a.impl, "unavailable":
                              "papers100M-shaped workload is defined for 8 GPUs (BASELINE configs[4]); "
                              "bench.py --emulate 8 runs one rank of it on one GPU"}))
        return

    if a.impl == "reference":
        # Reference arm = the CPU oracle (tier framing): rank 0 only.  Every step is
        # one WHOLE fp64 oracle epoch (no sampling, no scaling); the run stops after
        # K epochs or once --ref-budget-s is spent (at least one epoch), and
        # "steps" reports how many epochs were actually timed.
        if rank != 0:
            return
        g = synth.make_graph(wl)
        H0 = synth.features(wl.n, wl.f[0])
        Ws = synth.weights(wl.f)
        y = synth.labels(wl.n, wl.f[-1])
        msk = synth.train_mask(wl.n)
        threads = a.threads or os.cpu_count()
        lim = oracle_set_threads(threads)
        times = []
        t_run = time.perf_counter()
        while len(times) < a.steps:
            times.append(oracle_full_epoch_ms(g, H0, Ws, y, msk))
            if time.perf_counter() - t_run > a.ref_budget_s:
                break
        del lim
        v = float(np.mean(times))
        desc = (f"{len(times)} whole fp64 oracle epochs (forward, loss, backward incl. G^0, Adam) "
                f"at {threads} threads, wall clock each, not scaled; no warm-up (no caches or JIT "
                f"to warm); min {min(times):.0f} ms, max {max(times):.0f} ms")
        line = {"metric": METRIC, "value": v, "unit": "ms", "impl": "reference",
                "n_gpus": a.gpus, "steps": len(times), "requested_steps": a.steps, "warmup": 0,
                "ms_per_step": v, "higher_is_better": False, "scaling": "strong",
                "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": wl.name, "n": wl.n, "nnz": wl.nnz, "f": list(wl.f)},
                "cpu_baseline": {"value": v, "unit": "ms", "cores": threads, "kind": "oracle",
                                 "sample": desc, "host": host_cpu_info()},
                "e2e": {"value": v, "unit": "ms", "h2d_bytes_per_step": 0,
                        "d2h_bytes_per_step": 0}}
        print(json.dumps(line), flush=True)
        return

    import torch
    import torch.distributed as dist
    import paper_conf_ipps_kurtysps23_b200 as rdm

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
        obj = [rdm.get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        uid = obj[0]
    else:
        uid = None
    stream = torch.cuda.Stream(device=dev)
    torch.cuda.set_stream(stream)

    t0 = time.time()
    g = synth.make_graph(wl)
    H0 = synth.features(wl.n, wl.f[0])
    y = synth.labels(wl.n, wl.f[-1])
    msk = synth.train_mask(wl.n)
    Ws_h = synth.weights(wl.f)
    t_gen = time.time() - t0

    ctx = rdm.Context(rank=rank if world > 1 else 0, world=world, device=local_rank, stream=stream,
                      unique_id=uid)
    ctx.set_transport(a.transport)
    ctx.set_precision(a.precision)
    comm = None
    if world > 1:
        comm = ctx.comm_info()
        print(f"[bench] rank {rank}/{world}: NCCL {comm['nccl_version']} communicator of "
              f"{comm['ranks']} ranks, user rank {comm['rank']}, CUDA device {comm['device']}",
              file=sys.stderr, flush=True)
    panels = 0 < a.ra < world
    if panels:   # §III-E: R_A copies of A, row panels; tiles + column-group broadcasts
        ctx.set_graph_panels(a.ra, g.rowptr, g.col, g.val)
        pareto, chosen, _, _ = rdm.select_config_ra(list(wl.f), wl.n, wl.nnz, world, a.ra)
    else:
        ctx.set_graph(g.rowptr, g.col, g.val, symmetric=synth.symmetric_values(wl))
        pareto, chosen, comm_u, sparse_u = rdm.select_config(list(wl.f), wl.n, wl.nnz, world)
    lo, hi, _ = rdm.partition(world, rdm.ROW, wl.n, wl.f[0], rank if world > 1 else 0)
    H0_pin = torch.from_numpy(H0[lo:hi]).pin_memory()
    y_pin = torch.from_numpy(y[lo:hi]).pin_memory()
    m_pin = torch.from_numpy(msk[lo:hi]).pin_memory()
    H0_d, y_d, m_d = H0_pin.to(dev), y_pin.to(dev), m_pin.to(dev)
    Wd = [torch.from_numpy(w).to(dev) for w in Ws_h]
    dW = [torch.zeros_like(w) for w in Wd]
    mom = [torch.zeros_like(w) for w in Wd]
    vel = [torch.zeros_like(w) for w in Wd]
    loss = torch.zeros(1, dtype=torch.float64, device=dev)
    step = [0]
    cur = {}

    def build(cfg):
        if "model" in cur:
            cur["model"].close()
        m = rdm.GCN(ctx, wl.f, cfg, panels=panels)
        m.set_input([H0_d], [y_d], [m_d])
        cur["model"] = m
        return m

    def epoch():
        cur["model"].forward(Wd, loss)
        cur["model"].backward(Wd, dW)
        step[0] += 1
        ctx.adam_step(Wd, dW, mom, vel, step[0], lr=0.01)

    def time_epochs(k):
        """ms per epoch over k epochs: CUDA events on the library stream, max over ranks."""
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)
        s0 = torch.cuda.Event(enable_timing=True)
        s1 = torch.cuda.Event(enable_timing=True)
        s0.record(stream)
        for _ in range(k):
            epoch()
        s1.record(stream)
        torch.cuda.synchronize(dev)
        ms = s0.elapsed_time(s1) / k
        if world > 1:
            t = torch.tensor([ms], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
        return ms

    sweep = None
    if a.sweep or a.config == "trial":
        # NEXT-1 / PAPER.md L224: "after trying out each pareto-optimal configuration in
        # the first few epochs, we can dynamically determine the fastest configuration".
        cand = list(range(4 ** wl.L)) if a.sweep else list(pareto)
        sweep = {}
        for cid in cand:
            build(cid)
            time_epochs(2)
            sweep[cid] = time_epochs(3)
        trial_pick = min(pareto, key=lambda c: sweep[c])
    if a.config == "auto":
        cfg_id = chosen
    elif a.config == "trial":
        cfg_id = trial_pick
    else:
        cfg_id = int(a.config)
    model = build(cfg_id)

    for _ in range(max(3, a.warmup)):
        epoch()
    ctx.sync()
    torch.cuda.synchronize(dev)

    # ---------------- timed region (device clock, max over ranks)
    ctx.reset_counters()
    ctx.reset_phase_times()
    ctx.set_timing(True)
    clk = ClockSampler(local_rank)
    clk.start()
    time.sleep(0.3)
    t_w = time.time()
    while not clk.ready() and time.time() - t_w < 5.0:
        time.sleep(0.05)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    marks = [torch.cuda.Event(enable_timing=True) for _ in range(a.steps)]
    e0.record(stream)
    for i in range(a.steps):
        epoch()
        marks[i].record(stream)   # per-epoch mark (mean, median, p95)
    e1.record(stream)
    torch.cuda.synchronize(dev)
    clocks = clk.stop()
    ms_total = e0.elapsed_time(e1)
    ep_ms = [e0.elapsed_time(marks[0])] + [marks[i - 1].elapsed_time(marks[i]) for i in range(1, a.steps)]
    if world > 1:
        t = torch.tensor(ep_ms, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ep_ms = t.tolist()
    cnt = ctx.counters()
    ph_ms, ph_launch = ctx.phase_times()
    ctx.set_timing(False)
    if world > 1:
        t = torch.tensor([ms_total], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_total = float(t.item())
    ms_epoch = ms_total / a.steps

    # ---------------- e2e: host inputs → device each epoch, loss read back
    e2e = None
    if not a.no_e2e:
        loss_host = torch.zeros(1, dtype=torch.float64).pin_memory()
        h2d = H0_pin.numel() * 4 + y_pin.numel() * 4 + m_pin.numel()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)
        k2 = max(3, a.steps // 2)
        f0 = torch.cuda.Event(enable_timing=True)
        f1 = torch.cuda.Event(enable_timing=True)
        f0.record(stream)
        for _ in range(k2):
            model.set_input([H0_pin], [y_pin], [m_pin], on_host=True)
            epoch()
            loss_host.copy_(loss, non_blocking=True)
        f1.record(stream)
        torch.cuda.synchronize(dev)
        e_ms = f0.elapsed_time(f1)
        if world > 1:
            t = torch.tensor([e_ms], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e_ms = float(t.item())
        e2e = {"value": e_ms / k2, "unit": "ms", "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": 8}

    loss_main = float(loss.item())

    # ---------------- the other precision variant, same model and inputs (NEXT-3)
    variants = None
    if not a.no_variants:
        other = "fast" if a.precision == "fp32" else "fp32"
        ctx.set_precision(other)
        for _ in range(3):
            epoch()
        v_ms = time_epochs(a.steps)
        ctx.set_precision(a.precision)
        variants = {other: {"ms_per_step": v_ms, "dtype": DTYPES[other],
                            "parity_gate": GATES[other]}}

    # ---------------- roofline of the dominant kernel (SpMM)
    import json as _json
    peaks = {}
    try:
        peaks = _json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0))
    n, nnz = wl.n, wl.nnz
    info = model.info()
    # algorithmic bytes of all SpMM calls in the timed region: per call 8·nnz (col+val)
    # + 8·(N+1) (rowptr) + 8·N·w (read the slice once, write once); Σ w = spmm_nnz_cols/nnz
    spmm_calls = cnt["spmm_calls"]
    sum_w = cnt["spmm_nnz_cols"] / max(1, nnz)
    alg_bytes = spmm_calls * (8 * nnz + 8 * (n + 1)) + 8 * n * sum_w
    spmm_s = ph_ms["spmm"] / 1e3
    achieved = alg_bytes / spmm_s / 1e9 if spmm_s > 0 else 0.0
    # traffic: DRAM bytes per SpMM call from the committed ncu --set full capture
    # (profiles/r2_spmm_traffic.json, per width), averaged over this epoch's calls
    traffic, traffic_src = None, None
    try:
        tj = _json.load(open(os.path.join(ROOT, "profiles", "r2_spmm_traffic.json")))
        rec = tj.get(wl.name)
        if rec and world == 1 and a.precision == "fp32" and not panels:
            _, desc = rdm.plan_info(list(wl.f), cfg_id, 1, n)
            ws = [int(l.split("w=")[1].split()[0]) for l in desc.splitlines() if l.strip().startswith("SPMM")]
            per = rec["per_width_gb"]
            if ws and all(f"w{w}" in per for w in ws):
                traffic = sum(per[f"w{w}"] for w in ws) / len(ws)
                traffic_src = rec["source"]
    except Exception:
        pass
    roofline = {"bound": "hbm", "achieved": achieved, "peak": hbm_peak, "unit": "GB/s",
                "frac": achieved / hbm_peak, "traffic": traffic, "traffic_unit": "GB per SpMM call",
                "traffic_source": traffic_src,
                "algorithmic_gb_per_call": alg_bytes / max(1, spmm_calls) / 1e9,
                "peak_source": "MEASURED_PEAKS.json hbm_gbs (measured copy)",
                "kernel": "spmm call (tile panels + binary hub tiles + residual CSR + heavy-row reduce)",
                "spmm_share_of_step": ph_ms["spmm"] / max(1e-9, ms_total),
                "avg_call_ms": ph_ms["spmm"] / max(1, spmm_calls),
                "gather_gbs": (cnt["spmm_nnz_cols"] * 4) / spmm_s / 1e9 if spmm_s > 0 else 0.0}
    # the unit that actually paces the residual CSR kernels (committed ncu
    # capture of the same build, profiles/r2_spmm_units.json): L1/TEX, not HBM
    try:
        uj = _json.load(open(os.path.join(ROOT, "profiles", "r2_spmm_units.json"))).get(wl.name)
        if uj and world == 1 and a.precision == "fp32" and not panels:
            roofline["residual_kernels_pct_of_peak"] = {
                k: {"l1tex": round(v[0]["l1tex__throughput.avg.pct_of_peak_sustained_elapsed"], 1),
                    "l2": round(v[0]["lts__throughput.avg.pct_of_peak_sustained_elapsed"], 1),
                    "dram_read": round(v[0]["dram__bytes_read.sum.pct_of_peak_sustained_elapsed"], 1)}
                for k, v in uj["kernels"].items()}
            roofline["residual_kernels_source"] = uj["source"]
    except Exception:
        pass
    a2a_s = ph_ms["a2a"] / 1e3
    a2a_bus = (cnt["a2a_bytes_wire"] / a2a_s / 1e9) if a2a_s > 0 and cnt["a2a_bytes_wire"] else None

    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        cpu = cpu_baseline_full(a, wl, g, H0, Ws_h, y, msk)

    if rank == 0:
        line = {
            "metric": METRIC, "value": ms_epoch, "unit": "ms", "n_gpus": world, "steps": a.steps,
            "warmup": max(3, a.warmup), "ms_per_step": ms_epoch, "higher_is_better": False,
            "scaling": "strong", "vs_baseline": None, "dtype": DTYPES[a.precision],
            "data": "synthetic",
            "config": {
                "workload": wl.name, "model": f"GCN {wl.L}L f={'/'.join(map(str, wl.f))}",
                "precision": a.precision, "parity_gate": GATES[a.precision],
                "n": n, "nnz": nnz, "graph": graph_desc(wl), "global_batch": n, "seq_len": None,
                "parallelism": f"rdm{world} (A replicated, H row/col redistributed)",
                "transport": a.transport, "replicas_of_A": a.ra if panels else world,
                "config_id": cfg_id, "config_name": rdm.config_name(model.cfg),
                "pareto": pareto, "pick": a.config,
                "sweep_ms": ({str(k): round(v, 4) for k, v in sweep.items()} if sweep else None),
                "model_comm_units": info["model_comm_units"],
                "model_sparse_units": info["model_sparse_units"],
                "l2": (f"inputs larger than L2 (CSR {(8 * nnz + 8 * (n + 1)) / 1e9:.2f} GB streamed "
                       f"per SpMM; H0 {n * wl.f[0] * 4 / 1e6:.0f} MB)"),
                "gen_s": round(t_gen, 1)},
            "clocks": clocks, "e2e": e2e, "gpu_launches": cnt["kernel_launches"],
            "roofline": roofline, "cpu_baseline": cpu,
            "phases_ms_per_step": {k: v / a.steps for k, v in ph_ms.items()},
            "step_ms": {"mean": float(np.mean(ep_ms)), "median": float(np.median(ep_ms)),
                        "p95": float(np.percentile(ep_ms, 95)), "min": float(np.min(ep_ms)),
                        "max": float(np.max(ep_ms)),
                        "note": "per-epoch CUDA-event intervals on the library stream, max over ranks"},
            "spmm_hbm_gbs": achieved, "a2a_bus_gbs": a2a_bus,
            "a2a_bytes_per_step": cnt["a2a_bytes_wire"] / a.steps,
            "bcast_elems_per_step": cnt["bcast_elems"] / a.steps,
            "loss": loss_main, "variants": variants, "nccl": comm,
        }
        print(json.dumps(line), flush=True)
    ctx.sync()
    model.close()
    ctx.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
