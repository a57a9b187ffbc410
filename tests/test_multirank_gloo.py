"""N > 1 host logic on CPU with real processes (torch.distributed gloo,
world_size 2, 127.0.0.1): the executor's plan (rdm_plan_info step list), the
exchange plan (rdm_redist_plan: offsets, counts, ld-padded wire blocks) and
the partition rule, driven step by step in fp64 numpy on two ranks with the
all-to-all done by gloo send/recv, must reproduce the oracle's epoch — loss,
every Y^l after the gradient all-reduce (reading R16) and G^0.  The CUDA
kernels are exercised by the GPU tests; this covers the distributed control
logic that runs around them."""
import os
import re
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import paper_conf_ipps_kurtysps23_b200 as rdm
import synth
from oracle import gcn as og

ROW, COL = rdm.ROW, rdm.COL


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class Rank:
    def __init__(self, p, P, g, f):
        self.p, self.P, self.g, self.f, self.n = p, P, g, f, g.n
        self.t = {}  # (name, layout) -> array (row: r_p x f, col: n x w_p)

    def rows(self, q=None):
        return rdm.partition(self.P, ROW, self.n, 1, self.p if q is None else q)[:2]

    def cols(self, f, q=None):
        return rdm.partition(self.P, COL, self.n, f, self.p if q is None else q)[:2]

    # --- all-to-all following rdm_redist_plan's wire format (ld-padded blocks)
    def a2a(self, name, frm, f):
        P, p, n = self.P, self.p, self.n
        plan = rdm.redist_plan(P, p, frm, n, f)
        lds = [(self.cols(f, q)[1] - self.cols(f, q)[0] + 3) // 4 * 4 for q in range(P)]
        r0, r1 = self.rows()
        rp = r1 - r0
        c0, c1 = self.cols(f)
        ldp = lds[p]
        if frm == ROW:
            X = self.t[(name, ROW)]
            stage = np.concatenate([np.pad(X[:, slice(*self.cols(f, q))],
                                           ((0, 0), (0, lds[q] - (self.cols(f, q)[1] - self.cols(f, q)[0]))))
                                    .ravel() for q in range(P)]) if rp else np.zeros(0)
            colbuf = np.zeros(n * ldp)
            reqs = []
            for q in range(P):
                if q == p:
                    continue
                if plan["send_elems"][q]:
                    o = plan["send_off"][q]
                    reqs.append(dist.isend(torch.from_numpy(stage[o:o + plan["send_elems"][q]].copy()), q))
                if plan["recv_elems"][q]:
                    buf = torch.zeros(plan["recv_elems"][q], dtype=torch.float64)
                    reqs.append((dist.irecv(buf, q), buf, plan["recv_off"][q]))
            for r in reqs:
                if isinstance(r, tuple):
                    r[0].wait()
                    colbuf[r[2]:r[2] + len(r[1])] = r[1].numpy()
                else:
                    r.wait()
            C = colbuf.reshape(n, ldp)
            C[r0:r1, :c1 - c0] = X[:, c0:c1]     # self block
            self.t[(name, COL)] = C[:, :c1 - c0].copy()
        else:
            C = np.pad(self.t[(name, COL)], ((0, 0), (0, ldp - (c1 - c0)))).ravel()
            stage = np.zeros(rp * sum(lds))
            reqs = []
            for q in range(P):
                if q == p:
                    continue
                if plan["send_elems"][q]:
                    o = plan["send_off"][q]
                    reqs.append(dist.isend(torch.from_numpy(C[o:o + plan["send_elems"][q]].copy()), q))
                if plan["recv_elems"][q]:
                    buf = torch.zeros(plan["recv_elems"][q], dtype=torch.float64)
                    reqs.append((dist.irecv(buf, q), buf, plan["recv_off"][q]))
            for r in reqs:
                if isinstance(r, tuple):
                    r[0].wait()
                    stage[r[2]:r[2] + len(r[1])] = r[1].numpy()
                else:
                    r.wait()
            X = np.zeros((rp, f))
            off = 0
            for q in range(P):
                q0, q1 = self.cols(f, q)
                blk = stage[off:off + rp * lds[q]].reshape(rp, lds[q]) if rp else np.zeros((0, lds[q]))
                off += rp * lds[q]
                X[:, q0:q1] = blk[:, :q1 - q0]
            X[:, c0:c1] = self.t[(name, COL)][r0:r1]   # self block
            self.t[(name, ROW)] = X


def _run_plan(p, P, port, cfg, seed, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=p, world_size=P)
    try:
        f = (61, 24, 7)
        n = 300
        g = synth.rmat(n, 1500, seed=seed)
        H0 = synth.features(n, f[0]).astype(np.float64)
        Ws = [w.astype(np.float64) for w in synth.weights(f)]
        y = synth.labels(n, f[-1])
        m = synth.train_mask(n, 0.7, seed=9)
        info, desc = rdm.plan_info(list(f), cfg, P, n)
        R = Rank(p, P, g, f)
        r0, r1 = R.rows()
        R.t[("H0", ROW)] = H0[r0:r1]
        R.t[("H0", COL)] = H0[:, slice(*R.cols(f[0]))]
        n_train = float(m.sum())
        dW = [np.zeros_like(w) for w in Ws]
        loss_part = 0.0
        key = lambda s: (s.split(".")[0], ROW if s.endswith(".row") else COL)
        for line in desc.splitlines():
            line = line.strip()
            if not line or line.endswith(":"):
                continue
            op = line.split()[0]
            if op == "A2A":
                mm = re.match(r"A2A\s+(\w+)\.(row|col) -> \w+\.(row|col) f=(\d+)", line)
                R.a2a(mm.group(1), ROW if mm.group(2) == "row" else COL, int(mm.group(4)))
            elif op == "SPMM":
                mm = re.match(r"SPMM\s+(A\^T|A)\s+(\S+) -> (\S+) w=\d+", line)
                Xc = R.t[key(mm.group(2))]
                Y = og.spmm_t(g, Xc) if mm.group(1) == "A^T" else og.spmm(g, Xc)
                if "+relu" in line:
                    Y = np.maximum(Y, 0)
                mk = re.search(r"\*mask\((\S+)\)", line)
                if mk:
                    Y = Y * (R.t[key(mk.group(1))] > 0)
                R.t[key(mm.group(3))] = Y
            elif op == "GEMM":
                mm = re.match(r"GEMM\s+(NN|NT|TN)\s+(\S+?)(\^T)?\s+(\S+) -> (\S+)", line)
                kind = mm.group(1)
                if kind == "TN":
                    l = int(mm.group(5)[1:])
                    dW[l - 1] += R.t[key(mm.group(2))].T @ R.t[key(mm.group(4))]
                else:
                    l = int(mm.group(4)[1:])
                    X = R.t[key(mm.group(2))]
                    Y = X @ Ws[l - 1] if kind == "NN" else X @ Ws[l - 1].T
                    if "+relu" in line:
                        Y = np.maximum(Y, 0)
                    mk = re.search(r"\*mask\((\S+)\)", line)
                    if mk:
                        Y = Y * (R.t[key(mk.group(1))] > 0)
                    R.t[key(mm.group(5))] = Y
            elif op == "MASK":
                mm = re.match(r"MASK\s+(\S+) \*= 1\[(\S+) > 0\]", line)
                R.t[key(mm.group(1))] = R.t[key(mm.group(1))] * (R.t[key(mm.group(2))] > 0)
            elif op == "LOSS":
                mm = re.match(r"LOSS\s+(\S+) -> (\S+)", line)
                Z = R.t[key(mm.group(1))]
                lp, G = og.softmax_xent(Z, y[r0:r1], m[r0:r1], n_train=n_train)
                loss_part = lp
                R.t[key(mm.group(2))] = G
            else:
                raise AssertionError(line)
        # loss and Y^l all-reduce over ranks (reading R16)
        t = torch.tensor([loss_part], dtype=torch.float64)
        dist.all_reduce(t)
        for l in range(len(dW)):
            tw = torch.from_numpy(dW[l])
            dist.all_reduce(tw)
            dW[l] = tw.numpy()
        ref = og.epoch(g, H0, Ws, y, m)
        assert abs(float(t) - ref.loss) < 1e-12 * abs(ref.loss)
        for l in range(len(dW)):
            assert og.max_rel_err(dW[l], ref.Y[l + 1]) < 1e-11, (cfg, l)
        # G^0 in whichever layout the plan left it
        if ("G0", ROW) in R.t:
            assert og.max_rel_err(R.t[("G0", ROW)], ref.G[0][r0:r1]) < 1e-11
        else:
            c0, c1 = R.cols(f[0])
            assert og.max_rel_err(R.t[("G0", COL)], ref.G[0][:, c0:c1]) < 1e-11
        out.put((p, cfg, "ok"))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("cfg", [0, 2, 3, 5, 6, 9, 10, 12, 15])
def test_two_rank_plan_matches_oracle(cfg):
    ctx = mp.get_context("spawn")
    q = ctx.SimpleQueue()
    port = _free_port()
    procs = [ctx.Process(target=_run_plan, args=(p, 2, port, cfg, 5, q)) for p in range(2)]
    for pr in procs:
        pr.start()
    for pr in procs:
        pr.join(timeout=180)
    assert all(pr.exitcode == 0 for pr in procs), [pr.exitcode for pr in procs]
    res = [q.get() for _ in range(2)]
    assert sorted(r[0] for r in res) == [0, 1]


# ------------------------------------------------------------- R_A < P (NEXT-4)
def _run_panels(p, P, RA, port, q_out):
    """One layer's SpMM and redistribution on the P/R_A x R_A grid with real
    processes: tiles from rdm_partition_tile, the Fig. 6 broadcast of input
    tiles inside the column group (gloo send/recv), the row-panel product, and
    the tile → row-slice redistribution inside the panel group; every rank's
    result equals the oracle's slice."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=p, world_size=P)
    try:
        g = synth.rmat(700, 4000, seed=4)
        n, w = g.n, 13
        X = np.random.default_rng(0).standard_normal((n, w))
        i, j = p // RA, p % RA
        r0, r1, c0, c1, _ = rdm.partition_tile(P, RA, n, w, p)
        mine = torch.from_numpy(np.ascontiguousarray(X[r0:r1, c0:c1]))
        # broadcast inside column group j: gather In[:, c0:c1] from ranks i2·R_A + j
        full = np.zeros((n, c1 - c0))
        full[r0:r1] = mine.numpy()
        reqs = []
        bufs = {}
        for i2 in range(P // RA):
            qr = i2 * RA + j
            if qr == p:
                continue
            q0, q1, _, _, _ = rdm.partition_tile(P, RA, n, w, qr)
            bufs[qr] = torch.zeros((q1 - q0, c1 - c0), dtype=torch.float64)
            reqs.append(dist.isend(mine, qr))
            reqs.append(dist.irecv(bufs[qr], qr))
        for rq in reqs:
            rq.wait()
        for qr, b in bufs.items():
            q0, q1, _, _, _ = rdm.partition_tile(P, RA, n, w, qr)
            full[q0:q1] = b.numpy()
        # row-panel product: rows r0..r1 of A·In[:, c0:c1]
        out_tile = og.spmm(g, full)[r0:r1]
        ref = og.spmm(g, X)
        assert og.max_rel_err(out_tile, ref[r0:r1, c0:c1]) < 1e-12
        # tile → row slices inside panel group i
        lo, hi, _ = rdm.partition(P, ROW, n, w, p)
        row = np.zeros((hi - lo, w))
        row[:, c0:c1] = out_tile[lo - r0:hi - r0]
        reqs, got = [], {}
        for j2 in range(RA):
            qr = i * RA + j2
            if qr == p:
                continue
            qlo, qhi, _ = rdm.partition(P, ROW, n, w, qr)
            _, _, d0, d1, _ = rdm.partition_tile(P, RA, n, w, qr)
            reqs.append(dist.isend(torch.from_numpy(np.ascontiguousarray(out_tile[qlo - r0:qhi - r0])), qr))
            got[qr] = torch.zeros((hi - lo, d1 - d0), dtype=torch.float64)
            reqs.append(dist.irecv(got[qr], qr))
        for rq in reqs:
            rq.wait()
        for qr, b in got.items():
            _, _, d0, d1, _ = rdm.partition_tile(P, RA, n, w, qr)
            row[:, d0:d1] = b.numpy()
        assert og.max_rel_err(row, ref[lo:hi]) < 1e-12
        q_out.put((p, "ok"))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("P,RA", [(2, 1), (4, 2)])
def test_panels_grid_with_processes(P, RA):
    ctx = mp.get_context("spawn")
    q = ctx.SimpleQueue()
    port = _free_port()
    procs = [ctx.Process(target=_run_panels, args=(p, P, RA, port, q)) for p in range(P)]
    for pr in procs:
        pr.start()
    for pr in procs:
        pr.join(timeout=180)
    assert all(pr.exitcode == 0 for pr in procs), [pr.exitcode for pr in procs]
    assert sorted(q.get()[0] for _ in range(P)) == list(range(P))
