"""B200-native GNN-RDM hot path (Kurt et al., IPDPS'23) — Python binding.

Thin ctypes marshalling over the C ABI in ``include/rdm.h`` /
``lib/librdm.so``: every step of the path (SpMM, GEMM, redistribution,
loss, Adam) runs in the library's sm_100a kernels; PyTorch is used only for
device memory, streams and process groups.  There is no CPU fallback: if the
native library is missing this import fails.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "lib", "librdm.so")
if os.environ.get("RDM_LIB_VARIANT"):   # timing experiments only (tools/build_variant.sh)
    LIB_PATH = os.path.join(_HERE, "lib", f"librdm_{os.environ['RDM_LIB_VARIANT']}.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is missing: build the CUDA library first "
        "(`make -C <repo>` or `python -c 'import __graft_entry__ as g; g.build()'`)")

_lib = ctypes.CDLL(LIB_PATH)

# ------------------------------------------------------------ constants
OK, ERR_ARG, ERR_CUDA, ERR_NCCL, ERR_OOM, ERR_UNSUPPORTED, ERR_STATE = range(7)
ROW, COL = 0, 1
EPI_NONE, EPI_BIAS, EPI_RELU, EPI_MASK = 0, 1, 2, 4
GEMM_NN, GEMM_NT, GEMM_TN = 0, 1, 2
ALL_RANKS = -1
MAX_LAYERS = 8
UNIQUE_ID_BYTES = 128
GCN_INPUT_GRAD, GCN_BIAS, GCN_PANELS, GCN_LOW_MEMORY = 1, 2, 4, 8
T_H, T_Z, T_G, T_MEMO, T_DWP = range(5)
PHASES = ["spmm", "gemm", "pack", "a2a", "loss", "allreduce", "adam", "other", "sample"]
_STATUS = {0: "OK", 1: "ERR_ARG", 2: "ERR_CUDA", 3: "ERR_NCCL", 4: "ERR_OOM",
           5: "ERR_UNSUPPORTED", 6: "ERR_STATE"}

TRANSPORTS = {"nccl": 0, "p2p": 1}
PRECISIONS = {"fp32": 0, "fast": 1}

# C symbols declared in include/rdm.h (checked by tests/test_abi.py)
EXPORTS = [
    "rdm_get_unique_id", "rdm_init", "rdm_finalize", "rdm_last_error", "rdm_sync",
    "rdm_set_stream", "rdm_world", "rdm_num_local", "rdm_local_rank", "rdm_partition",
    "rdm_set_graph", "rdm_spmm", "rdm_gemm", "rdm_redistribute", "rdm_allreduce_sum",
    "rdm_config_from_id", "rdm_config_to_id", "rdm_config_costs", "rdm_select_config",
    "rdm_gcn_create", "rdm_gcn_destroy", "rdm_gcn_set_input", "rdm_gcn_forward",
    "rdm_gcn_backward", "rdm_gcn_get_info", "rdm_gcn_describe", "rdm_gcn_tensor",
    "rdm_adam_step", "rdm_get_counters", "rdm_reset_counters", "rdm_set_timing",
    "rdm_get_phase_times", "rdm_reset_phase_times", "rdm_redist_plan", "rdm_plan_info",
    "rdm_set_transport", "rdm_get_transport", "rdm_debug_disable_tc",
    "rdm_set_precision", "rdm_get_precision", "rdm_set_graph_panels", "rdm_partition_tile",
    "rdm_redistribute_panels", "rdm_spmm_panels", "rdm_max_replication", "rdm_select_config_ra",
    "rdm_saint_wait", "rdm_init_emulated", "rdm_is_emulated", "rdm_comm_info",
]


class RdmConfig(ctypes.Structure):
    _fields_ = [("L", ctypes.c_int), ("fwd_D", ctypes.c_uint8 * MAX_LAYERS),
                ("bwd_D", ctypes.c_uint8 * MAX_LAYERS)]


class RdmCounters(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int64) for n in (
        "a2a_calls", "a2a_elems_payload", "a2a_bytes_wire", "a2a_width_units", "spmm_calls",
        "spmm_nnz_cols", "spmm_width_units", "gemm_calls", "gemm_flops", "allreduce_bytes",
        "kernel_launches", "bcast_elems")]

    def as_dict(self):
        return {n: getattr(self, n) for n, _ in self._fields_}


class RdmGcnInfo(ctypes.Structure):
    _fields_ = [("model_comm_units", ctypes.c_int64), ("model_sparse_units", ctypes.c_int64),
                ("plan_comm_units", ctypes.c_int64), ("plan_hidden_comm_units", ctypes.c_int64),
                ("plan_sparse_units", ctypes.c_int64), ("a2a_elems", ctypes.c_int64),
                ("n_fwd_steps", ctypes.c_int), ("n_bwd_steps", ctypes.c_int),
                ("workspace_bytes", ctypes.c_int64)]

    def as_dict(self):
        return {n: getattr(self, n) for n, _ in self._fields_}


_vp, _i64, _int = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
_pp = ctypes.POINTER(ctypes.c_void_p)
_pi64 = ctypes.POINTER(ctypes.c_int64)
_sig = {
    "rdm_get_unique_id": [_vp],
    "rdm_init": [ctypes.POINTER(_vp), _int, _int, _vp, _int, _vp],
    "rdm_finalize": [_vp],
    "rdm_sync": [_vp],
    "rdm_set_stream": [_vp, _vp],
    "rdm_partition": [_int, _int, _i64, _i64, _int, _pi64, _pi64, _pi64],
    "rdm_set_graph": [_vp, _i64, _i64, _vp, _vp, _vp, _int, _int],
    "rdm_init_emulated": [ctypes.POINTER(_vp), _int, _int, _int, _vp],
    "rdm_comm_info": [_vp, ctypes.POINTER(_int), ctypes.POINTER(_int), ctypes.POINTER(_int),
                      ctypes.POINTER(_int)],
    "rdm_spmm": [_vp, _int, _vp, _i64, _vp, _i64, _i64, _int, _vp, _vp, _i64],
    "rdm_gemm": [_vp, _int, _vp, _i64, _vp, _i64, _vp, _i64, _i64, _i64, _i64, _int, _vp, _vp],
    "rdm_redistribute": [_vp, _int, _pp, _pp, _i64, _i64],
    "rdm_allreduce_sum": [_vp, _pp, _i64],
    "rdm_config_from_id": [_int, _i64, ctypes.POINTER(RdmConfig)],
    "rdm_config_costs": [_int, _pi64, _int, _i64, _pi64, _pi64],
    "rdm_select_config": [_int, _pi64, _i64, _i64, _int, _int, _pi64, ctypes.POINTER(_int),
                          _pi64, _pi64, _pi64],
    "rdm_gcn_create": [_vp, _int, _pi64, ctypes.POINTER(RdmConfig), _int, ctypes.POINTER(_vp)],
    "rdm_gcn_destroy": [_vp],
    "rdm_gcn_set_input": [_vp, _pp, _pp, _pp, _int],
    "rdm_gcn_forward": [_vp, _pp, _pp, _vp],
    "rdm_gcn_backward": [_vp, _pp, _pp, _pp],
    "rdm_gcn_get_info": [_vp, ctypes.POINTER(RdmGcnInfo)],
    "rdm_gcn_describe": [_vp, ctypes.c_char_p, ctypes.c_size_t],
    "rdm_gcn_tensor": [_vp, _int, _int, _int, _int, _pp, _pi64, _pi64, _pi64],
    "rdm_adam_step": [_vp, _int, _pp, _pp, _pp, _pp, _pi64, ctypes.c_float, ctypes.c_float,
                      ctypes.c_float, ctypes.c_float, _int],
    "rdm_get_counters": [_vp, ctypes.POINTER(RdmCounters)],
    "rdm_reset_counters": [_vp],
    "rdm_set_timing": [_vp, _int],
    "rdm_set_transport": [_vp, _int],
    "rdm_set_precision": [_vp, _int],
    "rdm_saint_wait": [_vp],
    "rdm_select_config_ra": [_int, _pi64, _i64, _i64, _int, _int, _int, _pi64, ctypes.POINTER(_int),
                             _pi64, ctypes.POINTER(ctypes.c_double), _pi64],
    "rdm_set_graph_panels": [_vp, _int, _i64, _i64, _vp, _vp, _vp, _int],
    "rdm_partition_tile": [_int, _int, _i64, _i64, _int, _pi64, _pi64, _pi64, _pi64, _pi64],
    "rdm_redistribute_panels": [_vp, _int, _pp, _pp, _i64, _i64],
    "rdm_spmm_panels": [_vp, _pp, _pp, _i64, _int, _vp, _pp],
    "rdm_get_phase_times": [_vp, ctypes.POINTER(ctypes.c_double), _pi64],
    "rdm_reset_phase_times": [_vp],
    "rdm_redist_plan": [_int, _int, _int, _i64, _i64, _pi64, _pi64, _pi64, _pi64],
    "rdm_plan_info": [_int, _pi64, ctypes.POINTER(RdmConfig), _int, _i64, _int,
                      ctypes.POINTER(RdmGcnInfo), ctypes.c_char_p, ctypes.c_size_t],
}
for _n, _a in _sig.items():
    getattr(_lib, _n).argtypes = _a
    getattr(_lib, _n).restype = _int
_lib.rdm_last_error.argtypes = [_vp]
_lib.rdm_last_error.restype = ctypes.c_char_p
_lib.rdm_config_to_id.argtypes = [ctypes.POINTER(RdmConfig)]
_lib.rdm_config_to_id.restype = _i64
for _n in ("rdm_world", "rdm_num_local", "rdm_get_transport", "rdm_get_precision", "rdm_is_emulated"):
    getattr(_lib, _n).argtypes = [_vp]
    getattr(_lib, _n).restype = _int
_lib.rdm_debug_disable_tc.argtypes = [_int]
_lib.rdm_debug_disable_tc.restype = _int
_lib.rdm_local_rank.argtypes = [_vp, _int]
_lib.rdm_local_rank.restype = _int
_lib.rdm_max_replication.argtypes = [_int, ctypes.c_double, ctypes.c_double, ctypes.c_double]
_lib.rdm_max_replication.restype = _int


class RdmError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


def _check(st, ctx=None, what=""):
    if st != OK:
        msg = _lib.rdm_last_error(ctx).decode() if ctx else what
        raise RdmError(st, msg or what)


def _ptr(t):
    """Device/host pointer of a torch tensor or numpy array (None → NULL)."""
    if t is None:
        return None
    if hasattr(t, "data_ptr"):
        return t.data_ptr()
    return t.ctypes.data


def _ld(t):
    """Leading dimension (elements) of a 2-D row-major tensor."""
    if t is None:
        return 0
    if hasattr(t, "stride"):
        s = t.stride()
        assert s[-1] == 1, "rows must be contiguous"
        return s[0] if t.dim() == 2 else t.shape[-1]
    return t.strides[0] // t.itemsize


def _parr(ts):
    arr = (ctypes.c_void_p * len(ts))(*[_ptr(t) for t in ts])
    return ctypes.cast(arr, _pp), arr


# --------------------------------------------------------- pure host calls
def get_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(UNIQUE_ID_BYTES)
    _check(_lib.rdm_get_unique_id(buf), what="rdm_get_unique_id")
    return buf.raw


def debug_disable_tc(disable=True):
    """Route GEMMs to the SIMT kernel instead of tcgen05 (rdm.h rdm_debug_disable_tc)."""
    _lib.rdm_debug_disable_tc(int(bool(disable)))


def partition(world, layout, n, f, rank):
    lo, hi, ld = _i64(), _i64(), _i64()
    _check(_lib.rdm_partition(world, layout, n, f, rank, ctypes.byref(lo), ctypes.byref(hi),
                              ctypes.byref(ld)), what="rdm_partition")
    return lo.value, hi.value, ld.value


def partition_tile(world, r_a, n, f, rank):
    """Tile of `rank` in the R_A < P grid (rdm.h rdm_partition_tile):
    (row_lo, row_hi, col_lo, col_hi, ld)."""
    v = [_i64() for _ in range(5)]
    _check(_lib.rdm_partition_tile(world, r_a, n, f, rank, *[ctypes.byref(x) for x in v]),
           what="rdm_partition_tile")
    return tuple(x.value for x in v)


def select_config_ra(f, n, nnz, P, r_a, input_grad=True):
    """R_A < P configuration choice (rdm.h rdm_select_config_ra):
    (pareto ids, chosen id, elements moved per epoch, sparse units)."""
    L = len(f) - 1
    fa = (ctypes.c_int64 * len(f))(*f)
    cap = 4 ** L
    ids = (ctypes.c_int64 * cap)()
    npar = _int(cap)
    ch, ce, su = _i64(), ctypes.c_double(), _i64()
    _check(_lib.rdm_select_config_ra(L, fa, n, nnz, P, r_a, int(input_grad), ids, ctypes.byref(npar),
                                     ctypes.byref(ch), ctypes.byref(ce), ctypes.byref(su)),
           what="rdm_select_config_ra")
    return list(ids[:npar.value]), ch.value, ce.value, su.value


def max_replication(world, mem_bytes, h_all_bytes, graph_bytes) -> int:
    """Largest feasible R_A (rdm.h rdm_max_replication)."""
    return int(_lib.rdm_max_replication(world, float(mem_bytes), float(h_all_bytes), float(graph_bytes)))


def config_from_id(L, cfg_id) -> RdmConfig:
    c = RdmConfig()
    _check(_lib.rdm_config_from_id(L, cfg_id, ctypes.byref(c)), what="rdm_config_from_id")
    return c


def config_to_id(c: RdmConfig) -> int:
    return _lib.rdm_config_to_id(ctypes.byref(c))


def config_name(c: RdmConfig) -> str:
    sd = "SD"
    return "F" + "".join(sd[c.fwd_D[l]] for l in range(c.L)) + "/B" + "".join(
        sd[c.bwd_D[l]] for l in range(c.L - 1, -1, -1))


def config_costs(f, cfg_id, need_input_grad=True):
    fa = (ctypes.c_int64 * len(f))(*f)
    c, s = _i64(), _i64()
    _check(_lib.rdm_config_costs(len(f) - 1, fa, int(need_input_grad), cfg_id, ctypes.byref(c),
                                 ctypes.byref(s)), what="rdm_config_costs")
    return c.value, s.value


def redist_plan(world, rank, from_layout, n, f):
    """→ dict of per-peer lists send_off, send_elems, recv_off, recv_elems."""
    arrs = [(ctypes.c_int64 * world)() for _ in range(4)]
    _check(_lib.rdm_redist_plan(world, rank, from_layout, n, f, *arrs), what="rdm_redist_plan")
    keys = ("send_off", "send_elems", "recv_off", "recv_elems")
    return {k: list(a) for k, a in zip(keys, arrs)}


def plan_info(f, cfg, P, n, input_grad=True, low_memory=False, bias=False):
    """→ (info dict, step list text) of the executor plan, without a GPU
    (workspace_bytes: rank 0's activation workspace)."""
    L = len(f) - 1
    c = config_from_id(L, cfg) if isinstance(cfg, int) else cfg
    fa = (ctypes.c_int64 * len(f))(*f)
    info = RdmGcnInfo()
    buf = ctypes.create_string_buffer(1 << 16)
    flags = ((GCN_INPUT_GRAD if input_grad else 0) | (GCN_LOW_MEMORY if low_memory else 0)
             | (GCN_BIAS if bias else 0))
    _check(_lib.rdm_plan_info(L, fa, ctypes.byref(c), P, n, flags,
                              ctypes.byref(info), buf, len(buf)), what="rdm_plan_info")
    return info.as_dict(), buf.value.decode()


def select_config(f, n, nnz, P, need_input_grad=True):
    """→ (pareto_ids, chosen_id, comm_units, sparse_units)."""
    fa = (ctypes.c_int64 * len(f))(*f)
    cap = 4 ** (len(f) - 1)
    ids = (ctypes.c_int64 * cap)()
    npar = _int(cap)
    ch, c, s = _i64(), _i64(), _i64()
    _check(_lib.rdm_select_config(len(f) - 1, fa, n, nnz, P, int(need_input_grad), ids,
                                  ctypes.byref(npar), ctypes.byref(ch), ctypes.byref(c),
                                  ctypes.byref(s)), what="rdm_select_config")
    return [ids[i] for i in range(npar.value)], ch.value, c.value, s.value


# ---------------------------------------------------------------- context
class Context:
    """One rank of a P-process job (NCCL), a single process (world=1), or a
    virtual group of `world` ranks on one GPU (rank=ALL_RANKS)."""

    def __init__(self, rank=0, world=1, device=0, stream=None, unique_id: bytes | None = None,
                 emulate=False):
        """emulate=True: rank `rank` of `world` with no peers (rdm_init_emulated;
        timing / memory measurement of one rank of a P-rank job on one GPU)."""
        import torch
        if stream is None:
            stream = torch.cuda.current_stream(device)
        self.stream = stream
        h = ctypes.c_void_p()
        if emulate:
            _check(_lib.rdm_init_emulated(ctypes.byref(h), rank, world, device, stream.cuda_stream),
                   what=f"rdm_init_emulated(rank={rank}, world={world}, device={device})")
        else:
            uid = ctypes.create_string_buffer(unique_id, UNIQUE_ID_BYTES) if unique_id else None
            _check(_lib.rdm_init(ctypes.byref(h), rank, world, uid, device, stream.cuda_stream),
                   what=f"rdm_init(rank={rank}, world={world}, device={device})")
        self.emulated = bool(emulate)
        self.h = h
        self.world = world
        self.device = device
        self.local_ranks = [_lib.rdm_local_rank(h, i) for i in range(_lib.rdm_num_local(h))]

    def close(self):
        if getattr(self, "h", None):
            _lib.rdm_finalize(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _c(self, st):
        _check(st, self.h)

    def sync(self):
        self._c(_lib.rdm_sync(self.h))

    def comm_info(self) -> dict:
        """NCCL version and the communicator's rank count / rank / device (rdm_comm_info)."""
        v, n, r, d = _int(), _int(), _int(), _int()
        self._c(_lib.rdm_comm_info(self.h, ctypes.byref(v), ctypes.byref(n), ctypes.byref(r),
                                   ctypes.byref(d)))
        return {"nccl_version": v.value, "ranks": n.value, "rank": r.value, "device": d.value}

    def set_graph(self, rowptr, col, val, symmetric=True):
        """CSR from numpy (host) or torch (device) arrays: int64 rowptr, int32 col, fp32 val."""
        on_host = not hasattr(rowptr, "data_ptr") or not rowptr.is_cuda
        n = len(rowptr) - 1
        nnz = int(rowptr[-1])
        self.n, self.nnz = n, nnz
        self._c(_lib.rdm_set_graph(self.h, n, nnz, _ptr(rowptr), _ptr(col), _ptr(val),
                                   int(symmetric), int(on_host)))

    def spmm(self, transpose, x, out, w, epilogue=EPI_NONE, bias=None, mask=None):
        self._c(_lib.rdm_spmm(self.h, int(transpose), _ptr(x), _ld(x), _ptr(out), _ld(out), w,
                              epilogue, _ptr(bias), _ptr(mask), _ld(mask)))

    def gemm(self, op, X, W, C, rows, k, m, epilogue=EPI_NONE, bias=None, mask=None):
        self._c(_lib.rdm_gemm(self.h, op, _ptr(X), _ld(X), _ptr(W), _ld(W), _ptr(C), _ld(C),
                              rows, k, m, epilogue, _ptr(bias), _ptr(mask)))

    def redistribute(self, from_layout, srcs, dsts, n, f):
        sp, _a = _parr(srcs)
        dp, _b = _parr(dsts)
        self._c(_lib.rdm_redistribute(self.h, from_layout, sp, dp, n, f))

    def set_graph_panels(self, r_a, rowptr, col, val):
        """Row panels of A for R_A < P (rdm.h rdm_set_graph_panels)."""
        on_host = not hasattr(rowptr, "data_ptr") or not rowptr.is_cuda
        n = len(rowptr) - 1
        self._c(_lib.rdm_set_graph_panels(self.h, r_a, n, int(rowptr[-1]), _ptr(rowptr), _ptr(col),
                                          _ptr(val), int(on_host)))

    def redistribute_panels(self, from_layout, srcs, dsts, n, f):
        sp, _a = _parr(srcs)
        dp, _b = _parr(dsts)
        self._c(_lib.rdm_redistribute_panels(self.h, from_layout, sp, dp, n, f))

    def spmm_panels(self, ins, outs, f, epilogue=EPI_NONE, bias=None, masks=None):
        ip, _a = _parr(ins)
        op, _b = _parr(outs)
        mp, _c2 = _parr(masks) if masks is not None else (None, None)
        self._c(_lib.rdm_spmm_panels(self.h, ip, op, f, epilogue, _ptr(bias), mp))

    def allreduce_sum(self, bufs):
        bp, _a = _parr(bufs)
        self._c(_lib.rdm_allreduce_sum(self.h, bp, bufs[0].numel()))

    def adam_step(self, params, grads, ms, vs, step, lr=0.01, betas=(0.9, 0.999), eps=1e-8):
        pp, _a = _parr(params)
        gp, _b = _parr(grads)
        mp, _c2 = _parr(ms)
        vp, _d = _parr(vs)
        sizes = (ctypes.c_int64 * len(params))(*[p.numel() for p in params])
        self._c(_lib.rdm_adam_step(self.h, len(params), pp, gp, mp, vp, sizes, lr, betas[0],
                                   betas[1], eps, step))

    def counters(self) -> dict:
        c = RdmCounters()
        self._c(_lib.rdm_get_counters(self.h, ctypes.byref(c)))
        return c.as_dict()

    def reset_counters(self):
        self._c(_lib.rdm_reset_counters(self.h))

    def set_timing(self, on=True):
        self._c(_lib.rdm_set_timing(self.h, int(on)))

    def set_transport(self, transport):
        """"nccl" (pack + all-to-all + unpack) or "p2p" (redistributions fused
        into their producing kernel's epilogue, rdm.h rdm_set_transport);
        applies to GCN instances created afterwards."""
        self._c(_lib.rdm_set_transport(self.h, TRANSPORTS[transport]))

    def set_precision(self, precision):
        """"fp32" (default; 3xTF32 GEMMs, 1e-4 gate) or "fast" (bf16 SpMM
        operand, 1xTF32 GEMMs, 2e-2 gate; rdm.h rdm_set_precision); applies to
        every later call on this context."""
        self._c(_lib.rdm_set_precision(self.h, PRECISIONS[precision]))

    @property
    def precision(self):
        return {v: k for k, v in PRECISIONS.items()}[_lib.rdm_get_precision(self.h)]

    @property
    def transport(self):
        return {v: k for k, v in TRANSPORTS.items()}[_lib.rdm_get_transport(self.h)]

    def phase_times(self):
        ms = (ctypes.c_double * len(PHASES))()
        ln = (ctypes.c_int64 * len(PHASES))()
        self._c(_lib.rdm_get_phase_times(self.h, ms, ln))
        return ({p: ms[i] for i, p in enumerate(PHASES)}, {p: ln[i] for i, p in enumerate(PHASES)})

    def reset_phase_times(self):
        self._c(_lib.rdm_reset_phase_times(self.h))


class GCN:
    """A GCN instance (L layers, widths f) running configuration `cfg` (ID or RdmConfig)."""

    def __init__(self, ctx: Context, f, cfg, input_grad=True, saint=None, panels=False,
                 low_memory=False, bias=False):
        self.ctx = ctx
        self.f = list(f)
        self.L = len(f) - 1
        self.cfg = config_from_id(self.L, cfg) if isinstance(cfg, int) else cfg
        fa = (ctypes.c_int64 * len(f))(*f)
        h = ctypes.c_void_p()
        flags = ((GCN_INPUT_GRAD if input_grad else 0) | (GCN_PANELS if panels else 0)
                 | (GCN_LOW_MEMORY if low_memory else 0) | (GCN_BIAS if bias else 0))
        self.bias = bool(bias)
        self.saint = saint   # keeps the sampler alive while this instance exists
        if saint is None:
            ctx._c(_lib.rdm_gcn_create(ctx.h, self.L, fa, ctypes.byref(self.cfg), flags,
                                       ctypes.byref(h)))
        else:
            ctx._c(_lib.rdm_saint_gcn_create(saint.h, self.L, fa, ctypes.byref(self.cfg), flags,
                                             ctypes.byref(h)))
        self.h = h

    def close(self):
        if getattr(self, "h", None):
            _lib.rdm_gcn_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @property
    def cfg_id(self):
        return config_to_id(self.cfg)

    def set_input(self, H0_rows, labels_rows, mask_rows=None, on_host=False):
        hp, _a = _parr(H0_rows)
        lp, _b = _parr(labels_rows)
        if mask_rows is None:
            mp = None
        else:
            mp, _c2 = _parr(mask_rows)
        self.ctx._c(_lib.rdm_gcn_set_input(self.h, hp, lp, mp, int(on_host)))

    def saint_input(self, H0_full, labels_full, mask_full=None):
        """GraphSAINT: gather the current subgraph's input from full-graph device
        tensors (rdm.h rdm_saint_set_input)."""
        self.ctx._c(_lib.rdm_saint_set_input(self.h, _ptr(H0_full), H0_full.stride(0),
                                             _ptr(labels_full),
                                             None if mask_full is None else _ptr(mask_full)))

    def forward(self, Ws, loss_dev, bs=None):
        """bs: the L bias vectors b^l (f_l floats each, device) of a bias=True model."""
        wp, _a = _parr(Ws)
        bp, _b = _parr(bs) if bs is not None else (None, None)
        self.ctx._c(_lib.rdm_gcn_forward(self.h, wp, bp, _ptr(loss_dev)))

    def backward(self, Ws, dWs, dbs=None):
        """dbs: the L bias gradients db^l (f_l floats each, device) of a bias=True model."""
        wp, _a = _parr(Ws)
        dp, _b = _parr(dWs)
        bp, _c2 = _parr(dbs) if dbs is not None else (None, None)
        self.ctx._c(_lib.rdm_gcn_backward(self.h, wp, dp, bp))

    def info(self) -> dict:
        i = RdmGcnInfo()
        self.ctx._c(_lib.rdm_gcn_get_info(self.h, ctypes.byref(i)))
        return i.as_dict()

    def describe(self) -> str:
        buf = ctypes.create_string_buffer(1 << 16)
        self.ctx._c(_lib.rdm_gcn_describe(self.h, buf, len(buf)))
        return buf.value.decode()

    def tensor(self, which, layer, slot=0, layout=ROW):
        """(device pointer, rows, cols, ld) of an internal tensor."""
        p, r, c, ld = ctypes.c_void_p(), _i64(), _i64(), _i64()
        self.ctx._c(_lib.rdm_gcn_tensor(self.h, which, layer, slot, layout, ctypes.byref(p),
                                        ctypes.byref(r), ctypes.byref(c), ctypes.byref(ld)))
        return p.value, r.value, c.value, ld.value

    def tensor_torch(self, which, layer, slot=0, layout=ROW):
        """Copy of an internal tensor as a torch tensor (rows x cols)."""
        import torch
        p, r, c, ld = self.tensor(which, layer, slot, layout)
        self.ctx.sync()
        if r * ld == 0:
            return torch.zeros((r, c), dtype=torch.float32, device=f"cuda:{self.ctx.device}")

        class _View:  # zero-copy view of library memory via __cuda_array_interface__
            __cuda_array_interface__ = {"shape": (r, ld), "typestr": "<f4", "data": (p, False),
                                        "version": 3, "strides": None}

        view = torch.as_tensor(_View(), device=f"cuda:{self.ctx.device}")
        return view[:, :c].clone()


def _dev_view(ptr, shape, typestr, device):
    """Zero-copy torch view of library device memory (via __cuda_array_interface__)."""
    import torch

    class _View:
        __cuda_array_interface__ = {"shape": tuple(shape), "typestr": typestr, "data": (ptr, False),
                                    "version": 3, "strides": None}

    return torch.as_tensor(_View(), device=device)


class Saint:
    """GraphSAINT-RDM random-walk sampler (rdm.h rdm_saint_*): `roots` walks of
    `walk_len` steps from the shared `seed`; every rank samples the same subgraph."""

    def __init__(self, ctx: Context, roots, walk_len=4, seed=1):
        self.ctx = ctx
        h = ctypes.c_void_p()
        ctx._c(_lib.rdm_saint_create(ctx.h, int(roots), int(walk_len), ctypes.c_uint64(seed),
                                     ctypes.byref(h)))
        self.h = h

    def sample(self, iteration):
        n, nnz = _i64(), _i64()
        self.ctx._c(_lib.rdm_saint_sample(self.h, int(iteration), ctypes.byref(n), ctypes.byref(nnz)))
        return n.value, nnz.value

    def wait(self):
        """The context's stream waits for the latest subgraph build (rdm.h rdm_saint_wait)."""
        self.ctx._c(_lib.rdm_saint_wait(self.h))

    def subgraph(self):
        """Copies of the current subgraph: nodes, rowptr, col, val (torch, on the device)."""
        ps = [ctypes.c_void_p() for _ in range(4)]
        n, nnz = _i64(), _i64()
        self.ctx._c(_lib.rdm_saint_subgraph(self.h, *[ctypes.byref(p) for p in ps],
                                            ctypes.byref(n), ctypes.byref(nnz)))
        self.ctx.sync()
        dev = f"cuda:{self.ctx.device}"
        shapes = [(n.value,), (n.value + 1,), (nnz.value,), (nnz.value,)]
        types = ["<i4", "<i8", "<i4", "<f4"]
        import torch
        tt = {"<i4": torch.int32, "<i8": torch.int64, "<f4": torch.float32}
        return tuple(_dev_view(p.value, s, t, dev).clone() if s[0] else
                     torch.zeros(s, dtype=tt[t], device=dev)
                     for p, s, t in zip(ps, shapes, types))

    def gcn(self, f, cfg, input_grad=True, bias=False):
        return GCN(self.ctx, f, cfg, input_grad=input_grad, saint=self, bias=bias)

    def close(self):
        if getattr(self, "h", None):
            _lib.rdm_saint_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


_lib.rdm_saint_create.argtypes = [_vp, _i64, _int, ctypes.c_uint64, ctypes.POINTER(_vp)]
_lib.rdm_saint_destroy.argtypes = [_vp]
_lib.rdm_saint_sample.argtypes = [_vp, _i64, _pi64, _pi64]
_lib.rdm_saint_subgraph.argtypes = [_vp, _pp, _pp, _pp, _pp, _pi64, _pi64]
_lib.rdm_saint_gcn_create.argtypes = [_vp, _int, _pi64, ctypes.POINTER(RdmConfig), _int,
                                      ctypes.POINTER(_vp)]
_lib.rdm_saint_set_input.argtypes = [_vp, _vp, _i64, _vp, _vp]
for _n in ("rdm_saint_create", "rdm_saint_destroy", "rdm_saint_sample", "rdm_saint_subgraph",
           "rdm_saint_gcn_create", "rdm_saint_set_input"):
    getattr(_lib, _n).restype = _int
    EXPORTS.append(_n)


class RdmGraphInfo(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int64) for n in ("n", "nnz", "n_light_rows", "n_heavy_rows",
                                               "n_segments", "max_degree", "core_K", "core_nnz")] + \
               [("symmetric", ctypes.c_int)] + \
               [(k, ctypes.c_int64) for k in ("tile_ranks", "n_tiles", "n_tile_items")]

    def as_dict(self):
        return {n: getattr(self, n) for n, _ in self._fields_}


_lib.rdm_get_graph_info.argtypes = [_vp, ctypes.POINTER(RdmGraphInfo)]
_lib.rdm_get_graph_info.restype = _int
EXPORTS.append("rdm_get_graph_info")


def _graph_info(self) -> dict:
    gi = RdmGraphInfo()
    self._c(_lib.rdm_get_graph_info(self.h, ctypes.byref(gi)))
    return gi.as_dict()


Context.graph_info = _graph_info
