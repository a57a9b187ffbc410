"""CPU oracle for the GNN-RDM hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import, call, link or
execute anything under ``oracle/``.  The product path
(``paper_conf_ipps_kurtysps23_b200``) never imports it and shares no code,
headers, tables or helpers with it; the only common dependency is the seeded
input generator module ``synth/`` (which holds none of the method's
arithmetic).

Contents (each function cites the PAPER.md passage it follows):

* ``gcn``           — fp64 GCN forward / loss / backward / Adam, the plain
                       definition of eqs. (1)–(4).
* ``cost_model``    — layout-tracking redistribution / sparse-op simulator,
                       Pareto filter (§IV-A/B, Tables II–IV, VI).
* ``redistribution``— partition rules and the virtual-rank row↔column
                       redistribution as a pure index map (§III-D, Fig. 7).

Pins (tests/test_oracle_*.py, ``-m "not gpu"``): scipy.sparse products,
torch.autograd gradients, central finite differences, associativity,
closed forms (Â = I, W^L = 0 → ℓ = ln C, complete graph, empty rows, star),
printed Table IV / Table VI values (tests/golden/).  Functions without a pin
are listed as "parity unpinned" in DESIGN.md; at the time of writing there
are none on the hot path.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def build():
    src = os.path.join(_HERE, "spmm.c")
    subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11", src,
                           "-o", _LIB_PATH])


def lib():
    """Load (building on first use) the fp64 C kernels of the oracle."""
    global _lib
    if _lib is None:
        src = os.path.join(_HERE, "spmm.c")
        if (not os.path.exists(_LIB_PATH)) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
            build()
        L = ctypes.CDLL(_LIB_PATH)
        vp, i64 = ctypes.c_void_p, ctypes.c_int64
        L.oracle_spmm.argtypes = [i64, vp, vp, vp, vp, i64, vp]
        L.oracle_spmm_t.argtypes = [i64, vp, vp, vp, vp, i64, vp]
        L.oracle_spmm_rows.argtypes = [vp, vp, vp, vp, i64, i64, vp, i64, vp]
        L.oracle_num_threads.restype = ctypes.c_int
        L.oracle_set_threads.argtypes = [ctypes.c_int]
        _lib = L
    return _lib
