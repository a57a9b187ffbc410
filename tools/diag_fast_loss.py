"""Diagnostic: relative loss error of the fast variant vs the fp64 oracle on the
Cora-shaped problem (tests/test_gpu_gcn._problem) for several configurations and
P, under the environment given (RDM_TILE_PIECES_FAST, RDM_BF16_WIRE)."""
import os, sys
sys.path.insert(0, '.')
sys.path.insert(0, 'tests')
import numpy as np
import paper_conf_ipps_kurtysps23_b200 as rdm
from oracle import gcn as og
from test_gpu_gcn import _problem, _run
g, H0, Ws, y, m = _problem()
ref = og.forward(g, H0, Ws, y, m)
out = []
for P in (1, 2, 4):
    for cfg in (2, 3, 5, 10, 15):
        loss, dW, model, ctx, _ = _run(rdm, g, H0, Ws, y, m, cfg, P=P, precision="fast")
        out.append(f"P{P}/ID{cfg}: {abs(loss - ref.loss) / abs(ref.loss):.2e}")
        model.close(); ctx.close()
print(os.environ.get("RDM_TILE_PIECES_FAST"), os.environ.get("RDM_BF16_WIRE"), " ".join(out), flush=True)
