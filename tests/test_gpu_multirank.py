"""Real multi-GPU execution of the NCCL data plane (one process per GPU).

Runs only where at least two CUDA devices are visible (skipped on the
one-GPU boxes): torchrun launches tests/mgpu_worker.py on P = 2 and on all
visible GPUs (up to 8).  Each rank exercises grouped ncclSend/ncclRecv
redistributions, ncclAllReduce of Y^l and the loss, and the CUDA-IPC
peer-store (P2P) transport, and checks itself against the virtual group on
its own GPU (bit-identical per-rank tensors) and the fp64 oracle
(PAPER.md L140-142 all-to-all personalized, L212 Fig. 7, L295 NCCL)."""
import glob
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _ngpu():
    import torch
    return torch.cuda.device_count() if torch.cuda.is_available() else 0


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("P", [2, 4, 8])
def test_nccl_ranks_match_virtual_group_and_oracle(P, tmp_path):
    if _ngpu() < P:
        pytest.skip(f"needs {P} GPUs, {_ngpu()} visible")
    env = dict(os.environ, RDM_MGPU_OUT=str(tmp_path), MASTER_ADDR="127.0.0.1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={P}",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()),
           os.path.join(ROOT, "tests", "mgpu_worker.py")]
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=900, cwd=ROOT)
    outs = sorted(glob.glob(str(tmp_path / "rank*.json")))
    assert len(outs) == P, (r.returncode, r.stdout[-2000:], r.stderr[-4000:])
    for fn in outs:
        res = json.load(open(fn))
        assert res["ok"], res.get("error")
        assert res["nccl"]["ranks"] == P
        assert len(res["checks"]) == 10
    assert r.returncode == 0, r.stderr[-4000:]
