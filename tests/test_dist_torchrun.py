"""Multi-process NCCL test of the dist layer: torchrun with one
rank per visible GPU (capped at 8; a one-GPU box runs world = 1).  Every rank
checks Y_full bit for bit against the single-GPU result for both the
grouped-broadcast all-gather and the fused peer-store path, and sampled rows
against the oracle (tests/dist_worker.py)."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("sym", ["window", "ipc"])
def test_dist_torchrun_bitwise_vs_single_gpu(sym):
    world = max(1, min(8, torch.cuda.device_count()))
    env = dict(os.environ)
    if sym == "ipc":
        env["TLP_SYM"] = "ipc"
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr=127.0.0.1", f"--master-port={_port()}",
           os.path.join(ROOT, "tests", "dist_worker.py")]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    assert r.returncode == 0, (r.stdout[-2000:], r.stderr[-4000:])
    line = [ln for ln in r.stdout.splitlines() if ln.startswith("{")][-1]
    d = json.loads(line)
    assert d["world"] == world
    assert all(v <= 1.0 for v in d["worst_err_over_tol"].values())
    assert (d["symmetric_buffer"] == "ipc") == (sym == "ipc"), d["symmetric_buffer"]
