"""One rank per GPU over NVLink with the library's NCCL transport.

Selected only with `-m multigpu` (conftest.py deselects it otherwise): it needs a box
with >= 2 GPUs, e.g.
    python -m pytest tests -m multigpu            (uses every visible GPU, up to 8)
It launches tests/_nccl_worker.py under torchrun (127.0.0.1 rendezvous) and requires
every check to pass on every rank: exchange_halos on rank-encoded planes, and
run_fused / run_unfused (C2, C3, C4, C5; C4 with peer push) bit-exact with the single
domain (P9).  bench.py --gpus N runs the weak-scaling measurement on the same path.
"""
import os
import socket
import subprocess
import sys

import pytest

pytestmark = [pytest.mark.gpu, pytest.mark.multigpu]
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _ngpus():
    import torch
    return torch.cuda.device_count()


@pytest.mark.parametrize("n,c5_full", [(2, False), (4, False), (8, False), (8, True)],
                         ids=["2", "4", "8", "8-C5-1024cubed"])
def test_torchrun_nccl_ranks(n, c5_full):
    """c5_full: additionally BASELINE configs[4] at full size (1024^3 fp64 over 8 GPUs),
    bit-exact against the undecomposed grid run on GPU 0 (tests/_nccl_worker.check_c5_full)."""
    have = _ngpus()
    if have < n:
        pytest.skip(f"needs {n} GPUs, {have} visible")
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr=127.0.0.1", f"--master-port={port}",
           os.path.join(ROOT, "tests", "_nccl_worker.py")]
    env = dict(os.environ, SF_MULTIGPU_C5_FULL="1" if c5_full else "0")
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=3600, env=env)
    print(r.stdout[-4000:])
    assert r.returncode == 0 and "MULTIGPU_OK" in r.stdout, r.stderr[-4000:]
