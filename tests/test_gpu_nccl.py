"""The NCCL halo-exchange transport, executed (pin P9).

Two processes share cuda:0 and form a real NCCL communicator through
sp_comm_create (ncclCommInitRank), each announcing its own host id so NCCL accepts
two ranks on one device (its socket transport then carries the planes over
loopback).  tests/_nccl_worker.py drives, in both processes:
  * exchange_halos on rank-encoded planes (ghost planes == the neighbour's interior
    planes, interior and true global ghosts untouched);
  * run_fused / run_unfused with the communicator (the executor's exchange schedule,
    interior launch overlapped with ncclSend/ncclRecv on the comm stream, boundary
    launch after it; xpush: TEMP epochs pushed by the kernels over CUDA IPC, IN
    epochs through NCCL), two steps, gathered == the single domain bit for bit.
The same worker runs one rank per GPU under torchrun in tests/test_multigpu.py.
"""
import os
import socket

import pytest

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _run_two_ranks(cases, timeout=900):
    import multiprocessing as mp
    from _nccl_worker import single_gpu_nccl_env, worker
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=worker, args=(r, 2, 0, cases, q, port, single_gpu_nccl_env(r)))
          for r in range(2)]
    for p in ps:
        p.start()
    res = {}
    try:
        for _ in range(2):
            r, status, out = q.get(timeout=timeout)
            res[r] = (status, out)
    finally:
        for p in ps:
            p.join(timeout=30)
            if p.is_alive():  # the exact processes this test started
                p.kill()
    for r, (status, out) in sorted(res.items()):
        assert status == "ok", f"rank {r}:\n{out}"
    return res[0][1]


def test_nccl_exchange_halos_and_runs_two_processes(cuda_device):
    from _nccl_worker import CASES
    out = _run_two_ranks(CASES)
    print("\n".join(out))
    assert len(out) == 1 + len(CASES)
