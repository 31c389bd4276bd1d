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
    ps = [ctx.Process(target=worker, args=(r, 2, 0, cases, q, port,
                                           dict(single_gpu_nccl_env(r), SF_MULTIGPU_C5_FULL="small")))
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
    # xpush kernels of one rank spin on flags the other rank's kernels set: on ONE GPU two
    # processes' waiting kernels are not guaranteed to be co-resident (the profiling guide
    # records Xid 109 context-switch timeouts for exactly that), so the concurrent peer-push
    # case runs only where each rank has its own GPU (tests/test_multigpu.py)
    cases = [c for c in CASES if not c[2]]
    out = _run_two_ranks(cases)
    print("\n".join(out))
    assert len(out) == 2 + len(cases)


def test_bench_multirank_path_two_processes(cuda_device):
    """bench.py --gpus 2 (the driver's multi-GPU launch: it re-executes itself under
    torch.distributed.run) runs end to end on one GPU with SF_BENCH_SHARE_GPU=1 (both ranks
    on cuda:0, NCCL across "hosts"): torch's NCCL process group, the library's NCCL halo
    exchange inside run_fused, the max-over-ranks timing and the e2e leg; rank 0 prints one
    JSON line with n_gpus 2, z-slab x2 and NCCL exchange.  C2 (small) keeps it quick."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, SF_BENCH_SHARE_GPU="1")
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--steps", "3",
                        "--warmup", "3", "--workload", "C2", "--no-cpu"], capture_output=True, text=True,
                       timeout=900, env=env, cwd=root)
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert r.returncode == 0 and len(lines) == 1, r.stdout[-3000:] + r.stderr[-3000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["config"]["parallelism"] == "z-slab x2"
    assert d["config"]["halo_exchange"] == "NCCL send/recv" and d["gpu_launches"] > 0
    assert "functional_test" in d
