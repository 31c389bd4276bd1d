"""Multi-rank checks over the library's REAL NCCL transport (comm.cpp: ncclSend/ncclRecv
inside ncclGroupStart/End on the communicator's stream), one process per rank.

Run two ways:
  * tests/test_gpu_nccl.py: two processes on ONE GPU.  NCCL refuses two ranks on one
    device within one host ("Duplicate GPU"), so each process announces its own host id
    (NCCL_HOSTID) and the ranks talk through NCCL's socket transport over loopback;
    everything above the wire (ncclCommInitRank, group calls, stream ordering, the
    executor's exchange schedule and interior/boundary overlap) is the production path.
  * tests/test_multigpu.py / `torchrun --nproc-per-node N tests/_nccl_worker.py`: one
    rank per GPU over NVLink (the deployment shape).

Checks (pin P9):
  1. exchange_halos on rank-encoded planes: every ghost plane equals the neighbour's
     interior plane, nothing else is touched;
  2. run_fused / run_unfused of C2, C4, C5 slabs (two steps) gathered == the single
     domain bit for bit; optionally with peer push (xpush) for TEMP epochs.
torch.distributed (gloo) only bootstraps the NCCL id and gathers results.
"""
from __future__ import annotations

import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
for _p in (ROOT, os.path.join(ROOT, "tests")):
    if _p not in sys.path:
        sys.path.insert(0, _p)


def single_gpu_nccl_env(rank):
    """Environment for two NCCL ranks sharing one GPU (see module docstring)."""
    return {"NCCL_HOSTID": f"stencilfuse-rank{rank}", "NCCL_SOCKET_IFNAME": "lo",
            "NCCL_IB_DISABLE": "1", "NCCL_P2P_DISABLE": "1", "NCCL_SHM_DISABLE": "1",
            "NCCL_NVLS_ENABLE": "0", "NCCL_COLLNET_ENABLE": "0"}


def encoded(aid, gz, shape, device="cuda"):
    """Exact fp64 code of (array, global plane, y, x) for the whole allocated plane."""
    import torch
    y = torch.arange(shape[0], dtype=torch.float64, device=device)[:, None]
    x = torch.arange(shape[1], dtype=torch.float64, device=device)[None, :]
    return ((aid * 1000.0 + (gz + 100)) * 1000.0 + y) * 1000.0 + x


def check_exchange_halos(rank, world, dev):
    import torch
    from paper_conf_hpdc_wahibm15_b200 import Comm, Program
    from synth import programs as P
    nzl, depth = 7, 3
    prog = P.c2(nx=40, ny=24, nz=nzl)
    comm = Comm(rank, world)
    p = Program(prog, comm=comm, nz_global=nzl * world, z_offset=rank * nzl, zhalo=depth)
    p.allocate(dev)  # NaN everywhere
    oz = p.layout["origin_z"]
    names = p.names
    for aid, n in enumerate(names):
        t = p.tensors[n]
        for z in range(nzl):
            t[oz + z].copy_(encoded(aid, rank * nzl + z, t.shape[1:], t.device).to(t.dtype))
    before = {n: p.tensors[n].clone() for n in names}
    s = torch.cuda.Stream(device=dev)
    p.exchange_halos(names, depth, s)
    s.synchronize()
    for aid, n in enumerate(names):
        t = p.tensors[n]
        for z in range(-depth, nzl + depth):
            gz = rank * nzl + z
            got = t[oz + z]
            if 0 <= z < nzl or gz < 0 or gz >= nzl * world:
                # interior planes and true global ghost planes are never touched
                assert torch.equal(got.nan_to_num(-1), before[n][oz + z].nan_to_num(-1)), (n, z)
            else:
                want = encoded(aid, gz, t.shape[1:], t.device).to(t.dtype)
                assert torch.equal(got, want), f"rank {rank} {n} ghost plane {z} (global {gz})"
    del p, comm
    return "exchange_halos ok"


def check_run(rank, world, dev, cfg, mode, xpush=False, nzl=12, steps=2, grid=None):
    import torch
    import torch.distributed as dist
    from paper_conf_hpdc_wahibm15_b200 import Comm, Program
    from test_gpu_multirank import MK, fill
    mk = MK[cfg] if grid is None else grid
    loc = mk(nzl)
    plan = loc["plans"]["fused"]
    probe = Program(loc, nz_global=nzl * world)
    probe.set_plan(plan)
    zhalo = max([max(r["z_below"], r["z_above"]) for m in ("fused", "unfused")
                 for r in probe.reports(m)] + [loc["grid"]["ghost"][2]])
    del probe
    comm = Comm(rank, world)
    s = Program(loc, comm=comm, nz_global=nzl * world, z_offset=rank * nzl, zhalo=zhalo,
                options={"xpush": 1} if xpush else None)
    s.set_plan(plan)
    s.allocate(dev)
    fill(s, loc, dev, rank * nzl, zhalo, nz_global=nzl * world)
    if xpush:
        s.connect_peers(rank, world)
    s.load(mode)
    torch.cuda.synchronize(dev)
    dist.barrier()
    st = torch.cuda.Stream(device=dev)
    for _ in range(steps):
        s.run(mode, st)
    st.synchronize()
    outs = [a["name"] for a in loc["arrays"] if a["role"] in ("out", "inout")]
    mine = {n: s.interior_view(s.tensors[n]).cpu() for n in outs}
    got = [None] * world if rank == 0 else None
    dist.gather_object(mine, got, dst=0)
    msg = f"{cfg} {mode}{' xpush' if xpush else ''} x{world}: ok"
    if rank == 0:
        glob = mk(nzl * world)
        single = Program(glob)
        single.set_plan(plan)
        single.allocate(dev)
        fill(single, glob, dev, 0, glob["grid"]["ghost"][2])
        for _ in range(steps):
            single.run(mode)
        torch.cuda.synchronize(dev)
        for n in outs:
            want = single.interior_view(single.tensors[n]).cpu()
            have = torch.cat([g[n] for g in got], dim=0)
            assert torch.equal(have, want), f"{cfg} {mode} {n}: NCCL multi-rank result differs"
        del single
    dist.barrier()
    del s, comm
    return msg


def check_c5_full(rank, world, dev, steps=1, n=1024, nz_total=1024):
    """BASELINE configs[4] at full size: C5 (3 tracers x gradient/flux/divergence/update,
    12 kernels) on 1024 x 1024 x 128 planes per GPU, 1024^3 fp64 in total at 8 ranks,
    fused plan, real NCCL halo exchange overlapped with the interior planes.  P9 at full
    scale: rank 0 also runs the undecomposed 1024^3 grid on its GPU (~138 GB of HBM) and
    compares SHA-1 digests of every rank's OUT slab with the same planes of the single
    domain (bit for bit)."""
    import hashlib
    import torch
    import torch.distributed as dist
    import bench
    from paper_conf_hpdc_wahibm15_b200 import Comm, Program
    from synth import programs as P
    nzl = nz_total // world
    loc = P.c5(nx=n, ny=n, nz=nzl)
    plan = loc["plans"]["fused"]
    probe = Program(loc, nz_global=nzl * world)
    probe.set_plan(plan)
    zhalo = max([max(r["z_below"], r["z_above"]) for r in probe.reports("fused")] + [1])
    del probe
    comm = Comm(rank, world)
    s = Program(loc, comm=comm, nz_global=nzl * world, z_offset=rank * nzl, zhalo=zhalo)
    s.set_plan(plan)
    s.allocate(dev, fill=0.0)
    bench.fill_inputs(s, loc, dev, rank * nzl, zhalo)
    s.load("fused")
    torch.cuda.synchronize(dev)
    dist.barrier()
    for _ in range(steps):
        s.run_fused()
    torch.cuda.synchronize(dev)
    outs = [a["name"] for a in loc["arrays"] if a["role"] in ("out", "inout")]
    mine = {nm: hashlib.sha1(s.interior_view(s.tensors[nm]).cpu().numpy().tobytes()).hexdigest()
            for nm in outs}
    del s, comm
    torch.cuda.empty_cache()
    got = [None] * world if rank == 0 else None
    dist.gather_object(mine, got, dst=0)
    if rank == 0:
        glob = P.c5(nx=n, ny=n, nz=nzl * world)
        single = Program(glob)
        single.set_plan(plan)
        single.allocate(dev, fill=0.0)
        bench.fill_inputs(single, glob, dev, 0, glob["grid"]["ghost"][2])
        for _ in range(steps):
            single.run_fused()
        torch.cuda.synchronize(dev)
        for nm in outs:
            full = single.interior_view(single.tensors[nm])
            for r in range(world):
                want = hashlib.sha1(full[r * nzl:(r + 1) * nzl].cpu().numpy().tobytes()).hexdigest()
                assert got[r][nm] == want, f"C5 {n}^2x{nz_total} x{world}: {nm} slab {r} differs"
        del single
    dist.barrier()
    return f"C5 {n}^2x{nz_total} fused x{world}: bit-exact with the single domain (SHA-1 per slab)"


CASES = [("C2", "fused", False), ("C2", "unfused", False), ("C4", "fused", False),
         ("C4", "unfused", False), ("C5", "fused", False), ("C3", "fused", False),
         ("C4", "fused", True)]


def worker(rank, world, device_index, cases=None, q=None, port=None, env=None):
    """Entry of one rank.  `port` set: bootstrap gloo at 127.0.0.1:port (spawned test);
    otherwise torchrun's environment."""
    for k, v in (env or {}).items():
        os.environ[k] = v
    import torch
    import torch.distributed as dist
    if port is not None:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
    else:
        dist.init_process_group("gloo")
    out = []
    try:
        dev = torch.device("cuda", device_index)
        torch.cuda.set_device(dev)
        out.append(check_exchange_halos(rank, world, dev))
        for cfg, mode, xpush in (CASES if cases is None else cases):
            out.append(check_run(rank, world, dev, cfg, mode, xpush))
        if os.environ.get("SF_MULTIGPU_C5_FULL") == "1" and world == 8:
            out.append(check_c5_full(rank, world, dev))
        elif os.environ.get("SF_MULTIGPU_C5_FULL") == "small":  # the same check, reduced
            out.append(check_c5_full(rank, world, dev, n=96, nz_total=48 * world))
        if q is not None:
            q.put((rank, "ok", out))
    except Exception:
        import traceback
        if q is not None:
            q.put((rank, "error", traceback.format_exc()))
        else:
            raise
    finally:
        dist.destroy_process_group()
    return out


if __name__ == "__main__":  # torchrun --nproc-per-node N tests/_nccl_worker.py
    r = int(os.environ["RANK"])
    res = worker(r, int(os.environ["WORLD_SIZE"]), int(os.environ.get("LOCAL_RANK", "0")))
    if r == 0:
        print("\n".join(res))
        print("MULTIGPU_OK", flush=True)
