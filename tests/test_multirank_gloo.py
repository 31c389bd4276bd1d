"""N > 1 host path on CPU: world_size 2 over gloo (pin P9).

Each rank creates its z-slab Program (nz_global, z_offset, deep halo zhalo — the
library's host side: layout, plan analysis, exchange schedule), bootstraps the
NCCL-id broadcast path of Comm's helper over gloo, and then executes the plan
group by group with the CPU oracle standing in for the GPU kernels: before each
group it exchanges exactly the arrays and depth that sp_plan_exchange names, with
torch.distributed send/recv of contiguous z-planes, then evaluates the group's
statements on its slab extended by the deep halo (clipped to the global interior).
Rank 0 gathers the OUT arrays and compares them bit for bit with the oracle on the
undecomposed grid.  This checks that the library's exchange schedule and deep-halo
depth are sufficient for the fused plan, independently of the GPU.
"""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.host


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, cfg, q, shrink=0):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    sys.path.insert(0, os.path.join(root, "tests"))
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import OracleProgram
        from paper_conf_hpdc_wahibm15_b200 import Program
        from synth import programs as P
        from synth.fields import field
        nzl = 10
        mk = {"C2": lambda nz: P.c2(nx=12, ny=9, nz=nz),
              "C3": lambda nz: P.c3(nx=14, ny=8, nz=nz),
              "C5": lambda nz: P.c5(nx=10, ny=8, nz=nz),
              "chain3": lambda nz: P.resize(P.chain3(), 9, 7, nz)}[cfg]
        loc = mk(nzl)
        plan = loc["plans"]["fused"] if cfg != "C3" else loc["plans"]["fission_fused"]
        probe = Program(loc)
        probe.set_plan(plan)
        D = max([max(r["z_below"], r["z_above"]) for r in probe.reports("fused")] + [1])
        prog = Program(loc, nz_global=nzl * world, z_offset=rank * nzl, zhalo=D)
        prog.set_plan(plan)
        assert prog.layout["origin_z"] == D
        # the NCCL unique-id broadcast path of Comm, over gloo
        buf = torch.arange(128, dtype=torch.uint8) if rank == 0 else torch.zeros(128, dtype=torch.uint8)
        dist.broadcast(buf, src=0)
        assert torch.equal(buf, torch.arange(128, dtype=torch.uint8))
        hx, hy, hz = loc["grid"]["ghost"]
        # slab extended by the deep halo as the oracle's "interior": planes p <-> global z = z0 - D + p
        ext = (loc["grid"]["nx"], loc["grid"]["ny"], nzl + 2 * D)
        z0 = rank * nzl
        arrs = {}
        for aid, a in enumerate(loc["arrays"]):
            arrs[a["name"]] = np.ascontiguousarray(
                field(21, aid, ext, (hx, hy, hz), loc["dtype"], z_offset=z0 - D))
        # a rank holds no neighbour data until exchanged: deep-halo planes that are
        # global interior start poisoned (true global ghosts keep their values)
        for a in arrs.values():
            for pz in list(range(0, D)) + list(range(D + nzl, nzl + 2 * D)):
                if 0 <= z0 - D + pz < nzl * world:  # x-y ghosts are physical (R1)
                    a[hz + pz, hy:hy + ext[1], hx:hx + ext[0]] = np.nan
        box_k = (max(0, D - z0), min(nzl + 2 * D, nzl * world - z0 + D))
        sub_programs = []
        names = [k["name"] for k in loc["kernels"]]
        for gi, grp in enumerate(plan):
            stmts = []
            for ref in grp:
                if ":" in ref:
                    k, s = ref.rsplit(":", 1)
                    stmts.append(loc["kernels"][names.index(k)]["stmts"][int(s)])
                else:
                    stmts += loc["kernels"][names.index(ref)]["stmts"]
            sub = dict(loc, kernels=[{"name": f"g{gi}", "stmts": [st]} for st in stmts])
            sub["grid"] = dict(loc["grid"], nz=ext[2])
            sub_programs.append(OracleProgram(sub))

        def planes(a, p0, n):  # dense planes p0..p0+n of the extended window (incl. ghost hz)
            return a[hz + p0:hz + p0 + n]

        for gi in range(len(plan)):
            xs = prog.exchange_plan("fused", gi)
            reqs = []
            dt = torch.float64 if loc["dtype"] == "f64" else torch.float32
            for n, below, above in xs:
                below, above = max(0, below - shrink), max(0, above - shrink)
                a = arrs[n]
                if rank + 1 < world:   # my top `below` planes -> up's bottom ghost; up's bottom -> my top
                    if below:
                        dist.send(torch.from_numpy(planes(a, D + nzl - below, below).copy()), dst=rank + 1)
                    if above:
                        recv = torch.empty(planes(a, 0, above).shape, dtype=dt)
                        dist.recv(recv, src=rank + 1)
                        planes(a, D + nzl, above)[...] = recv.numpy()
                if rank > 0:
                    if below:
                        recv = torch.empty(planes(a, 0, below).shape, dtype=dt)
                        dist.recv(recv, src=rank - 1)
                        planes(a, D - below, below)[...] = recv.numpy()
                    if above:
                        dist.send(torch.from_numpy(planes(a, D, above).copy()), dst=rank - 1)
            del reqs
            box = (0, ext[0], 0, ext[1], box_k[0], box_k[1])
            sub_programs[gi].run(arrs, box=box, n=ext)
            if os.environ.get("SF_DEBUG_GLOO"):
                for n, a in arrs.items():
                    own = a[hz + D:hz + D + nzl]
                    if np.isnan(own).any():
                        print(f"rank {rank} after group {gi} exchange {xs}: {n} own NaN planes "
                              f"{sorted(set(np.argwhere(np.isnan(own))[:, 0].tolist()))}", flush=True)
        outs = [a["name"] for a in loc["arrays"] if a["role"] in ("out", "inout")]
        mine = {n: arrs[n][hz + D:hz + D + nzl, hy:hy + ext[1], hx:hx + ext[0]].copy() for n in outs}
        gathered = [None] * world if rank == 0 else None
        dist.gather_object(mine, gathered, dst=0)
        if rank == 0:
            glob = mk(nzl * world)
            g = {}
            for aid, a in enumerate(glob["arrays"]):
                g[a["name"]] = np.ascontiguousarray(field(21, aid, (glob["grid"]["nx"], glob["grid"]["ny"],
                                                                    nzl * world), (hx, hy, hz), glob["dtype"]))
            OracleProgram(glob).run(g)
            ok = True
            for n in outs:
                want = g[n][hz:hz + nzl * world, hy:hy + ext[1], hx:hx + ext[0]]
                got = np.concatenate([gathered[r][n] for r in range(world)], axis=0)
                same = got.tobytes() == want.tobytes()
                if not same:
                    bad = np.argwhere(~(got == want))
                    print(f"[{cfg}] {n}: {len(bad)} differing points, first {bad[:3].tolist()}, "
                          f"nan {int(np.isnan(got).sum())}", flush=True)
                ok &= same
            q.put(("ok" if ok else "mismatch", D))
    except Exception as e:  # noqa: BLE001
        if rank == 0:
            q.put(("error", repr(e)))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("cfg", ["C2", "C3", "C5", "chain3"])
def test_two_rank_slab_execution_matches_global(cfg):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, cfg, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
    res = q.get(timeout=10)
    assert res[0] == "ok", res
    assert all(p.exitcode == 0 for p in procs)


def test_too_shallow_exchange_is_detected():
    """Mutation check of the harness: one plane less than the schedule must break P9."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, "chain3", q, 1)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=300)
    assert q.get(timeout=10)[0] == "mismatch"
