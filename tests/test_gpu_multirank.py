"""z-slab decomposition on ONE GPU ("virtual ranks", test-only).

Each rank is a Program over its slab (nz_global, z_offset, deep halo zhalo) with no
communicator; before every fused group the test moves the ghost planes the library's
exchange schedule names (sp_plan_exchange: arrays, planes below/above) between the slab tensors
with device-to-device copies — exactly the planes run_fused would ncclSend/ncclRecv.
The P-rank result must equal the single-domain result bit for bit: initialisation is
a function of global coordinates and the fused kernels recompute intermediates on
deep-halo planes that are global interior (reading R1).
"""
import json
import os

import pytest

from synth import programs as P
from synth.fields import field_torch

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def c4_small(nz):
    from synth.scale_les import c4
    prog = c4(nx=64, ny=32, nz=nz)
    prog["plans"]["fused"] = json.load(open(os.path.join(ROOT, "configs", "c4_plan.json")))["groups"]
    return prog


def fill(p, prog, dev, z_offset, zhalo, nz_global=None):
    hz = p.ghost[2]
    nzl = p.n[2]
    for aid, a in enumerate(prog["arrays"]):
        v = field_torch(13, aid, p.n, p.ghost, prog["dtype"], dev, z_offset=z_offset,
                        nz_alloc_extra=(zhalo - hz, zhalo - hz))
        if nz_global is not None:
            # no neighbour data before an exchange: poison deep-halo planes that are global interior
            for pz in list(range(zhalo)) + list(range(zhalo + nzl, nzl + 2 * zhalo)):
                if 0 <= z_offset - zhalo + pz < nz_global:  # x-y ghosts are physical (R1)
                    hx, hy = p.ghost[0], p.ghost[1]
                    v[pz, hy:hy + p.n[1], hx:hx + p.n[0]] = float("nan")
        p.padded_view(p.tensors[a["name"]], hz=zhalo).copy_(v)


def plane(p, t, z, depth):
    """Planes [z, z+depth) (local interior coordinates) of an allocation."""
    oz = p.layout["origin_z"]
    return t[oz + z:oz + z + depth]


def c2_boxed(nz):
    """C2 whose update kernel has loop bounds (reading R2') crossing the slab boundary
    (global z in [5, 20) for 2 x 12 planes), so boxed stages meet deep-halo planes."""
    prog = P.c2(nx=40, ny=24, nz=nz)
    prog["kernels"][3]["box"] = [3, 30, 2, 20, 5, 20]
    return prog


@pytest.mark.parametrize("cfg,ranks", [("C2", 2), ("C5", 3), ("C3", 2), ("C4", 2), ("chain3", 3),
                                       ("C2box", 2), ("chain3box", 2), ("chain3box", 3)])
@pytest.mark.parametrize("fmad", [0, 1])
def test_virtual_ranks_bitexact(cuda_device, cfg, ranks, fmad):
    import torch
    from paper_conf_hpdc_wahibm15_b200 import Program
    nzl = 12
    mk = {"C2": lambda nz: P.c2(nx=40, ny=24, nz=nz), "C5": lambda nz: P.c5(nx=32, ny=16, nz=nz),
          "C3": lambda nz: P.c3(nx=48, ny=20, nz=nz), "C4": c4_small,
          "chain3": lambda nz: P.resize(P.chain3(), 20, 12, nz), "C2box": c2_boxed,
          "chain3box": chain3_boxed}[cfg]
    glob = mk(nzl * ranks)
    plan = glob["plans"]["fused"]
    opts = {"fmad": fmad}
    dev = cuda_device
    # single domain
    single = Program(glob, options=opts)
    single.set_plan(plan)
    single.allocate(dev)
    fill(single, glob, dev, 0, glob["grid"]["ghost"][2])
    single.run_fused()
    # slabs
    loc = mk(nzl)
    probe = Program(loc, nz_global=nzl * ranks, options=opts)
    probe.set_plan(plan)
    zhalo = max([max(r["z_below"], r["z_above"]) for r in probe.reports("fused")] +
                [loc["grid"]["ghost"][2]])
    slabs = []
    for r in range(ranks):
        s = Program(loc, nz_global=nzl * ranks, z_offset=r * nzl, zhalo=zhalo, options=opts)
        s.set_plan(plan)
        s.allocate(dev)
        fill(s, loc, dev, r * nzl, zhalo, nz_global=nzl * ranks)
        slabs.append(s)
    for i in range(slabs[0].n_launches("fused")):
        for n, below, above in slabs[0].exchange_plan("fused", i):
            assert below <= zhalo and above <= zhalo
            for r in range(ranks - 1):  # r <-> r+1
                lo, hi = slabs[r], slabs[r + 1]
                if below:
                    plane(hi, hi.tensors[n], -below, below).copy_(plane(lo, lo.tensors[n], nzl - below, below))
                if above:
                    plane(lo, lo.tensors[n], nzl, above).copy_(plane(hi, hi.tensors[n], 0, above))
        for s in slabs:
            s.run_launch("fused", i)
    torch.cuda.synchronize()
    outs = [a["name"] for a in glob["arrays"] if a["role"] in ("out", "inout")]
    for n in outs:
        want = single.interior_view(single.tensors[n])
        got = torch.cat([s.interior_view(s.tensors[n]) for s in slabs], dim=0)
        assert torch.equal(got, want), f"{cfg} {n}: slab result differs from single domain"


@pytest.mark.parametrize("cfg,ranks,mode,opts", [("C2", 2, "fused", {}), ("C5", 3, "fused", {}),
                                                 ("C3", 2, "fused", {}), ("C4", 2, "fused", {}),
                                                 ("C4", 3, "unfused", {}), ("chain3", 3, "fused", {}),
                                                 ("C2box", 2, "fused", {}), ("C2", 3, "unfused", {}),
                                                 ("C4", 4, "fused", {}), ("chain3box", 3, "fused", {}),
                                                 ("C4", 3, "fused", {"fastpath": 1}),
                                                 ("C5", 2, "fused", {"fastpath": 1}),
                                                 ("C3", 3, "unfused", {"fastpath": 1}),
                                                 ("C3", 2, "fused", {"frame": 1}),
                                                 ("C3", 3, "fused", {"frame": 2}),
                                                 ("C2", 2, "fused", {"frame": 1, "fastpath": 1}),
                                                 ("C5", 2, "fused", {"frame": 2}),
                                                 ("C4", 2, "fused", {"psleep": 0})])
def test_loopback_ranks_run_bitexact(cuda_device, cfg, ranks, mode, opts):
    """The executor's own multi-rank path (run_fused / run_unfused with a communicator:
    exchange schedule, interior planes overlapped with the exchange on the comm stream,
    boundary planes after its event, no PDL) on in-process virtual ranks, one host
    thread and one stream each; the loopback transport stands in for ncclSend/ncclRecv.
    Two steps; the result must equal the single-domain result bit for bit (P9)."""
    import threading
    import torch
    from paper_conf_hpdc_wahibm15_b200 import Comm, Program
    nzl = 12
    mk = {"C2": lambda nz: P.c2(nx=40, ny=24, nz=nz), "C5": lambda nz: P.c5(nx=32, ny=16, nz=nz),
          "C3": lambda nz: P.c3(nx=48, ny=20, nz=nz), "C4": c4_small,
          "chain3": lambda nz: P.resize(P.chain3(), 20, 12, nz), "C2box": c2_boxed,
          "chain3box": chain3_boxed}[cfg]
    glob = mk(nzl * ranks)
    plan = glob["plans"]["fused"]
    dev = cuda_device
    single = Program(glob)
    single.set_plan(plan)
    single.allocate(dev)
    fill(single, glob, dev, 0, glob["grid"]["ghost"][2])
    single.run(mode)
    single.run(mode)
    loc = mk(nzl)
    probe = Program(loc, nz_global=nzl * ranks)
    probe.set_plan(plan)
    zhalo = max([max(r["z_below"], r["z_above"]) for m in ("fused", "unfused")
                 for r in probe.reports(m)] + [loc["grid"]["ghost"][2]])
    comms = Comm.loopback(ranks)
    slabs = []
    for r in range(ranks):
        # opts: codegen variants (e.g. the fastpath step body, whose fast-step window must
        # treat deep-halo planes of the global interior like interior planes)
        s = Program(loc, comm=comms[r], nz_global=nzl * ranks, z_offset=r * nzl, zhalo=zhalo,
                    options=opts)
        s.set_plan(plan)
        s.allocate(dev)
        fill(s, loc, dev, r * nzl, zhalo, nz_global=nzl * ranks)
        s.load(mode)  # no module load mid-step (see sp_load)
        slabs.append(s)
    torch.cuda.synchronize()
    errs = []

    def drive(r):
        try:
            st = torch.cuda.Stream(device=dev)
            for _ in range(2):
                slabs[r].run(mode, st)
            st.synchronize()
        except Exception as e:  # surfaced below
            errs.append(e)

    th = [threading.Thread(target=drive, args=(r,)) for r in range(ranks)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    assert not errs, errs
    torch.cuda.synchronize()
    outs = [a["name"] for a in glob["arrays"] if a["role"] in ("out", "inout")]
    for n in outs:
        want = single.interior_view(single.tensors[n])
        got = torch.cat([s.interior_view(s.tensors[n]) for s in slabs], dim=0)
        assert torch.equal(got, want), f"{cfg} {n}: loopback multi-rank result differs from single domain"


def chain3_boxed(nz):
    """chain3 whose K2 (T2, read by K3 one plane above) has loop bounds crossing the slab
    boundaries (global z in [8, 20) of 2-3 x 12 planes, x/y boxes inside the interior): in
    the fused group the boxed stage runs one plane ahead (lead 1), so at a slab's top it is
    evaluated on the neighbour's first plane, where outside its box it loads T2's previous
    value — the exchange schedule must deliver T2's ghost planes (reading R2')."""
    prog = P.resize(P.chain3(), 20, 12, nz)
    prog["kernels"][1]["box"] = [2, 17, 1, 10, 8, 20]
    return prog


MK = {"C2": lambda nz: P.c2(nx=40, ny=24, nz=nz), "C5": lambda nz: P.c5(nx=32, ny=16, nz=nz),
      "C3": lambda nz: P.c3(nx=48, ny=20, nz=nz), "C4": c4_small,
      "chain3": lambda nz: P.resize(P.chain3(), 20, 12, nz), "C2box": c2_boxed,
      "chain3box": chain3_boxed}


@pytest.mark.parametrize("cfg,ranks,mode", [("C3", 2, "fused"), ("C3", 3, "unfused"), ("C4", 2, "fused"),
                                            ("C4", 3, "fused"), ("C4", 2, "unfused"),
                                            ("chain3", 3, "unfused"), ("C2", 2, "unfused"),
                                            ("C2box", 3, "unfused")])
def test_peer_push_lockstep_bitexact(cuda_device, cfg, ranks, mode):
    """Peer-push halo exchange (option xpush, NEXT #2) on virtual ranks: every TEMP
    epoch travels as peer stores from the producing kernel into the neighbours' ghost
    planes, and every kernel runs the progress protocol (edge chunks wait until both
    neighbours completed the previous launch; the last CTA publishes completion).
    One GPU cannot run ranks whose kernels wait on each other concurrently without
    risking a shared hardware queue (a waiting kernel queued ahead of the work it
    waits for), so the ranks' launches are issued in lockstep on one stream — a
    valid schedule of the protocol, in which every wait is already satisfied.  The
    step-start epochs (IN arrays) are copied as sp_plan_exchange names them.  Two
    steps; bit-exact with the single domain (P9)."""
    import torch
    from paper_conf_hpdc_wahibm15_b200 import Comm, Program
    nzl = 12
    mk = MK[cfg]
    glob = mk(nzl * ranks)
    plan = glob["plans"]["fused"]
    dev = cuda_device
    single = Program(glob)
    single.set_plan(plan)
    single.allocate(dev)
    fill(single, glob, dev, 0, glob["grid"]["ghost"][2])
    single.run(mode)
    loc = mk(nzl)
    probe = Program(loc, nz_global=nzl * ranks)
    probe.set_plan(plan)
    zhalo = max([max(r["z_below"], r["z_above"]) for m in ("fused", "unfused")
                 for r in probe.reports(m)] + [loc["grid"]["ghost"][2]])
    comms = Comm.loopback(ranks)
    slabs = []
    for r in range(ranks):
        s = Program(loc, comm=comms[r], nz_global=nzl * ranks, z_offset=r * nzl, zhalo=zhalo,
                    options={"xpush": 1})
        s.set_plan(plan)
        s.allocate(dev)
        fill(s, loc, dev, r * nzl, zhalo, nz_global=nzl * ranks)
        s.load(mode)
        slabs.append(s)
    Program.connect_peers_local(slabs)
    n = slabs[0].n_launches(mode)
    nopush = Program(loc, comm=comms[0], nz_global=nzl * ranks, zhalo=zhalo)
    nopush.set_plan(plan)
    xfers = [slabs[0].exchange_plan(mode, i) for i in range(n)]
    # TEMP epochs left the communicator's schedule (they are pushed)
    temps = {a["name"] for a in loc["arrays"] if a["role"] == "temp"}
    assert not any(a in temps for x in xfers for a, _, _ in x)
    if cfg in ("C4", "C3", "chain3"):
        assert sum(map(len, xfers)) < sum(len(nopush.exchange_plan(mode, i)) for i in range(n))
    torch.cuda.synchronize()
    for step in range(2):
        for i in range(n):
            for a, below, above in xfers[i]:
                for r in range(ranks - 1):
                    lo, hi = slabs[r], slabs[r + 1]
                    if below:
                        plane(hi, hi.tensors[a], -below, below).copy_(plane(lo, lo.tensors[a], nzl - below, below))
                    if above:
                        plane(lo, lo.tensors[a], nzl, above).copy_(plane(hi, hi.tensors[a], 0, above))
            for s in slabs:
                s.run_launch(mode, i)
    torch.cuda.synchronize()
    outs = [a["name"] for a in glob["arrays"] if a["role"] in ("out", "inout")]
    for nm in outs:
        want = single.interior_view(single.tensors[nm])
        got = torch.cat([s.interior_view(s.tensors[nm]) for s in slabs], dim=0)
        assert torch.equal(got, want), f"{cfg} {nm}: peer-push multi-rank result differs from single domain"


def _ipc_worker(rank, world, port, cfg, q, concurrent=False):
    """One process per virtual rank on the same GPU: peer buffers and signal blocks
    wired through CUDA IPC (Program.connect_peers over gloo).  Lockstep: launch i of
    rank r runs after launch i of ranks < r and launch i-1 of all.  Concurrent: after
    the step-start exchange each process enqueues its whole step at once and the
    kernels order themselves through the in-kernel progress protocol (the two
    contexts time-slice the GPU, so a waiting kernel is preempted, not a deadlock)."""
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
        from paper_conf_hpdc_wahibm15_b200 import Comm, Program
        from test_gpu_multirank import MK, fill, plane
        dev = torch.device("cuda:0")
        torch.cuda.set_device(dev)
        nzl, mode = 12, "fused"
        loc = MK[cfg](nzl)
        plan = loc["plans"]["fused"]
        probe = Program(loc, nz_global=nzl * world)
        probe.set_plan(plan)
        zhalo = max([max(r["z_below"], r["z_above"]) for m in ("fused", "unfused")
                     for r in probe.reports(m)] + [loc["grid"]["ghost"][2]])
        comm = Comm.loopback(world)[rank]  # only its rank count is used (no run_fused here)
        s = Program(loc, comm=comm, nz_global=nzl * world, z_offset=rank * nzl, zhalo=zhalo,
                    options={"xpush": 1})
        s.set_plan(plan)
        s.allocate(dev)
        fill(s, loc, dev, rank * nzl, zhalo, nz_global=nzl * world)
        s.load(mode)
        s.connect_peers(rank, world)
        torch.cuda.synchronize()
        n = s.n_launches(mode)
        for step in range(2):
            for i in range(n):
                for a, below, above in s.exchange_plan(mode, i):  # step-start epochs over gloo
                    t = s.tensors[a]
                    if rank + 1 < world:
                        if below:
                            dist.send(plane(s, t, nzl - below, below).cpu().contiguous(), dst=rank + 1)
                        if above:
                            buf = torch.empty_like(plane(s, t, 0, above), device="cpu")
                            dist.recv(buf, src=rank + 1)
                            plane(s, t, nzl, above).copy_(buf)
                    if rank > 0:
                        if below:
                            buf = torch.empty_like(plane(s, t, 0, below), device="cpu")
                            dist.recv(buf, src=rank - 1)
                            plane(s, t, -below, below).copy_(buf)
                        if above:
                            dist.send(plane(s, t, 0, above).cpu().contiguous(), dst=rank - 1)
                if concurrent:
                    if i == 0:
                        torch.cuda.synchronize()
                        dist.barrier()
                    s.run_launch(mode, i)
                    continue
                torch.cuda.synchronize()
                dist.barrier()
                for r in range(world):
                    if r == rank:
                        s.run_launch(mode, i)
                        torch.cuda.synchronize()
                    dist.barrier()
            assert all(not x for i in range(1, n) for x in s.exchange_plan(mode, i)) or not concurrent
            torch.cuda.synchronize()
            dist.barrier()
        outs = [a["name"] for a in loc["arrays"] if a["role"] in ("out", "inout")]
        mine = {nm: s.interior_view(s.tensors[nm]).cpu() for nm in outs}
        got = [None] * world if rank == 0 else None
        dist.gather_object(mine, got, dst=0)
        if rank == 0:
            glob = MK[cfg](nzl * world)
            single = Program(glob)
            single.set_plan(plan)
            single.allocate(dev)
            fill(single, glob, dev, 0, glob["grid"]["ghost"][2])
            single.run(mode)
            torch.cuda.synchronize()
            for nm in outs:
                want = single.interior_view(single.tensors[nm]).cpu()
                have = torch.cat([g[nm] for g in got], dim=0)
                assert torch.equal(have, want), f"{cfg} {nm}: IPC peer-push result differs"
        q.put((rank, "ok"))
    except Exception as e:  # surfaced in the parent
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


# lockstep only: concurrent launches whose kernels wait on the other process's kernels are
# not run on one GPU (no co-residency guarantee; Xid 109 recorded on this driver)
@pytest.mark.parametrize("cfg,concurrent", [("C4", False), ("C3", False)])
def test_peer_push_ipc_processes(cuda_device, cfg, concurrent):
    """Peer push across PROCESSES (the real deployment shape: one process per rank):
    each rank maps its neighbours' TEMP buffers and signal blocks with CUDA IPC
    (sp_ipc_export / sp_ipc_open via Program.connect_peers).  Both processes share
    one GPU here; their launches run in lockstep.  Bit-exact with the single domain."""
    import multiprocessing as mp
    import socket
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    world = 2
    ps = [ctx.Process(target=_ipc_worker, args=(r, world, port, cfg, q, concurrent)) for r in range(world)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
    assert all(v == "ok" for v in res.values()), res


@pytest.mark.parametrize("ranks", [2, 3])
def test_loopback_exchange_halos_rank_encoded(cuda_device, ranks):
    """exchange_halos (§8(b)) unit test on in-process virtual ranks: every array's whole
    allocated planes carry an exact code of (array, global plane, y, x); after
    exchange_halos(depth) each rank's ghost planes equal its neighbours' interior
    planes, and interior planes and true global ghost planes are untouched."""
    import threading
    import torch
    from _nccl_worker import encoded
    from paper_conf_hpdc_wahibm15_b200 import Comm, Program
    nzl, depth = 7, 3
    prog = P.c2(nx=40, ny=24, nz=nzl)
    comms = Comm.loopback(ranks)
    progs = []
    for r in range(ranks):
        p = Program(prog, comm=comms[r], nz_global=nzl * ranks, z_offset=r * nzl, zhalo=depth)
        p.allocate(cuda_device)
        oz = p.layout["origin_z"]
        for aid, n in enumerate(p.names):
            t = p.tensors[n]
            for z in range(nzl):
                t[oz + z].copy_(encoded(aid, r * nzl + z, t.shape[1:], t.device))
        progs.append(p)
    torch.cuda.synchronize()
    errs = []

    def drive(r):
        try:
            st = torch.cuda.Stream(device=cuda_device)
            progs[r].exchange_halos(progs[r].names, depth, st)
            st.synchronize()
        except Exception as e:  # surfaced below
            errs.append(e)

    th = [threading.Thread(target=drive, args=(r,)) for r in range(ranks)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    assert not errs, errs
    for r, p in enumerate(progs):
        oz = p.layout["origin_z"]
        for aid, n in enumerate(p.names):
            t = p.tensors[n]
            for z in range(-depth, nzl + depth):
                gz = r * nzl + z
                if 0 <= z < nzl:
                    assert torch.equal(t[oz + z], encoded(aid, gz, t.shape[1:], t.device)), (r, n, z)
                elif gz < 0 or gz >= nzl * ranks:
                    assert torch.isnan(t[oz + z]).all(), (r, n, z)
                else:
                    assert torch.equal(t[oz + z], encoded(aid, gz, t.shape[1:], t.device)), (r, n, z)
