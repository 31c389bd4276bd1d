"""Peer-push multi-rank step on ONE GPU under MPS (dev tool; a proxy, not a scaling number).

DO NOT RUN on the shared B200 pool: its kernels wait on kernels of other processes on the
same GPU, which has no co-residency guarantee (the pool's driver recorded Xid 109
context-switch timeouts for exactly this); kept for reference with its round-1 results.

python tools/mps_xpush.py [--workload C4] [--ranks 2] [--steps 10] [--no-mps]

Starts an MPS daemon (CUDA_MPS_PIPE_DIRECTORY under /tmp), so that the P rank
processes' kernels run CONCURRENTLY on the GPU with separate work queues (unlike
threads of one process, which may share hardware queues).  Each rank
owns a z-slab of the workload's per-GPU grid (total work fixed), maps its
neighbours' TEMP buffers and signal blocks with CUDA IPC (Program.connect_peers),
receives the step-start epochs over gloo (host copies, outside the timed region),
then enqueues the whole step; the kernels order themselves through the in-kernel
progress protocol.  Reported: per-step GPU time (CUDA events around the enqueued
launches, max over ranks) against the single-domain step, and whether the result
is bit-identical to the single domain.  The ranks share one GPU's SMs and HBM, so
the ratio bounds the decomposition's extra work, not NVLink effects.
"""
import argparse
import json
import os
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def worker(rank, world, port, workload, steps, q, independent=False, xpush=1):
    sys.path.insert(0, ROOT)
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import bench
        from paper_conf_hpdc_wahibm15_b200 import Comm, Program
        dev = torch.device("cuda:0")
        torch.cuda.set_device(dev)
        prog = bench.load_workload(workload)
        plan = bench.plan_of(prog, "fused")
        nz = prog["grid"]["nz"] // world
        loc = json.loads(json.dumps(prog))
        loc["grid"]["nz"] = nz
        probe = Program(loc, nz_global=nz * world)
        probe.set_plan(plan)
        zhalo = max([max(r["z_below"], r["z_above"]) for m in ("fused", "unfused")
                     for r in probe.reports(m)] + [loc["grid"]["ghost"][2]])
        comm = Comm.loopback(world)[rank]  # rank count only; no run_fused transport here
        if independent:  # baseline: the same slabs as unrelated single-domain problems
            p = Program(loc)
            zhalo = loc["grid"]["ghost"][2]
        else:
            p = Program(loc, comm=comm, nz_global=nz * world, z_offset=rank * nz, zhalo=zhalo,
                        options={"xpush": xpush})
        p.set_plan(plan)
        bench.apply_tuning(p, prog)
        p.allocate(dev, fill=0.0)
        bench.fill_inputs(p, loc, dev, rank * nz, zhalo)
        p.load("fused")
        if not independent and xpush:
            p.connect_peers(rank, world)
        oz = p.layout["origin_z"]
        n = p.n_launches("fused")
        x0 = [] if independent else p.exchange_plan("fused", 0)
        assert independent or all(not p.exchange_plan("fused", i) for i in range(1, n))
        times = []
        for step in range(steps + 2):
            torch.cuda.synchronize()
            for a, below, above in x0:  # step-start epochs over gloo (untimed)
                t = p.tensors[a]
                if rank + 1 < world:
                    if below:
                        dist.send(t[oz + nz - below:oz + nz].cpu().contiguous(), dst=rank + 1)
                    if above:
                        buf = torch.empty_like(t[oz:oz + above], device="cpu")
                        dist.recv(buf, src=rank + 1)
                        t[oz + nz:oz + nz + above].copy_(buf)
                if rank > 0:
                    if below:
                        buf = torch.empty_like(t[oz:oz + below], device="cpu")
                        dist.recv(buf, src=rank - 1)
                        t[oz - below:oz].copy_(buf)
                    if above:
                        dist.send(t[oz:oz + above].cpu().contiguous(), dst=rank - 1)
            torch.cuda.synchronize()
            dist.barrier()
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            for i in range(n):
                p.run_launch("fused", i)
            e.record()
            e.synchronize()
            if step >= 2:
                times.append(s.elapsed_time(e))
        outs = [a["name"] for a in loc["arrays"] if a["role"] in ("out", "inout")]
        mine = {nm: p.interior_view(p.tensors[nm]).cpu() for nm in outs}
        got = [None] * world if rank == 0 else None
        dist.gather_object(mine, got, dst=0)
        tall = [None] * world
        dist.all_gather_object(tall, sorted(times)[len(times) // 2])
        res = {"ms_per_step_ranks": max(tall)}
        if rank == 0:
            single = Program(prog)
            single.set_plan(plan)
            bench.apply_tuning(single, prog)
            single.allocate(dev, fill=0.0)
            bench.fill_inputs(single, prog, dev, 0, prog["grid"]["ghost"][2])
            single.load("fused")
            ts = []
            for step in range(steps + 2):
                s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                s.record()
                for i in range(single.n_launches("fused")):
                    single.run_launch("fused", i)
                e.record()
                e.synchronize()
                if step >= 2:
                    ts.append(s.elapsed_time(e))
            res["ms_per_step_single"] = sorted(ts)[len(ts) // 2]
            res["bitexact"] = independent or all(torch.equal(torch.cat([g[nm] for g in got], dim=0),
                                              single.interior_view(single.tensors[nm]).cpu())
                                  for nm in outs)
        q.put((rank, res))
    except Exception:
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C4")
    ap.add_argument("--ranks", type=int, default=2)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--no-mps", action="store_true")
    ap.add_argument("--xpush", type=int, default=1, help="0: plain multi-rank kernels (valid only "
                    "when every exchange is a step-start one, e.g. C5)")
    ap.add_argument("--independent", action="store_true",
                    help="baseline: the slabs as unrelated problems (no protocol, no exchange)")
    a = ap.parse_args()
    env = dict(os.environ)
    tmp = tempfile.mkdtemp(prefix="sf_mps_")
    if not a.no_mps:
        os.environ["CUDA_MPS_PIPE_DIRECTORY"] = os.path.join(tmp, "pipe")
        os.environ["CUDA_MPS_LOG_DIRECTORY"] = os.path.join(tmp, "log")
        os.makedirs(os.environ["CUDA_MPS_PIPE_DIRECTORY"])
        os.makedirs(os.environ["CUDA_MPS_LOG_DIRECTORY"])
        subprocess.run(["nvidia-cuda-mps-control", "-d"], check=True, env=dict(os.environ))
    try:
        import multiprocessing as mp
        import socket
        sk = socket.socket()
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
        sk.close()
        ctx = mp.get_context("spawn")
        q = ctx.Queue()
        ps = [ctx.Process(target=worker, args=(r, a.ranks, port, a.workload, a.steps, q, a.independent, a.xpush))
              for r in range(a.ranks)]
        for p in ps:
            p.start()
        res = dict(q.get(timeout=600) for _ in range(a.ranks))
        for p in ps:
            p.join(timeout=60)
        r0 = res[0]
        if isinstance(r0, str):
            print(r0)
            sys.exit(1)
        r0.update(workload=a.workload, ranks=a.ranks, mps=not a.no_mps, independent=a.independent, xpush=a.xpush,
                  overhead=r0["ms_per_step_ranks"] / r0["ms_per_step_single"] - 1)
        print(json.dumps(r0), flush=True)
    finally:
        if not a.no_mps:
            subprocess.run(["nvidia-cuda-mps-control"], input=b"quit\n", env=dict(os.environ))
        del env


if __name__ == "__main__":
    main()
