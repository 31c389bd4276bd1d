"""Cost of the multi-rank schedule on ONE GPU (dev tool; a proxy, not a scaling number).

python tools/loopback_overhead.py [--workload C4] [--ranks 2 4] [--steps 50]

The single-domain step over the workload's per-GPU grid is compared with the same
grid cut into P z-slabs driven as P in-process virtual ranks (loopback transport,
one host thread and one stream each): every launch that receives ghost planes runs
as interior planes (overlapping the exchange copies) + two boundary launches, as
on P GPUs.  Total work is fixed, so t(P)/t(1) - 1 is the schedule's overhead on
one GPU: extra launches, few-plane boundary launches, events, host barriers and
the ghost copies (which on P GPUs travel over NVLink instead).  Warp-level
concurrency between the virtual ranks' kernels makes this an optimistic proxy.
"""
import argparse
import json
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_hpdc_wahibm15_b200 import Comm, Program  # noqa: E402


def resize_nz(prog, nz):
    q = json.loads(json.dumps(prog))
    q["grid"]["nz"] = nz
    return q


def time_ranks(prog, plan, tuned, P, steps, warmup, dev, mode):
    nz = prog["grid"]["nz"] // P
    loc = resize_nz(prog, nz)
    probe = Program(loc, nz_global=nz * P) if P > 1 else Program(loc)
    probe.set_plan(plan)
    zhalo = max([max(r["z_below"], r["z_above"]) for m in ("fused", "unfused") for r in probe.reports(m)]
                + [loc["grid"]["ghost"][2]]) if P > 1 else loc["grid"]["ghost"][2]
    comms = Comm.loopback(P) if P > 1 else [None]
    progs = []
    for r in range(P):
        kw = dict(comm=comms[r], nz_global=nz * P, z_offset=r * nz, zhalo=zhalo) if P > 1 else {}
        p = Program(loc, **kw)
        p.set_plan(plan)
        if tuned:
            for i, c in enumerate(tuned):
                if c:
                    p.tune("fused", i, c)
        p.allocate(dev, fill=0.0)
        bench.fill_inputs(p, loc, dev, r * nz, zhalo)
        p.load(mode)
        progs.append(p)
    torch.cuda.synchronize()
    out = [0.0] * P
    host = [0.0] * P

    def drive(r):
        st = torch.cuda.Stream(device=dev)
        for _ in range(warmup):
            progs[r].run(mode, st)
        st.synchronize()
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record(st)
        h0 = time.perf_counter()
        for _ in range(steps):
            progs[r].run(mode, st)
        host[r] = (time.perf_counter() - h0) * 1e3 / steps
        e.record(st)
        e.synchronize()
        out[r] = s.elapsed_time(e) / steps

    th = [threading.Thread(target=drive, args=(r,)) for r in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    # host-thread start skew is small next to `steps` steps; take the slowest rank
    return max(out), max(host)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C4")
    ap.add_argument("--ranks", type=int, nargs="*", default=[2, 4])
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--mode", default="fused")
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    prog = bench.load_workload(a.workload)
    plan = bench.plan_of(prog, "fused")
    tuned = bench.tuned_configs(prog, "fused")
    t1, h1 = time_ranks(prog, plan, tuned, 1, a.steps, a.warmup, dev, a.mode)
    res = {"workload": a.workload, "mode": a.mode, "ms_1": t1, "host_enqueue_ms_1": h1}
    for P in a.ranks:
        tp, hp = time_ranks(prog, plan, tuned, P, a.steps, a.warmup, dev, a.mode)
        res[f"ms_{P}"] = tp
        res[f"host_enqueue_ms_{P}"] = hp  # ~ ms_P: the host, not the GPU, sets the pace
        res[f"overhead_{P}"] = tp / t1 - 1
    print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
