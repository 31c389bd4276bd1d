"""Interleaved A/B of option sets on a workload's fused step, with per-launch times (dev tool).

python tools/ab_launch.py C4 'fastpath=0' 'fastpath=1' [--rounds 5] [--steps 30] [--plan fused]

Each round runs every option set for --steps back-to-back steps (step time from CUDA
events around them) and then one step with an event between launches; medians over
rounds are printed per option set: step ms, per-launch us and algorithmic GB/s.
"""
import argparse
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_hpdc_wahibm15_b200 import Program  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("workload")
ap.add_argument("specs", nargs="+")
ap.add_argument("--rounds", type=int, default=5)
ap.add_argument("--steps", type=int, default=30)
ap.add_argument("--plan", default="fused")
ap.add_argument("--untuned", action="store_true", help="chooser configurations (no pins)")
a = ap.parse_args()
prog = bench.load_workload(a.workload)
dev = torch.device("cuda:0")
g = prog["grid"]
pts = g["nx"] * g["ny"] * g["nz"]
progs, base = [], None
for spec in a.specs:
    opts = {kv.split("=")[0]: int(kv.split("=")[1]) for kv in spec.split(",") if kv}
    p = Program(prog, options=opts)
    p.set_plan(bench.plan_of(prog, a.plan))
    if not a.untuned:
        bench.apply_tuning(p, prog, a.plan)
    if base is None:
        p.allocate(dev, fill=0.0)
        bench.fill_inputs(p, prog, dev, 0, g["ghost"][2])
        base = p.tensors
    else:
        for n, t in base.items():
            p.bind(n, t)
    p.load("fused")
    for _ in range(3):
        p.run_fused()
    progs.append(p)
torch.cuda.synchronize()
nl = progs[0].n_launches("fused")
res = [{"step": [], "launch": [[] for _ in range(nl)]} for _ in progs]
for r in range(a.rounds):
    for k, p in enumerate(progs):
        s, e = torch.cuda.Event(True), torch.cuda.Event(True)
        s.record()
        for _ in range(a.steps):
            p.run_fused()
        e.record()
        ev = [torch.cuda.Event(True) for _ in range(nl + 1)]
        for i in range(nl):
            ev[i].record()
            p.run_launch("fused", i)
        ev[nl].record()
        torch.cuda.synchronize()
        res[k]["step"].append(s.elapsed_time(e) / a.steps)
        for i in range(nl):
            res[k]["launch"][i].append(ev[i].elapsed_time(ev[i + 1]))
for k, spec in enumerate(a.specs):
    reps = progs[k].reports("fused")
    st = statistics.median(res[k]["step"])
    alg = sum(x["bytes_alg"] for x in reps) * pts
    print(f"[{spec}] step {st:.4f} ms  ({alg / st / 1e6:.0f} GB/s alg)  rounds {['%.4f' % x for x in res[k]['step']]}")
    for i in range(nl):
        t = statistics.median(res[k]["launch"][i])
        print(f"   L{i:02d} {t * 1e3:8.1f} us  {reps[i]['bytes_alg'] * pts / t / 1e6:7.0f} GB/s  regs {reps[i]['regs_per_thread']}")
