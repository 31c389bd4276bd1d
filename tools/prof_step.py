"""Run W warm-up + S steps of a workload's fused (and optionally unfused) path for ncu captures.

python tools/prof_step.py C4 --steps 2 [--unfused]   (no timing: launch list / --set full runs)
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_hpdc_wahibm15_b200 import Program  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("workload")
ap.add_argument("--steps", type=int, default=2)
ap.add_argument("--warmup", type=int, default=1)
ap.add_argument("--unfused", action="store_true")
ap.add_argument("--opt", action="append", default=[])
ap.add_argument("--plan", default="fused")
ap.add_argument("--cfg", help="per-launch pins (tools/frame_tune.py --out) instead of the bench's")
a = ap.parse_args()
prog = bench.load_workload(a.workload)
opts = {kv.split("=")[0]: int(kv.split("=")[1]) for kv in a.opt}
p = Program(prog, options=opts)
p.set_plan(bench.plan_of(prog, a.plan))
if a.cfg:
    import json
    for i, c in enumerate(json.load(open(a.cfg))["configs"]):
        if c:
            p.tune("fused", i, c)
else:
    bench.apply_tuning(p, prog, a.plan)
dev = torch.device("cuda:0")
p.allocate(dev, fill=0.0)
bench.fill_inputs(p, prog, dev, 0, prog["grid"]["ghost"][2])
p.compile("fused")
if a.unfused:
    p.compile("unfused")
torch.cuda.synchronize()
for _ in range(a.warmup + a.steps):
    p.run_fused()
    if a.unfused:
        p.run_unfused()
torch.cuda.synchronize()
print("done")
