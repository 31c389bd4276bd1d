"""A/B of whole-step times for option sets (dev tool): python tools/ab_step.py C4 'pdl=0' 'pdl=1'"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_hpdc_wahibm15_b200 import Program  # noqa: E402

prog = bench.load_workload(sys.argv[1])
dev = torch.device("cuda:0")
base = None
for spec in sys.argv[2:]:
    opts = {kv.split("=")[0]: int(kv.split("=")[1]) for kv in spec.split(",") if kv}
    p = Program(prog, options=opts)
    plan = os.environ.get("SF_PLAN", "fused")
    p.set_plan(bench.plan_of(prog, plan))
    bench.apply_tuning(p, prog, plan)
    if base is None:
        p.allocate(dev, fill=0.0)
        bench.fill_inputs(p, prog, dev, 0, prog["grid"]["ghost"][2])
        base = p.tensors
    else:
        for n, t in base.items():
            p.bind(n, t)
    for mode in ("fused", "unfused"):
        for _ in range(5):
            p.run(mode)
        torch.cuda.synchronize()
        s, e = torch.cuda.Event(True), torch.cuda.Event(True)
        s.record()
        for _ in range(50):
            p.run(mode)
        e.record()
        torch.cuda.synchronize()
        print(f"{spec:20s} {mode:8s} {s.elapsed_time(e) / 50:.4f} ms/step", flush=True)
