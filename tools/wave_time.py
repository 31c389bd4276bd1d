"""Step time of the z-wave schedule vs the plain plan order, with a bit-exact check (dev tool).

python tools/wave_time.py C4 --waves 0:1 32:2 64:2 ... [--steps 100] [--pdl 1]
Each --waves entry is zwave:zwave_streams (0 = plain plan order).
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_hpdc_wahibm15_b200 import Program  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("--waves", nargs="+", default=["0:1", "32:2", "64:2"])
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--opt", action="append", default=[])
    ap.add_argument("--plan", default="fused", help="named plan (e.g. unfused: one group per kernel)")
    a = ap.parse_args()
    prog = bench.load_workload(a.workload)
    plan = bench.plan_of(prog, a.plan)
    dev = torch.device("cuda:0")
    stream = torch.cuda.current_stream(dev)
    pts = prog["grid"]["nx"] * prog["grid"]["ny"] * prog["grid"]["nz"]
    outs = [x["name"] for x in prog["arrays"] if x["role"] in ("out", "inout")]
    base = None
    ref = None
    extra = {kv.split("=")[0]: int(kv.split("=")[1]) for kv in a.opt}
    for spec in a.waves:
        zw, ns = (int(v) for v in spec.split(":"))
        p = Program(prog, options=dict(extra, zwave=zw, zwave_streams=ns))
        p.set_plan(plan)
        if a.plan == "fused":
            bench.apply_tuning(p, prog)
        if base is None:
            p.allocate(dev, fill=0.0)
            bench.fill_inputs(p, prog, dev, 0, prog["grid"]["ghost"][2])
            base = p.tensors
        else:
            for n, t in base.items():
                p.bind(n, t)
        for n in outs:
            base[n].fill_(0.0)
        p.run_fused(stream)
        torch.cuda.synchronize()
        got = {n: base[n].clone() for n in outs}
        if ref is None:
            ref = got
        exact = all(torch.equal(got[n], ref[n]) for n in outs)
        for _ in range(5):
            p.run_fused(stream)
        s, e = torch.cuda.Event(True), torch.cuda.Event(True)
        torch.cuda.synchronize()
        s.record(stream)
        for _ in range(a.steps):
            p.run_fused(stream)
        e.record(stream)
        torch.cuda.synchronize()
        ms = s.elapsed_time(e) / a.steps
        alg = sum(r["bytes_alg"] for r in p.reports("fused")) * pts
        print(f"{a.plan} zwave {zw:4d} streams {ns}: {ms:.4f} ms/step  {alg / ms / 1e6:7.0f} GB/s alg  "
              f"{pts * len(prog['kernels']) / ms / 1e6:.3e} upd/s  bit-exact {exact}", flush=True)
        del p


if __name__ == "__main__":
    main()
