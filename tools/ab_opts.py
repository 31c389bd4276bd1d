"""Interleaved A/B of codegen option sets on one workload's fused step (dev tool).

python tools/ab_opts.py C3 --plan fission_fused --rounds 5 'halo_sel=0' 'halo_sel=1'
python tools/ab_opts.py C4 'psleep=32' 'pin_fastpath=2'      (pin_<k>: override every launch pin)

Every option set gets its own Program over the SAME device arrays; rounds alternate
the sets (drift on the box is +-5 %, larger than most single-option effects).  Prints
per round the step time of each set, then the median step and the median per-launch
times (CUDA events around each launch, inside the running step).
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


def parse(spec):
    return {kv.split("=")[0]: int(kv.split("=")[1]) for kv in spec.split(",") if kv}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("specs", nargs="+")
    ap.add_argument("--plan", default="fused")
    ap.add_argument("--rounds", type=int, default=5)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--no-tune", action="store_true", help="chooser configurations, not the pins")
    a = ap.parse_args()
    prog = bench.load_workload(a.workload)
    dev = torch.device("cuda:0")
    plan = bench.plan_of(prog, a.plan)
    progs, base = [], None
    for spec in a.specs:
        # keys "pin_<k>" override <k> in every per-launch pin; the rest are program options
        kv = parse(spec)
        over = {k[4:]: v for k, v in kv.items() if k.startswith("pin_")}
        p = Program(prog, options={k: v for k, v in kv.items() if not k.startswith("pin_")})
        p.set_plan(plan)
        if not a.no_tune:
            bench.apply_tuning(p, prog, a.plan)
            if over:
                for i, c in enumerate(bench.tuned_configs(prog, a.plan) or []):
                    p.tune("fused", i, dict(c or {}, **over))
        if base is None:
            p.allocate(dev, fill=0.0)
            bench.fill_inputs(p, prog, dev, 0, prog["grid"]["ghost"][2])
            base = p.tensors
        else:
            for n, t in base.items():
                p.bind(n, t)
        p.compile("fused")
        for _ in range(3):
            p.run_fused()
        progs.append(p)
    torch.cuda.synchronize()
    pts = prog["grid"]["nx"] * prog["grid"]["ny"] * prog["grid"]["nz"]
    step = {s: [] for s in a.specs}
    per = {s: [] for s in a.specs}
    for r in range(a.rounds):
        line = []
        for spec, p in zip(a.specs, progs):
            s, e = torch.cuda.Event(True), torch.cuda.Event(True)
            s.record()
            for _ in range(a.steps):
                p.run_fused()
            e.record()
            torch.cuda.synchronize()
            t = s.elapsed_time(e) / a.steps
            step[spec].append(t)
            n = p.n_launches("fused")
            ev = [(torch.cuda.Event(True), torch.cuda.Event(True)) for _ in range(n)]
            for i in range(n):
                ev[i][0].record()
                p.run_launch("fused", i)
                ev[i][1].record()
            torch.cuda.synchronize()
            per[spec].append([x.elapsed_time(y) * 1e3 for x, y in ev])
            line.append(f"{t:.4f}")
        print(f"round {r}: " + "  ".join(line), flush=True)
    for spec, p in zip(a.specs, progs):
        reps = p.reports("fused")
        m = statistics.median(step[spec])
        alg = sum(x["bytes_alg"] for x in reps) * pts
        print(f"{a.workload} {a.plan} [{spec}]: median {m:.4f} ms/step  {alg / m / 1e6:.0f} GB/s alg  "
              f"regs {[x['regs_per_thread'] for x in reps]}")
        for i in range(len(reps)):
            us = statistics.median(v[i] for v in per[spec])
            print(f"    L{i:02d} {us:9.1f} us  {reps[i]['bytes_alg'] * pts / us / 1e3:7.0f} GB/s")


if __name__ == "__main__":
    main()
