"""Per-launch tuning of a plan's groups over candidate tile configurations (dev tool):
isolated launches with a read-only L2 flush, candidates JIT-compiled in parallel.

python tools/frame_tune.py C3 fission_fused --opt frame=1 [--out configs/variants/x.json]

Every candidate is applied to all launches of the plan (a launch whose rings do not fit
skips it); the best configuration per launch and the sum of the best times are printed
and, with --out, written as {"configs": [...], "group_us": [...]} (bench's pin format).
"""
import argparse
import itertools
import json
import os
import statistics
import sys
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_hpdc_wahibm15_b200 import Program, StencilError  # noqa: E402


def candidates(dtype, wide):
    txs = [32, 64, 128] if dtype == "f32" else [16, 32, 64]
    tys = [4, 8, 16, 32] if wide else [4, 8, 16]
    nts = [64, 128, 256, 512] if wide else [128, 256]
    zcs = [8, 16, 32, 64] if wide else [16, 32]
    pfs = [1, 2] if wide else [1]
    for tx, ty, nt, zc, pf in itertools.product(txs, tys, nts, zcs, pfs):
        yield dict(tile_x=tx, tile_y=ty, threads=nt, zchunk=zc, prefetch=pf)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("plan")
    ap.add_argument("--opt", action="append", default=[])
    ap.add_argument("--wide", action="store_true")
    ap.add_argument("--iters", type=int, default=5)
    ap.add_argument("--out")
    ap.add_argument("--plan-file", help="groups from a plan file (\"groups\") instead of the named plan")
    a = ap.parse_args()
    opts = {kv.split("=")[0]: int(kv.split("=")[1]) for kv in a.opt}
    prog = bench.load_workload(a.workload)
    plan = json.load(open(a.plan_file))["groups"] if a.plan_file else bench.plan_of(prog, a.plan)
    dev = torch.device("cuda:0")
    base = Program(prog, options=opts)
    base.set_plan(plan)
    base.allocate(dev, fill=0.0)
    bench.fill_inputs(base, prog, dev, 0, prog["grid"]["ghost"][2])
    n = base.n_launches("fused")
    cands = [{}] + list(candidates(prog["dtype"], a.wide))  # {}: the model-driven chooser

    def build(c):
        p = Program(prog, options=opts)
        p.set_plan(plan)
        ok = []
        for i in range(n):
            try:
                p.tune("fused", i, dict(c, **({"frame": opts["frame"]} if "frame" in opts else {})))
                ok.append(i)
            except StencilError:
                p.tune("fused", i, None)
        try:
            p.compile("fused")
        except StencilError:
            return c, None, []
        return c, p, ok

    with ThreadPoolExecutor(16) as ex:
        built = [b for b in ex.map(build, cands) if b[1] is not None]
    flush = torch.ones(32 << 20, dtype=torch.float64, device=dev)
    pts = prog["grid"]["nx"] * prog["grid"]["ny"] * prog["grid"]["nz"]
    best = [(1e30, None)] * n
    for c, p, ok in built:
        for nm, t in base.tensors.items():
            p.bind(nm, t)
        for i in ok:
            p.run_launch("fused", i)
            torch.cuda.synchronize()
            ts = []
            for _ in range(a.iters):
                flush.sum()
                s, e = torch.cuda.Event(True), torch.cuda.Event(True)
                s.record()
                p.run_launch("fused", i)
                e.record()
                torch.cuda.synchronize()
                ts.append(s.elapsed_time(e) * 1e3)
            us = statistics.median(ts)
            if us < best[i][0]:
                best[i] = (us, dict(c, regs=p.report("fused", i)["regs_per_thread"]))
        del p
    reps = base.reports("fused")
    tot = 0.0
    for i, (us, c) in enumerate(best):
        tot += us
        print(f"L{i:02d} {us:9.1f} us  {reps[i]['bytes_alg'] * pts / us / 1e3:7.0f} GB/s alg  {c}")
    print(f"{a.workload} {a.plan} {opts}: sum of best launches {tot / 1e3:.4f} ms "
          f"({len(built)} candidates compiled)")
    if a.out:
        cfgs = []
        for us, c in best:
            c = dict(c or {})
            c.pop("regs", None)
            if "frame" in opts:
                c["frame"] = opts["frame"]
            cfgs.append(c or None)
        json.dump({"workload": a.workload, "plan": a.plan, "options": opts, "configs": cfgs,
                   "group_us": [b[0] for b in best]}, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
