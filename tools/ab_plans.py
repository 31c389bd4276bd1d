"""Interleaved A/B of whole-step times for plan variants (dev tool).

python tools/ab_plans.py C4 configs/c4_plan.json /tmp/variant.json ... [--rounds 7] [--tune-new]

Each plan file holds "groups" and "configs".  With --tune-new, groups whose config is
null get the best configuration of an isolated-launch sweep (read-only L2 flush;
tools/step_tune.py candidates).  Step times are measured in interleaved rounds
(A B C A B C ...) so that clock/power drift hits every variant alike; the median
per variant is reported, and the tuned plan files are written next to --outdir.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_hpdc_wahibm15_b200 import Program, StencilError  # noqa: E402
from step_tune import candidates  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("plans", nargs="+")
    ap.add_argument("--rounds", type=int, default=7)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--tune-new", action="store_true")
    ap.add_argument("--outdir", default="gpurun_out")
    a = ap.parse_args()
    os.makedirs(a.outdir, exist_ok=True)
    prog = bench.load_workload(a.workload)
    dev = torch.device("cuda:0")
    stream = torch.cuda.current_stream(dev)
    flush = torch.ones(32 << 20, dtype=torch.float64, device=dev)
    tensors = None
    progs = []
    for path in a.plans:
        pj = json.load(open(path))
        cfgs = pj.get("configs") or [None] * len(pj["groups"])
        p = Program(prog)
        p.set_plan(pj["groups"])
        for i, c in enumerate(cfgs):
            if c:
                p.tune("fused", i, c)
        if tensors is None:
            p.allocate(dev, fill=0.0)
            bench.fill_inputs(p, prog, dev, 0, prog["grid"]["ghost"][2])
            tensors = p.tensors
        else:
            for n, t in tensors.items():
                p.bind(n, t)
        if a.tune_new:
            for i, c in enumerate(cfgs):
                if c:
                    continue
                best = (float("inf"), None)
                for cand in candidates(prog["grid"]["ny"]):
                    try:
                        p.tune("fused", i, cand)
                        p.run_launch("fused", i)
                        torch.cuda.synchronize()
                        ts = []
                        for _ in range(5):
                            flush.sum()
                            s, e = torch.cuda.Event(True), torch.cuda.Event(True)
                            s.record()
                            p.run_launch("fused", i)
                            e.record()
                            torch.cuda.synchronize()
                            ts.append(s.elapsed_time(e))
                        t = sorted(ts)[2]
                    except StencilError:
                        continue
                    if t < best[0]:
                        best = (t, cand)
                cfgs[i] = best[1]
                p.tune("fused", i, best[1])
                print(f"{os.path.basename(path)} group {i}: isolated {best[0]*1e3:.1f} us {best[1]}",
                      flush=True)
            pj["configs"] = cfgs
            out = os.path.join(a.outdir, "tuned_" + os.path.basename(path))
            json.dump(pj, open(out, "w"), indent=1)
        alg = sum(r["bytes_alg"] for r in p.reports("fused"))
        p.run_fused(stream)
        torch.cuda.synchronize()
        progs.append((path, p, alg))
    times = {path: [] for path, _, _ in progs}
    for r in range(a.rounds):
        for path, p, _ in progs:
            for _ in range(3):
                p.run_fused(stream)
            s, e = torch.cuda.Event(True), torch.cuda.Event(True)
            s.record(stream)
            for _ in range(a.steps):
                p.run_fused(stream)
            e.record(stream)
            torch.cuda.synchronize()
            times[path].append(s.elapsed_time(e) / a.steps)
    pts = prog["grid"]["nx"] * prog["grid"]["ny"] * prog["grid"]["nz"]
    for path, p, alg in progs:
        t = statistics.median(times[path])
        print(f"{path:40s} median {t:.4f} ms/step (min {min(times[path]):.4f}, max "
              f"{max(times[path]):.4f})  {alg:.0f} B/pt  {alg * pts / t / 1e6:.0f} GB/s alg", flush=True)


if __name__ == "__main__":
    main()
