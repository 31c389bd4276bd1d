"""Check the tile chooser's model against measured sweeps (host only, no GPU).

python tools/model_fit.py profiles/sweeps/C2_g0.log:C2:fused:0 ...
For each sweep (tools/sweep.py output: config -> measured launch time), re-evaluates
the model time of every configuration with the current library build, then reports
the Spearman rank correlation and the regret: measured time of the model's pick over
the best measured time (and the chooser's own pick, unconstrained).
"""
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
from paper_conf_hpdc_wahibm15_b200 import Program, StencilError  # noqa: E402


def parse(path):
    rows = []
    for line in open(path):
        m = re.match(r"(\S+)\s+([\d.]+) us alg", line)
        if m and "=" in m.group(1):
            cfg = {kv.split("=")[0]: int(kv.split("=")[1]) for kv in m.group(1).split(",")}
            rows.append((cfg, float(m.group(2))))
    return rows


def rank(v):
    order = sorted(range(len(v)), key=lambda i: v[i])
    r = [0] * len(v)
    for k, i in enumerate(order):
        r[i] = k
    return r


def main():
    tot_regret = []
    for spec in sys.argv[1:]:
        path, wl, plan, g = spec.split(":")
        prog = bench.load_workload(wl)
        plan_groups = prog["plans"][plan]
        rows = parse(path)
        model, meas = [], []
        for cfg, t in rows:
            try:
                p = Program(prog, options=cfg)
                p.set_plan(plan_groups)
                model.append(p.report("fused", int(g))["t_model_us"])
                meas.append(t)
            except StencilError:
                continue
        p = Program(prog)
        p.set_plan(plan_groups)
        r = p.report("fused", int(g))
        pick = min(range(len(model)), key=lambda i: model[i])
        rm, rt = rank(model), rank(meas)
        n = len(meas)
        rho = 1 - 6 * sum((a - b) ** 2 for a, b in zip(rm, rt)) / (n * (n * n - 1))
        best = min(meas)
        tot_regret.append(meas[pick] / best)
        print(f"{spec}: n={n} spearman {rho:.2f}  model pick {meas[pick]:.1f} us "
              f"(best {best:.1f}, regret {meas[pick]/best:.2f}x)  chooser: {r['tile_x']}x{r['tile_y']}x"
              f"{r['zchunk']} nt{r['threads']} b{r['block_x']}x{r['block_y']}x{r['block_cby']} "
              f"model {r['t_model_us']:.0f} us")
    if tot_regret:
        import math
        print(f"geomean regret {math.exp(sum(math.log(x) for x in tot_regret) / len(tot_regret)):.3f}")


if __name__ == "__main__":
    main()
