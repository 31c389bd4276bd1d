"""The library's own plan search on the device (sp_plan_search_ex, objective = measured):
metadata pre-step, DP over contiguous kernel segments, lazy-fission GA with the dynamic
penalty f_p; every candidate group timed at the tile chooser's configuration and at each
CANDIDATES entry (a group costs its fastest).  Writes a plan file bench.py can load.

python tools/search_plan.py C4 [--out configs/c4_plan_search.json] [--generations 12]
                               [--population 16] [--seed 1]
(bench: SF_C4_PLAN=<out> python bench.py)
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

# candidate launch configurations (tile_x, tile_y, threads, block_x, block_y, block_cby,
# zchunk, prefetch): the shapes the r1/r2 in-context tuners pinned for the C2-C5 groups
CANDIDATES = [
    dict(tile_x=32, tile_y=16, threads=64, block_x=1, block_y=8, block_cby=1, zchunk=16, prefetch=2),
    dict(tile_x=32, tile_y=8, threads=128, block_x=1, block_y=2, block_cby=1, zchunk=16, prefetch=3),
    dict(tile_x=32, tile_y=8, threads=64, block_x=2, block_y=2, block_cby=1, zchunk=32, prefetch=1),
    dict(tile_x=32, tile_y=16, threads=256, block_x=1, block_y=1, block_cby=2, zchunk=16, prefetch=2),
    dict(tile_x=32, tile_y=32, threads=64, block_x=1, block_y=4, block_cby=4, zchunk=8, prefetch=3),
    dict(tile_x=64, tile_y=4, threads=128, block_x=1, block_y=2, block_cby=1, zchunk=32, prefetch=3),
    dict(tile_x=128, tile_y=2, threads=128, block_x=1, block_y=2, block_cby=1, zchunk=32, prefetch=3),
    dict(tile_x=32, tile_y=16, threads=128, block_x=1, block_y=4, block_cby=1, zchunk=16, prefetch=2),
    dict(tile_x=32, tile_y=16, threads=128, block_x=2, block_y=2, block_cby=1, zchunk=16, prefetch=3),
    dict(tile_x=32, tile_y=8, threads=128, block_x=1, block_y=2, block_cby=1, zchunk=32, prefetch=2),
]
CANDIDATES += [
    dict(tile_x=64, tile_y=8, threads=128, block_x=2, block_y=2, block_cby=1, zchunk=16, prefetch=2),
    dict(tile_x=32, tile_y=16, threads=128, block_x=1, block_y=4, block_cby=1, zchunk=16, prefetch=3),
    dict(tile_x=32, tile_y=8, threads=64, block_x=2, block_y=2, block_cby=1, zchunk=16, prefetch=2),
    dict(tile_x=32, tile_y=8, threads=128, block_x=1, block_y=2, block_cby=1, zchunk=32, prefetch=3),
]
# fp32 shapes (C3): wider tiles, 4-float register blocks (LDS.128 / STG.128)
CANDIDATES_F32 = [
    dict(tile_x=64, tile_y=8, threads=128, block_x=4, block_y=2, block_cby=1, zchunk=16, prefetch=2),
    dict(tile_x=128, tile_y=8, threads=128, block_x=4, block_y=4, block_cby=1, zchunk=16, prefetch=2),
    dict(tile_x=64, tile_y=16, threads=128, block_x=2, block_y=4, block_cby=1, zchunk=16, prefetch=2),
    dict(tile_x=128, tile_y=4, threads=128, block_x=4, block_y=1, block_cby=1, zchunk=32, prefetch=2),
]
# the predicate-free step body (codegen option "fastpath") as a per-group variant of each shape
CANDIDATES += [dict(c, fastpath=1) for c in list(CANDIDATES)]
CANDIDATES_F32 += [dict(c, fastpath=1) for c in list(CANDIDATES_F32)]


# region-vector (frame) evaluation: the shapes tools/frame_tune.py picked for the C2/C3/C5 groups
CANDIDATES_FRAME_F32 = [
    dict(tile_x=32, tile_y=16, threads=256, zchunk=64, prefetch=2, frame=1),
    dict(tile_x=32, tile_y=32, threads=256, zchunk=32, prefetch=1, frame=1),
    dict(tile_x=32, tile_y=16, threads=256, zchunk=32, prefetch=1, frame=1),
    dict(tile_x=64, tile_y=8, threads=256, zchunk=32, prefetch=1, frame=1),
    dict(tile_x=32, tile_y=16, threads=128, zchunk=32, prefetch=2, frame=1),
]
CANDIDATES_FRAME_F64 = [
    dict(tile_x=32, tile_y=8, threads=128, zchunk=8, prefetch=1, frame=1),
    dict(tile_x=16, tile_y=16, threads=128, zchunk=32, prefetch=1, frame=1),
    dict(tile_x=32, tile_y=16, threads=128, zchunk=16, prefetch=1, frame=1),
]


def measured_search(workload, generations=12, population=16, seed=1, candidates=None, reps=3,
                    frame=False):
    """Run the search on a full-size instance of the workload; returns the plan-file dict."""
    import torch
    import bench
    from paper_conf_hpdc_wahibm15_b200 import Program
    prog = bench.load_workload(workload)
    if candidates is None:
        candidates = CANDIDATES + (CANDIDATES_F32 if prog["dtype"] == "f32" else [])
        if frame:
            candidates += CANDIDATES_FRAME_F32 if prog["dtype"] == "f32" else CANDIDATES_FRAME_F64
    dev = torch.device("cuda:0")
    p = Program(prog)
    p.allocate(dev, fill=0.0)
    bench.fill_inputs(p, prog, dev, 0, prog["grid"]["ghost"][2])
    t0 = time.time()
    plan, cfgs, rep = p.plan_search_ex(generations=generations, population=population, seed=seed,
                                       objective="measured", reps=reps, configs=candidates,
                                       with_configs=True)
    out = {"workload": workload,
           "planner": f"sp_plan_search_ex (objective=measured, generations {generations}, population "
                      f"{population}, seed {seed}, {len(candidates)} candidate configurations; "
                      f"tools/search_plan.py)",
           "search_seconds": time.time() - t0, "search_report": rep, "groups": plan, "configs": cfgs}
    if workload == "C4":  # the unfused baseline's per-kernel pins are plan independent
        fz = json.load(open(os.path.join(ROOT, "configs", "c4_plan.json")))
        out["unfused_configs"] = fz.get("unfused_configs")
        out["unfused_tuner"] = fz.get("unfused_tuner")
    del p
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("--out", default=None)
    ap.add_argument("--generations", type=int, default=12)
    ap.add_argument("--population", type=int, default=16)
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--frame", action="store_true", help="add region-vector (frame) candidates")
    ap.add_argument("--name", default="searched", help="plan name written into C2/C3/C5 plan files")
    a = ap.parse_args()
    out = measured_search(a.workload, a.generations, a.population, a.seed, frame=a.frame)
    print(json.dumps(out["search_report"]), f"{out['search_seconds']:.0f} s")
    for g, c in zip(out["groups"], out["configs"]):
        print(g, c)
    if a.out:
        if a.workload != "C4" and os.path.exists(a.out):
            # C2/C3/C5 plan files hold named plans: add / replace the "searched" entry
            pj = json.load(open(a.out))
            pj.setdefault("plans", {})[a.name] = {"groups": out["groups"], "configs": out["configs"],
                                                      "planner": out["planner"],
                                                      "search_report": out["search_report"]}
            out = pj
        json.dump(out, open(a.out, "w"), indent=1)
        print("wrote", a.out)


if __name__ == "__main__":
    main()
