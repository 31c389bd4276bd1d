"""Time one launch of a workload across explicit tile/block configurations (dev tool).

python tools/sweep.py C2 --group 0 [--plan file.json] [--mode fused] --cfg "tile_x=32,block_x=2,threads=64,block_y=2,block_cby=1,zchunk=32" ...
Each --cfg is a comma-separated option list; prints time, GB/s (alg/exec), regs, smem, model.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_hpdc_wahibm15_b200 import Program, StencilError  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload")
    ap.add_argument("--group", type=int, default=0)
    ap.add_argument("--mode", default="fused")
    ap.add_argument("--plan", default=None)
    ap.add_argument("--plan-name", default="fused", help="named plan of the workload")
    ap.add_argument("--cfg", action="append", default=[])
    ap.add_argument("--iters", type=int, default=10)
    ap.add_argument("--grid", action="store_true", help="enumerate tile/block combinations")
    ap.add_argument("--zchunk", default="32", help="comma list of z-chunk lengths")
    ap.add_argument("--tx", default="32,64")
    ap.add_argument("--pf", default="", help="comma list of prefetch depths to cross with --grid")
    ap.add_argument("--apply-tuning", action="store_true", help="pin the plan's tuned configs first")
    a = ap.parse_args()
    if a.grid:
        for tx in [int(v) for v in a.tx.split(",")]:
            for bx in (1, 2, 4):
                for nt in (64, 128, 256):
                    xt = tx // bx
                    if tx % bx or nt % xt or xt > nt:
                        continue
                    for by in (1, 2, 4):
                        for cb in (1, 2):
                            ty = nt // xt * by * cb
                            if ty > 32:
                                continue
                            for zc in a.zchunk.split(","):
                                c = (f"tile_x={tx},block_x={bx},threads={nt},block_y={by},"
                                     f"block_cby={cb},tile_y={ty},zchunk={zc}")
                                if a.pf:
                                    a.cfg += [c + f",prefetch={pf}" for pf in a.pf.split(",")]
                                else:
                                    a.cfg.append(c)
    if a.workload.startswith("probe:"):
        from probe_programs import probe
        prog = probe(a.workload)
    else:
        prog = bench.load_workload(a.workload)
    plan = json.load(open(a.plan))["groups"] if a.plan else bench.plan_of(prog, a.plan_name)
    dev = torch.device("cuda:0")
    flush = torch.ones(32 << 20, dtype=torch.float64, device=dev)  # read-only L2 flush (no dirty lines)
    base = None
    pts = prog["grid"]["nx"] * prog["grid"]["ny"] * prog["grid"]["nz"]
    for cfg in [""] + a.cfg:
        opts = {}
        for kv in filter(None, cfg.split(",")):
            k, v = kv.split("=")
            opts[k.strip()] = int(v)
        try:
            p = Program(prog, options=opts)
            if a.mode == "fused":
                p.set_plan(plan)
                if a.apply_tuning:
                    bench.apply_tuning(p, prog)
            if base is None:
                p.allocate(dev, fill=0.0)
                bench.fill_inputs(p, prog, dev, 0, prog["grid"]["ghost"][2])
                base = p.tensors
            else:
                for n, t in base.items():
                    p.bind(n, t)
            r = p.report(a.mode, a.group)
            p.run_launch(a.mode, a.group)
            torch.cuda.synchronize()
            ts = []
            for _ in range(a.iters):
                flush.sum()
                s, e = torch.cuda.Event(True), torch.cuda.Event(True)
                s.record()
                p.run_launch(a.mode, a.group)
                e.record()
                torch.cuda.synchronize()
                ts.append(s.elapsed_time(e))
            t = sorted(ts)[len(ts) // 2] * 1e-3
            r = p.report(a.mode, a.group)
            print(f"{cfg or 'chooser':70s} {t*1e6:8.1f} us alg {r['bytes_alg']*pts/t/1e9:6.0f} exec "
                  f"{r['bytes_exec']*pts/t/1e9:6.0f} GB/s | {r['tile_x']}x{r['tile_y']}x{r['zchunk']} "
                  f"nt{r['threads']} b{r['block_x']}x{r['block_y']}x{r['block_cby']} regs "
                  f"{r['regs_per_thread']} smem {r['smem_bytes']} ctas {r['grid_ctas']} model "
                  f"{r['t_model_us']:.0f} us smem/pt {r['smem_bytes_pt']:.0f}", flush=True)
        except StencilError as ex:
            print(f"{cfg:70s} ERROR {ex}", flush=True)


if __name__ == "__main__":
    main()
