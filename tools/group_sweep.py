"""Isolated timing of one fused group under variants of its pinned configuration and of
program options (dev tool).

python tools/group_sweep.py C4 3 'prefetch=1' 'prefetch=2,minblocks=4' ...

Each spec is comma-separated key=value; keys of sp_tile_config modify the group's pin,
other keys are program options.  Every variant: median of 9 launches, each after a
read-only L2 flush; regs / smem / resident CTAs from the library's report.
"""
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_hpdc_wahibm15_b200 import Program, StencilError  # noqa: E402
from paper_conf_hpdc_wahibm15_b200._abi import SpTileConfig  # noqa: E402

TILE_KEYS = {f for f, _ in SpTileConfig._fields_}


def main():
    w, g = sys.argv[1], int(sys.argv[2])
    prog = bench.load_workload(w)
    dev = torch.device("cuda:0")
    base_pin = dict((bench.tuned_configs(prog) or [None] * 64)[g] or {})
    pts = prog["grid"]["nx"] * prog["grid"]["ny"] * prog["grid"]["nz"]
    flush = torch.ones(32 << 20, dtype=torch.float64, device=dev)
    tensors = None
    for spec in [""] + sys.argv[3:]:
        kv = {k: int(v) for k, v in (x.split("=") for x in spec.split(",") if x)}
        pin = dict(base_pin, **{k: v for k, v in kv.items() if k in TILE_KEYS})
        opts = {k: v for k, v in kv.items() if k not in TILE_KEYS}
        p = Program(prog, options=opts)
        p.set_plan(bench.plan_of(prog))
        bench.apply_tuning(p, prog)
        try:
            p.tune("fused", g, pin)
        except StencilError as e:
            print(f"{spec or 'base':34s} does not fit: {e}")
            continue
        if tensors is None:
            p.allocate(dev, fill=0.0)
            bench.fill_inputs(p, prog, dev, 0, prog["grid"]["ghost"][2])
            tensors = p.tensors
        else:
            for n, t in tensors.items():
                p.bind(n, t)
        p.run_launch("fused", g)
        torch.cuda.synchronize()
        ts = []
        for _ in range(9):
            flush.sum()
            s, e = torch.cuda.Event(True), torch.cuda.Event(True)
            s.record()
            p.run_launch("fused", g)
            e.record()
            torch.cuda.synchronize()
            ts.append(s.elapsed_time(e))
        t = statistics.median(ts)
        r = p.report("fused", g)
        print(f"{spec or 'base':34s} {t * 1e3:8.1f} us  {r['bytes_alg'] * pts / t / 1e6:6.0f} GB/s  "
              f"regs {r['regs_per_thread']:3d} smem {r['smem_bytes']:6d} thr {r['threads']} "
              f"tile {r['tile_x']}x{r['tile_y']}x{r['zchunk']} pf {r['prefetch']}", flush=True)


if __name__ == "__main__":
    main()
