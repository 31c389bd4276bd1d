"""Quick device timing of a config's launches (dev tool, not the bench contract).

python tools/quick_time.py C2 [plan] [--opt key=val ...]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_hpdc_wahibm15_b200 import Program  # noqa: E402
from synth import programs as P  # noqa: E402
from synth.fields import field_torch  # noqa: E402


def get_prog(name):
    if name == "C4":
        from synth.scale_les import c4
        return c4()
    return P.CONFIGS[name]()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("plans", nargs="*", default=None)
    ap.add_argument("--opt", action="append", default=[])
    ap.add_argument("--iters", type=int, default=10)
    a = ap.parse_args()
    prog = get_prog(a.config)
    opts = {kv.split("=")[0]: int(kv.split("=")[1]) for kv in a.opt}
    dev = torch.device("cuda:0")
    p = Program(prog, options=opts)
    p.allocate(dev, fill=0.0)
    for aid, arr in enumerate(prog["arrays"]):
        v = field_torch(1, aid, p.n, p.ghost, prog["dtype"], dev)
        p.padded_view(p.tensors[arr["name"]]).copy_(v)
    pts = p.n[0] * p.n[1] * p.n[2]
    flush = torch.ones(32 << 20, dtype=torch.float64, device=dev)  # read-only L2 flush (no dirty lines)
    plans = a.plans or [k for k in prog["plans"] if k != "unfused"]
    for mode, plan in [("unfused", None)] + [("fused", pl) for pl in plans]:
        if plan:
            p.set_plan(prog["plans"][plan])
        reps = p.reports(mode)
        for _ in range(3):
            p.run(mode)
        torch.cuda.synchronize()
        # per-launch times
        tot = 0.0
        for i, r in enumerate(reps):
            ts = []
            for _ in range(a.iters):
                flush.sum()
                s, e = torch.cuda.Event(True), torch.cuda.Event(True)
                s.record()
                p.run_launch(mode, i)
                e.record()
                torch.cuda.synchronize()
                ts.append(s.elapsed_time(e))
            t = sorted(ts)[len(ts) // 2] * 1e-3
            tot += t
            print(f"  {mode:8s} {plan or '':14s} L{i:02d} {t*1e6:9.1f} us  alg {r['bytes_alg']*pts/t/1e9:7.1f} GB/s"
                  f"  exec {r['bytes_exec']*pts/t/1e9:7.1f} GB/s  tile {r['tile_x']}x{r['tile_y']}x{r['zchunk']}"
                  f" nt {r['threads']} smem {r['smem_bytes']} regs {r['regs_per_thread']} ctas {r['grid_ctas']}")
        alg = sum(r["bytes_alg"] for r in reps) * pts
        print(f"{a.config} {mode} {plan or ''}: {tot*1e3:.3f} ms/step  {alg/tot/1e9:.1f} GB/s alg  "
              f"{pts/tot/1e9:.2f} Gpt/s")


if __name__ == "__main__":
    main()
