"""Run one config/mode on the GPU and compare with the oracle (dev tool).

python tools/debug_one.py CONFIG MODE [plan] [key=val ...]
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

from _harness import gpu_run, oracle_outputs, rel_err  # noqa: E402
from synth import programs as P  # noqa: E402


def main():
    cfg, mode = sys.argv[1], sys.argv[2]
    rest = sys.argv[3:]
    plan = "fused"
    opts = {}
    for r in rest:
        if "=" in r:
            k, v = r.split("=")
            opts[k] = int(v)
        else:
            plan = r
    small = {"C1": P.c1(), "C2": P.c2(nx=45, ny=37, nz=29), "C3": P.c3(nx=70, ny=41, nz=33),
             "C5": P.c5(nx=40, ny=23, nz=19), "chain3": P.chain3(),
             "chain3big": P.resize(P.chain3(), 33, 17, 13)}
    prog = small[cfg]
    ref = oracle_outputs(prog, seed=3)
    got = gpu_run(prog, mode, 3, options=opts, plan=prog["plans"][plan])
    for n in ref:
        e = rel_err(got[n], ref[n])
        exact = got[n].tobytes() == ref[n].tobytes()
        print(f"{cfg} {mode} {plan} {opts} {n}: rel err {e:.3e} bit-exact {exact}")


if __name__ == "__main__":
    main()
