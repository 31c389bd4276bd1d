"""Workload for compute-sanitizer runs (tests/test_gpu_sanitizer.py): small C1, C2,
chain3, C3 and C4 programs, unfused and fused (parity build; fused also in the
region-vector "frame" form), each checked bit-exact against the oracle.  Usage: python tests/_sanitize_case.py [case ...]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))


def cases():
    from synth import programs as P
    from synth.scale_les import c4
    c4p = c4(nx=64, ny=32, nz=8)
    c4p["plans"]["fused"] = json.load(open(os.path.join(ROOT, "configs", "c4_plan.json")))["groups"]
    return {"C1": (P.c1(n=16), "fused"), "C2": (P.c2(nx=24, ny=16, nz=8), "fused"),
            "chain3": (P.resize(P.chain3(), 19, 11, 7), "fused"),
            "C3": (P.c3(nx=40, ny=12, nz=6), "fission_fused"), "C4": (c4p, "fused")}


def main(names):
    from _harness import assert_close, gpu_run, oracle_outputs
    all_cases = cases()
    for name in names or list(all_cases):
        prog, plan = all_cases[name]
        ref = oracle_outputs(prog, seed=3)
        for mode in ("unfused", "fused"):
            got = gpu_run(prog, mode, 3, options={"fmad": 0}, plan=prog["plans"][plan])
            assert_close(prog, got, ref, exact=True)
        # region-vector (frame) form: edge lanes read past row ends into the plane guards
        for opts in ({"frame": 1}, {"frame": 1, "tile_x": 16, "tile_y": 3, "threads": 64, "zchunk": 2},
                     {"frame": 1, "fastpath": 1}):
            got = gpu_run(prog, "fused", 3, options=dict(opts, fmad=0), plan=prog["plans"][plan])
            assert_close(prog, got, ref, exact=True)
        print(f"{name}: ok", flush=True)


if __name__ == "__main__":
    main(sys.argv[1:])
