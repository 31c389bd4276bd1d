"""Streaming probe programs for kernel studies (dev tool, not a workload):
one kernel on the C4 grid (1280x32x256 fp64, ghost 2) whose only statement reads
n_pt inputs at offset 0 and n_st inputs through a 7- or 19-point stencil.

    python tools/sweep.py probe:8:0 --grid ...     (8 point-wise inputs, none stencilled)
    python tools/sweep.py probe:4:4:19 ...         (4 point-wise, 4 through a 19-point stencil)
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from synth.programs import PT7, PT19, kernel, stmt, tap  # noqa: E402


def probe(spec, nx=1280, ny=32, nz=256):
    parts = [int(v) for v in spec.split(":")[1:]]
    n_pt, n_st = parts[0], parts[1]
    offs = PT19 if (len(parts) > 2 and parts[2] == 19) else PT7
    arrays = [{"name": f"P{i}", "role": "in"} for i in range(n_pt)]
    arrays += [{"name": f"Q{i}", "role": "in"} for i in range(n_st)]
    arrays.append({"name": "O", "role": "out"})
    terms = [{"c": 0.125, "a": tap(f"P{i}", (0, 0, 0))} for i in range(n_pt)]
    for i in range(n_st):
        terms += [{"c": 1.0 / 64, "a": tap(f"Q{i}", o)} for o in offs]
    return {"name": spec, "dtype": "f64",
            "grid": {"nx": nx, "ny": ny, "nz": nz, "ghost": [2, 2, 2]},
            "arrays": arrays, "kernels": [kernel("probe", stmt("O", terms))],
            "plans": {"fused": [["probe"]]}}
