"""Shared test plumbing: run a program on the GPU through the C-ABI binding and
on the CPU oracle, on the same seeded inputs, and compare (reading R17).

The two sides share only synth/ (input generator + program descriptions)."""
from __future__ import annotations

import numpy as np

from oracle import OracleProgram, dense_arrays


def tolerance(dtype):
    return 1e-12 if dtype == "f64" else 1e-5


def compared_arrays(prog):
    return [a["name"] for a in prog["arrays"] if a["role"] in ("out", "inout")]


def interior(prog, dense):
    g = prog["grid"]
    hx, hy, hz = g["ghost"]
    return dense[hz:hz + g["nz"], hy:hy + g["ny"], hx:hx + g["nx"]]


def oracle_outputs(prog, seed, poison=True, inputs=None):
    arrs = inputs if inputs is not None else dense_arrays(prog, seed, poison_temp=poison)
    arrs = {k: v.copy() for k, v in arrs.items()}
    OracleProgram(prog).run(arrs)
    return {n: interior(prog, arrs[n]).copy() for n in compared_arrays(prog)}


def gpu_program(prog, options=None, plan=None):
    from paper_conf_hpdc_wahibm15_b200 import Program
    p = Program(prog, options=options or {})
    if plan is not None:
        p.set_plan(plan)
    return p


def gpu_run(prog, mode, seed, options=None, plan=None, poison=True, inputs=None, program=None,
            repeat=1):
    """Returns {name: interior ndarray} of OUT/INOUT arrays after one run."""
    import torch
    p = program or gpu_program(prog, options, plan if mode == "fused" else None)
    if program is not None and plan is not None and mode == "fused":
        p.set_plan(plan)
    dev = torch.device("cuda:0")
    arrs = inputs if inputs is not None else dense_arrays(prog, seed, poison_temp=poison)
    p.allocate(dev)
    for name, dense in arrs.items():
        p.padded_view(p.tensors[name]).copy_(torch.from_numpy(dense))
    for _ in range(repeat):
        p.run(mode)
    torch.cuda.synchronize()
    return {n: p.interior_view(p.tensors[n]).cpu().numpy().copy() for n in compared_arrays(prog)}


def rel_err(got, ref):
    if not np.all(np.isfinite(got)):
        return float("inf")
    den = max(float(np.max(np.abs(ref))), 1e-300)
    return float(np.max(np.abs(got.astype(np.float64) - ref.astype(np.float64)))) / den


def assert_close(prog, got, ref, exact=False):
    for name in ref:
        assert got[name].shape == ref[name].shape, name
        if exact:
            eq = got[name].tobytes() == ref[name].tobytes()
            if not eq:
                bad = np.argwhere(got[name] != ref[name])
                raise AssertionError(f"{name}: not bit-exact, {len(bad)} differing points, first "
                                     f"{bad[:5].tolist()} got {got[name][tuple(bad[0])]} "
                                     f"want {ref[name][tuple(bad[0])]}")
        else:
            e = rel_err(got[name], ref[name])
            assert e <= tolerance(prog["dtype"]), f"{name}: rel err {e}"


def window_field(seed, aid, origin, n, h, dtype):
    """Generated values (synth/fields.py recipe) of one array on the window whose interior
    starts at global `origin`, with ghost width h: the same numbers the GPU slab holds."""
    from synth.fields import bits_to_unit, pack, seed_mix, splitmix64
    i = np.arange(origin[0] - h[0], origin[0] + n[0] + h[0], dtype=np.int64)
    j = np.arange(origin[1] - h[1], origin[1] + n[1] + h[1], dtype=np.int64)
    k = np.arange(origin[2] - h[2], origin[2] + n[2] + h[2], dtype=np.int64)
    key = pack(i[None, None, :], j[None, :, None], k[:, None, None])
    return np.ascontiguousarray(bits_to_unit(splitmix64(key ^ seed_mix(seed, aid)), dtype))


def accumulated_reach(prog):
    """Per axis, the sum over kernels of each kernel's largest tap offset: a window of the
    grid evaluated alone is exact this far inside its edges (conservative)."""
    m = [0, 0, 0]
    for k in prog["kernels"]:
        for d in range(3):
            m[d] += max(abs(t[x][1 + d]) for s in k["stmts"] for t in s["terms"]
                        for x in ("a", "b") if x in t)
    return m
