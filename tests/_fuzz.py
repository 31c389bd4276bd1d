"""Random legal stencil programs and random plans for fuzz parity.

Programs follow the library's program model (roles respected, reading R3 inside a
kernel, taps within the ghost width); kernels optionally carry loop bounds (R2').
Plans are contiguous cuts of the statement list in program order (every
dependency edge then goes forward), so they fail only on in-group hazards
(R11/R2'), which the library must report instead of computing a wrong result.
"""
import numpy as np


def random_box(rng, n):
    box = []
    for d in range(3):
        lo = int(rng.integers(0, n[d]))
        hi = int(rng.integers(lo + 1, n[d] + 1))
        box += [lo, hi]
    return box


def random_lib_program(rng, n=None, dtype="f64", boxes=False, ghost=2, max_kernels=6):
    if n is None:
        n = (int(rng.integers(5, 70)), int(rng.integers(3, 40)), int(rng.integers(2, 24)))
    n_in = int(rng.integers(1, 3))
    n_w = int(rng.integers(2, 5))
    names = [f"i{a}" for a in range(n_in)] + [f"w{a}" for a in range(n_w)]
    roles = ["in"] * n_in + [str(rng.choice(["temp", "out", "inout", "temp"])) for _ in range(n_w)]
    if "out" not in roles and "inout" not in roles:
        roles[-1] = "out"
    writable = [nm for nm, r in zip(names, roles) if r != "in"]
    kernels = []
    for kk in range(int(rng.integers(2, max_kernels + 1))):
        stmts = []
        outs = [str(v) for v in rng.choice(writable, size=int(rng.integers(1, 3)), replace=False)]
        for out in outs:
            terms = []
            for _ in range(int(rng.integers(1, 7))):
                def rtap():
                    arr = names[int(rng.integers(0, len(names)))]
                    if arr in outs:  # R3: arrays the kernel writes are read at offset 0 only
                        return [arr, 0, 0, 0]
                    if rng.random() < 0.3:
                        return [arr, 0, 0, 0]
                    o = [int(v) for v in rng.integers(-ghost, ghost + 1, size=3)]
                    return [arr] + o
                t = {"c": float(rng.uniform(-1, 1)), "a": rtap()}
                if rng.random() < 0.25:
                    t["b"] = rtap()
                terms.append(t)
            stmts.append({"out": out, "terms": terms})
        k = {"name": f"K{kk}", "stmts": stmts}
        if boxes and rng.random() < 0.5:
            k["box"] = random_box(rng, n)
        kernels.append(k)
    prog = {"name": "fuzz", "dtype": dtype,
            "grid": {"nx": n[0], "ny": n[1], "nz": n[2], "ghost": [ghost] * 3},
            "arrays": [{"name": a, "role": r} for a, r in zip(names, roles)], "kernels": kernels}
    prog["plans"] = {"unfused": [[k["name"]] for k in kernels]}
    return prog


def random_plans(rng, prog, count=3):
    """The single-group plan plus `count` random contiguous cuts (statement granularity,
    so kernels may be split: fission)."""
    refs = [f"{k['name']}:{i}" for k in prog["kernels"] for i in range(len(k["stmts"]))]
    plans = [[refs]]
    for _ in range(count):
        cuts = sorted(set(int(v) for v in rng.integers(1, len(refs), size=int(rng.integers(1, 4)))))
        groups, prev = [], 0
        for c in cuts + [len(refs)]:
            if c > prev:
                groups.append(refs[prev:c])
                prev = c
        plans.append(groups)
    return plans
