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


def _fuses_boxed(prog, plan):
    """Does some group hold a statement of a boxed kernel together with another statement?"""
    boxed = {k["name"] for k in prog["kernels"] if k.get("box") is not None}
    return any(len(g) > 1 and any(r.split(":")[0] in boxed for r in g) for g in plan)


def legal_plans(rng, prog, want=4, tries=60):
    """Up to `want` fusion plans the library accepts (host-side fusion_plan_set: partition,
    order, R11/R2' hazards, resources), each with at least one multi-statement group:
    the single group, the model's greedy plan, then random contiguous cuts.  Plans that
    fuse a boxed kernel with another statement come first.  Returns (plans, rejected),
    rejected = [(plan, sp_status)] for the candidates refused with a plan error."""
    from paper_conf_hpdc_wahibm15_b200 import Program, StencilError
    p = Program(prog)
    cands = random_plans(rng, prog, count=tries)
    try:
        cands.insert(1, p.plan_greedy())
    except StencilError:
        pass
    ok, rejected, seen = [], [], set()
    for plan in cands:
        key = tuple(tuple(g) for g in plan)
        if key in seen or all(len(g) == 1 for g in plan):
            continue
        seen.add(key)
        try:
            p.set_plan(plan)
        except StencilError as e:
            rejected.append((plan, e.code))
            continue
        ok.append(plan)
    ok.sort(key=lambda pl: not _fuses_boxed(prog, pl))  # stable: boxed fusions first
    return ok[:want], rejected


def fuzz_case(seed, boxes, max_draws=12):
    """Seeded fuzz case: programs are drawn from one generator stream until one admits at
    least two accepted fusion plans (boxed cases: the first of them fuses a boxed kernel
    with another statement), so every case really runs fused plans.  Returns
    (program, plans, rejected, draws)."""
    rng = np.random.default_rng(100 * seed + boxes)
    for draw in range(1, max_draws + 1):
        prog = random_lib_program(rng, dtype="f32" if seed % 4 == 3 else "f64", boxes=boxes)
        plans, rejected = legal_plans(rng, prog)
        has_box = any(k.get("box") is not None for k in prog["kernels"])
        if len(plans) >= 2 and (not boxes or (has_box and _fuses_boxed(prog, plans[0]))):
            return prog, plans, rejected, draw
    raise RuntimeError(f"fuzz seed {seed}: no program with fusable plans in {max_draws} draws")
