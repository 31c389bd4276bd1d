"""C4: synthetic SCALE-LES-shaped kernel DAG (BASELINE configs[3]).

The paper gives only counts for SCALE-LES ("over a hundred kernels and tens of
data arrays", mostly memory-bound iterative stencils in the dynamical core,
P:L305 §6.1.1; Table 1 / Table 2: 142 kernels fused into 38 new kernels) and for
HOMME (43 kernels, 30 arrays in Table 1 c1/c2).  This generator builds a
deterministic dynamical-core-like step of 40 kernels over ~30 arrays:

  arrays: S0..S4 (IN, prognostic state), S0n..S4n (OUT, next state),
          M0..M3 (IN, static metric/velocity-like), t* (TEMP pool)
  per state variable v (8 kernels, 5 variables -> 40 kernels):
    2 x diag   d = stencil(S_v or S_{v-1}) [* M_r at p]   (7-pt 70 %, point-wise 30 %)
    4 x flux   f = stencil(7:50 %, 13:25 %, 19:25 %) over a diag temp of v or v-1
                   [* point-wise multiplier from {M_*, S_v}]; one flux kernel per v is
                   multi-output (2 statements: separable for even v, sharing the
                   source for odd v -> fission candidates, §4.1)
    1 x sum    tend = normalised sum of the 5 flux outputs
    1 x update S_v' = 1*S_v + dt*tend  (dt = 1/64)
  TEMPs are assigned by a linear scan in program order (a TEMP is free after its
  last reader; the lowest free id is reused), which creates the WAR/WAW reuse of
  real codes (§3.2.3).  Stencil coefficients are uniform(-1,1) normalised
  to sum|c| = 1 so values stay O(1) through the chain (reading R19).

Data only (no evaluation happens here).
"""
from __future__ import annotations

import numpy as np

from .programs import PT7, PT13, PT19, kernel, stmt, tap, unfused_plan

DT = 1.0 / 64


def _coefs(rng, n):
    c = rng.uniform(-1.0, 1.0, size=n)
    c /= np.sum(np.abs(c))
    return [float(x) for x in c]


def c4(nx=1280, ny=32, nz=256, seed=40, n_vars=5, reuse_temps=True):
    rng = np.random.default_rng(seed)
    # kernels are first built with symbolic temps ("d{v}_{i}", "f{v}_{i}", "tend{v}")
    ks = []
    for v in range(n_vars):
        diag = []
        for i in range(2):
            src = f"S{v}" if (v == 0 or rng.random() < 0.6) else f"S{v-1}"
            shape = PT7 if rng.random() < 0.7 else [(0, 0, 0)]
            mult = f"M{int(rng.integers(0, 4))}" if rng.random() < 0.5 else None
            terms = []
            for o, c in zip(shape, _coefs(rng, len(shape))):
                t = {"c": c, "a": tap(src, o)}
                if mult:
                    t["b"] = tap(mult, (0, 0, 0))
                terms.append(t)
            name = f"d{v}_{i}"
            ks.append(kernel(f"diag{v}_{i}", stmt(name, terms)))
            diag.append(name)
        fluxes = []
        multi_at = int(rng.integers(0, 4))
        for i in range(4):
            def flux_stmt(out, src):
                r = rng.random()
                shape = PT7 if r < 0.5 else (PT13 if r < 0.75 else PT19)
                mult = None
                if rng.random() < 0.5:
                    mult = [f"M{j}" for j in range(4)] + [f"S{v}"]
                    mult = mult[int(rng.integers(0, len(mult)))]
                terms = []
                for o, c in zip(shape, _coefs(rng, len(shape))):
                    t = {"c": c, "a": tap(src, o)}
                    if mult:
                        t["b"] = tap(mult, (0, 0, 0))
                    terms.append(t)
                return stmt(out, terms)

            pool = diag + ([f"d{v-1}_0", f"d{v-1}_1"] if v > 0 else [])
            src = pool[int(rng.integers(0, len(pool)))]
            out = f"f{v}_{i}"
            if i == multi_at:
                if v % 2 == 0:   # separable: second statement reads another diag temp
                    other = [d for d in pool if d != src]
                    src2 = other[int(rng.integers(0, len(other)))]
                else:            # shares the source: not separable
                    src2 = src
                ks.append(kernel(f"flux{v}_{i}", flux_stmt(out, src), flux_stmt(out + "b", src2)))
                fluxes += [out, out + "b"]
            else:
                ks.append(kernel(f"flux{v}_{i}", flux_stmt(out, src)))
                fluxes.append(out)
        ks.append(kernel(f"sum{v}", stmt(f"tend{v}", [{"c": c, "a": tap(f, (0, 0, 0))} for f, c in
                                                      zip(fluxes, _coefs(rng, len(fluxes)))])))
        ks.append(kernel(f"update{v}", stmt(f"S{v}n", [{"c": 1.0, "a": tap(f"S{v}", (0, 0, 0))},
                                                       {"c": DT, "a": tap(f"tend{v}", (0, 0, 0))}])))

    # linear-scan TEMP allocation in program order
    def is_sym(n):
        return n[0] in "dft" and not n.startswith("t_")
    last_read = {}
    for ki, k in enumerate(ks):
        for s in k["stmts"]:
            for t in s["terms"]:
                for key in ("a", "b"):
                    if key in t and is_sym(t[key][0]):
                        last_read[t[key][0]] = ki
    if not reuse_temps:  # every symbolic temp its own array (no WAR/WAW through reuse)
        syms = []
        for k in ks:
            for st in k["stmts"]:
                if is_sym(st["out"]) and st["out"] not in syms:
                    syms.append(st["out"])
        last_read = {n: 1 << 30 for n in syms}  # never freed
    assign, free, used = {}, list(range(64)), 0
    live = {}
    for ki, k in enumerate(ks):
        for s in k["stmts"]:
            n = s["out"]
            if is_sym(n) and n not in assign:
                tid = min(free)
                free.remove(tid)
                assign[n] = tid
                used = max(used, tid + 1)
                live[n] = last_read.get(n, ki)
        for n, lr in list(live.items()):
            if lr <= ki:
                free.append(assign[n])
                del live[n]
    if used > 16 and reuse_temps:
        raise RuntimeError(f"TEMP pool needs {used} > 16 arrays")

    def ren(n):
        return f"t{assign[n]}" if is_sym(n) else n
    for k in ks:
        for s in k["stmts"]:
            s["out"] = ren(s["out"])
            for t in s["terms"]:
                for key in ("a", "b"):
                    if key in t:
                        t[key][0] = ren(t[key][0])
    arrays = [(f"S{v}", "in") for v in range(n_vars)] + [(f"S{v}n", "out") for v in range(n_vars)] + \
             [(f"M{j}", "in") for j in range(4)] + [(f"t{i}", "temp") for i in range(used)]
    p = {
        "name": "C4", "dtype": "f64",
        "grid": {"nx": nx, "ny": ny, "nz": nz, "ghost": [2, 2, 2]},
        "arrays": [{"name": a, "role": r} for a, r in arrays],
        "kernels": ks,
    }
    p["plans"] = {"unfused": unfused_plan(p)}
    return p
