"""Program descriptions for the configurations C1-C5.

These are DATA (kernels, arrays, taps, coefficients, plans) — the same JSON-able
dict is handed to the oracle's own loader and to the product binding's own
loader.  No evaluation happens here.

Program dict schema
-------------------
{
  "name": str, "dtype": "f64" | "f32",
  "grid": {"nx": int, "ny": int, "nz": int, "ghost": [hx, hy, hz]},
  "arrays":  [{"name": str, "role": "in"|"out"|"inout"|"temp"}, ...],
  "kernels": [{"name": str, "stmts": [{"out": str, "terms": [term, ...]}, ...]}, ...],
  "plans":   {plan_name: [[member, ...], ...]}      # groups in execution order
}
term   = {"c": float, "a": [array, dx, dy, dz]}                  -> c * a[p+da]
       | {"c": float, "a": [...], "b": [array, dx, dy, dz]}      -> (c * a[p+da]) * b[p+db]
member = "K"        (every statement of kernel K, program order)
       | "K:i"      (statement i of kernel K — a fission piece)
"""
from __future__ import annotations

import copy

# 7-point neighbourhood in a fixed term order: centre, -x, +x, -y, +y, -z, +z
PT7 = [(0, 0, 0), (-1, 0, 0), (1, 0, 0), (0, -1, 0), (0, 1, 0), (0, 0, -1), (0, 0, 1)]
# 13-point: centre and +-1, +-2 along each axis
PT13 = [(0, 0, 0)] + [o for r in (1, 2) for o in
                      ((-r, 0, 0), (r, 0, 0), (0, -r, 0), (0, r, 0), (0, 0, -r), (0, 0, r))]
# 19-point: centre, 6 faces, 12 edges
PT19 = PT7 + [(dx, dy, 0) for dx in (-1, 1) for dy in (-1, 1)] \
           + [(dx, 0, dz) for dx in (-1, 1) for dz in (-1, 1)] \
           + [(0, dy, dz) for dy in (-1, 1) for dz in (-1, 1)]


def tap(arr, o):
    return [arr, int(o[0]), int(o[1]), int(o[2])]


def stencil_terms(arr, offsets, coefs):
    return [{"c": float(c), "a": tap(arr, o)} for o, c in zip(offsets, coefs)]


def stmt(out, terms):
    return {"out": out, "terms": terms}


def kernel(name, *stmts):
    return {"name": name, "stmts": list(stmts)}


def unfused_plan(prog):
    return [[k["name"]] for k in prog["kernels"]]


# ---------------------------------------------------------------- C1 -----
def c1(n=32, dyadic=False):
    """2-kernel chain: 7-point Jacobi then 7-point Laplacian (BASELINE configs[0])."""
    jac = [0.25] + [0.125] * 6 if dyadic else [1.0 / 7.0] * 7
    lap = [1.0] * 6 + [-6.0]
    lap_off = PT7[1:] + [PT7[0]]
    return {
        "name": "C1", "dtype": "f64",
        "grid": {"nx": n, "ny": n, "nz": n, "ghost": [1, 1, 1]},
        "arrays": [{"name": "A", "role": "in"}, {"name": "T", "role": "temp"},
                   {"name": "B", "role": "out"}],
        "kernels": [kernel("K1", stmt("T", stencil_terms("A", PT7, jac))),
                    kernel("K2", stmt("B", stencil_terms("T", lap_off, lap)))],
        "plans": {"unfused": [["K1"], ["K2"]], "fused": [["K1", "K2"]]},
    }


# ---------------------------------------------------------------- C2 -----
def c2_kernels(phi, phin, u, v, w, gx, gy, gz, fx, fy, fz, d, kappa=1.0 / 16, dt=1.0 / 64,
               suffix=""):
    """Diffusion-advection step: gradient, flux, divergence, update (4 kernels)."""
    return [
        kernel("grad" + suffix,
               stmt(gx, [{"c": 0.5, "a": tap(phi, (1, 0, 0))}, {"c": -0.5, "a": tap(phi, (-1, 0, 0))}]),
               stmt(gy, [{"c": 0.5, "a": tap(phi, (0, 1, 0))}, {"c": -0.5, "a": tap(phi, (0, -1, 0))}]),
               stmt(gz, [{"c": 0.5, "a": tap(phi, (0, 0, 1))}, {"c": -0.5, "a": tap(phi, (0, 0, -1))}])),
        kernel("flux" + suffix,
               stmt(fx, [{"c": -kappa, "a": tap(gx, (0, 0, 0))},
                         {"c": 1.0, "a": tap(u, (0, 0, 0)), "b": tap(phi, (0, 0, 0))}]),
               stmt(fy, [{"c": -kappa, "a": tap(gy, (0, 0, 0))},
                         {"c": 1.0, "a": tap(v, (0, 0, 0)), "b": tap(phi, (0, 0, 0))}]),
               stmt(fz, [{"c": -kappa, "a": tap(gz, (0, 0, 0))},
                         {"c": 1.0, "a": tap(w, (0, 0, 0)), "b": tap(phi, (0, 0, 0))}])),
        kernel("div" + suffix,
               stmt(d, [{"c": 0.5, "a": tap(fx, (1, 0, 0))}, {"c": -0.5, "a": tap(fx, (-1, 0, 0))},
                        {"c": 0.5, "a": tap(fy, (0, 1, 0))}, {"c": -0.5, "a": tap(fy, (0, -1, 0))},
                        {"c": 0.5, "a": tap(fz, (0, 0, 1))}, {"c": -0.5, "a": tap(fz, (0, 0, -1))}])),
        kernel("update" + suffix,
               stmt(phin, [{"c": 1.0, "a": tap(phi, (0, 0, 0))}, {"c": -dt, "a": tap(d, (0, 0, 0))}])),
    ]


def c2(n=256, nx=None, ny=None, nz=None):
    """4-kernel diffusion-advection chain (BASELINE configs[1]); kappa=1/16, dt=1/64."""
    arrays = [("phi", "in"), ("u", "in"), ("v", "in"), ("w", "in"),
              ("gx", "temp"), ("gy", "temp"), ("gz", "temp"),
              ("Fx", "temp"), ("Fy", "temp"), ("Fz", "temp"), ("D", "temp"), ("phin", "out")]
    p = {
        "name": "C2", "dtype": "f64",
        "grid": {"nx": nx or n, "ny": ny or n, "nz": nz or n, "ghost": [1, 1, 1]},
        "arrays": [{"name": a, "role": r} for a, r in arrays],
        "kernels": c2_kernels("phi", "phin", "u", "v", "w", "gx", "gy", "gz", "Fx", "Fy", "Fz", "D"),
    }
    p["plans"] = {"unfused": unfused_plan(p), "fused": [["grad", "flux", "div", "update"]]}
    return p


# ---------------------------------------------------------------- C3 -----
def c3(n=512, nx=None, ny=None, nz=None):
    """Fission+fusion case (BASELINE configs[2]): K0 is multi-output and separable.

    Dyadic normalised stencils (sum|c| = 1): 7-pt (1/4, 6 x 1/8), 13-pt (1/4, 12 x 1/16).
    """
    s7 = [0.25] + [0.125] * 6
    s13 = [0.25] + [0.0625] * 12
    plus = lambda arr: {"c": 1.0, "a": tap(arr, (0, 0, 0))}
    ks = [
        kernel("K0", stmt("P", stencil_terms("A", PT7, s7)), stmt("Q", stencil_terms("B", PT7, s7))),
        kernel("K1", stmt("P1", stencil_terms("P", PT7, s7))),
        kernel("K2", stmt("P2", stencil_terms("P1", PT13, s13))),
        kernel("K3", stmt("O1", stencil_terms("P2", PT7, s7) + [plus("A")])),
        kernel("K4", stmt("Q1", stencil_terms("Q", PT7, s7))),
        kernel("K5", stmt("Q2", stencil_terms("Q1", PT13, s13))),
        kernel("K6", stmt("O2", stencil_terms("Q2", PT7, s7) + [plus("B")])),
        kernel("K7", stmt("OUT", [plus("O1"), plus("O2")])),
    ]
    arrays = [("A", "in"), ("B", "in"), ("P", "temp"), ("Q", "temp"), ("P1", "temp"),
              ("P2", "temp"), ("Q1", "temp"), ("Q2", "temp"), ("O1", "temp"), ("O2", "temp"),
              ("OUT", "out")]
    p = {
        "name": "C3", "dtype": "f32",
        "grid": {"nx": nx or n, "ny": ny or n, "nz": nz or n, "ghost": [2, 2, 2]},
        "arrays": [{"name": a, "role": r} for a, r in arrays],
        "kernels": ks,
    }
    p["plans"] = {
        "unfused": unfused_plan(p),
        "fused": [["K0", "K1", "K2", "K3"], ["K4", "K5", "K6", "K7"]],
        "fission_fused": [["K0:0", "K1", "K2", "K3"], ["K0:1", "K4", "K5", "K6", "K7"]],
        "single": [["K0", "K1", "K2", "K3", "K4", "K5", "K6", "K7"]],
    }
    return p


# ---------------------------------------------------------------- C5 -----
def c5(nx=1024, ny=1024, nz=128, ntracers=3):
    """Weak-scaling DAG (BASELINE configs[4]): 3 tracers x C2's 4 kernels, shared u, v, w.

    TEMPs are reused across tracers (WAW/WAR across groups); nz is the per-GPU slab.
    """
    temps = ["gx", "gy", "gz", "Fx", "Fy", "Fz", "D"]
    arrays = [(f"phi{t}", "in") for t in range(ntracers)] + \
             [(f"phin{t}", "out") for t in range(ntracers)] + \
             [("u", "in"), ("v", "in"), ("w", "in")] + [(a, "temp") for a in temps]
    ks = []
    for t in range(ntracers):
        ks += c2_kernels(f"phi{t}", f"phin{t}", "u", "v", "w", *temps, suffix=str(t))
    p = {
        "name": "C5", "dtype": "f64",
        "grid": {"nx": nx, "ny": ny, "nz": nz, "ghost": [1, 1, 1]},
        "arrays": [{"name": a, "role": r} for a, r in arrays],
        "kernels": ks,
    }
    p["plans"] = {
        "unfused": unfused_plan(p),
        "fused": [[k["name"] for k in ks[4 * t:4 * t + 4]] for t in range(ntracers)],
        "single": [[k["name"] for k in ks]],
    }
    return p


def chain3():
    """Hand-computed 3-kernel chain (SURVEY.md §8(c) pin P4), 4^3 grid, ghost 1."""
    p = {
        "name": "chain3", "dtype": "f64",
        "grid": {"nx": 4, "ny": 4, "nz": 4, "ghost": [1, 1, 1]},
        "arrays": [{"name": "A", "role": "in"}, {"name": "B", "role": "in"},
                   {"name": "T1", "role": "temp"}, {"name": "T2", "role": "temp"},
                   {"name": "O", "role": "out"}],
        "kernels": [
            kernel("K1", stmt("T1", [{"c": 1.0, "a": tap("A", (0, 0, 0))},
                                     {"c": 1.0, "a": tap("A", (1, 0, 0))}])),
            kernel("K2", stmt("T2", [{"c": 2.0, "a": tap("T1", (0, 0, 0))},
                                     {"c": -1.0, "a": tap("T1", (0, -1, 0))}])),
            kernel("K3", stmt("O", [{"c": 0.5, "a": tap("T2", (0, 0, 1))},
                                    {"c": 0.25, "a": tap("T2", (-1, 0, 0))},
                                    {"c": 1.0, "a": tap("B", (0, 0, 0))}])),
        ],
    }
    p["plans"] = {"unfused": unfused_plan(p), "fused": [["K1", "K2", "K3"]]}
    return p


def resize(prog, nx, ny, nz):
    """Same program on another grid (parity tests at oracle-friendly sizes)."""
    q = copy.deepcopy(prog)
    q["grid"].update({"nx": nx, "ny": ny, "nz": nz})
    return q


CONFIGS = {"C1": c1, "C2": c2, "C3": c3, "C5": c5}
