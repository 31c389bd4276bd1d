"""Pins of the CPU oracle against what the paper and mathematics fix.

Every test here checks oracle/ against something other than itself: closed
forms, hand values (tests/golden/), exactness properties of binary arithmetic,
an independent slicing evaluator, and the rejection of ill-defined programs.
Chosen so a dropped term, a wrong sign, a transposed axis or a wrong summation
order fails at least one of them.
"""
import json
import os

import numpy as np
import pytest

import _numpy_eval
from oracle import OracleProgram, dense_arrays
from synth import programs as P

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def coords(prog):
    g = prog["grid"]
    hx, hy, hz = g["ghost"]
    i = np.arange(-hx, g["nx"] + hx)[None, None, :]
    j = np.arange(-hy, g["ny"] + hy)[None, :, None]
    k = np.arange(-hz, g["nz"] + hz)[:, None, None]
    return i, j, k


def filled(prog, funcs, default=0.0):
    """Dense padded arrays whose every point (ghosts included) holds funcs[name](i,j,k)."""
    i, j, k = coords(prog)
    dt = np.float64 if prog["dtype"] == "f64" else np.float32
    shape = np.broadcast(i, j, k).shape
    out = {}
    for a in prog["arrays"]:
        f = funcs.get(a["name"])
        v = np.full(shape, default, dtype=dt) if f is None else \
            np.ascontiguousarray(np.broadcast_to(f(i, j, k), shape).astype(dt))
        out[a["name"]] = v
    return out


def interior(prog, arr):
    g = prog["grid"]
    hx, hy, hz = g["ghost"]
    return arr[hz:hz + g["nz"], hy:hy + g["ny"], hx:hx + g["nx"]]


def poison(prog, arrays, names):
    for n in names:
        interior(prog, arrays[n])[...] = np.nan


# ------------------------------------------------------------- P1 constant field
@pytest.mark.parametrize("dtype", ["f64", "f32"])
@pytest.mark.parametrize("const", [0.75, -3.5, 1024.0])
def test_p1_constant_field_dyadic_exact(dtype, const):
    """Normalised dyadic 7-pt stencil (1/4, 6 x 1/8) maps a constant field to itself exactly."""
    prog = P.c1(n=6, dyadic=True)
    prog["dtype"] = dtype
    # K2 (Laplacian) of a constant is exactly 0; K1 of a constant is exactly const
    arrs = filled(prog, {"A": lambda i, j, k: const + 0 * i, "T": lambda i, j, k: const + 0 * i})
    poison(prog, arrs, ["T", "B"])
    OracleProgram(prog).run(arrs)
    assert np.all(interior(prog, arrs["T"]) == const)
    assert np.all(interior(prog, arrs["B"]) == 0.0)


def test_p1_constant_field_one_seventh_within_ulp():
    prog = P.c1(n=5, dyadic=False)
    c = 0.3
    arrs = filled(prog, {"A": lambda i, j, k: c + 0 * i, "T": lambda i, j, k: c + 0 * i})
    OracleProgram(prog).run(arrs)
    t = interior(prog, arrs["T"])
    assert np.max(np.abs(t - c)) <= 4 * np.spacing(c)


# ------------------------------------------------------------- P2 linear field
@pytest.mark.parametrize("abcd", [(1, 0, 0, 0), (0, 1, 0, 0), (0, 0, 1, 0), (3, -2, 5, 7),
                                  (-1, 4, -3, 0.5)])
def test_p2_centred_difference_of_linear_field_is_exact(abcd):
    """0.5 f[p+e] - 0.5 f[p-e] of f = a i + b j + c k + d is exactly the slope along e;
    separate axes catch a transposed offset, asymmetric slopes a wrong sign."""
    a, b, c, d = abcd
    prog = P.c2(nx=6, ny=5, nz=4)
    f = lambda i, j, k: a * i + b * j + c * k + d + 0.0 * i
    arrs = filled(prog, {"phi": f})
    poison(prog, arrs, ["gx", "gy", "gz"])
    prog1 = dict(prog, kernels=prog["kernels"][:1])  # gradient kernel only
    OracleProgram(prog1).run(arrs)
    assert np.all(interior(prog, arrs["gx"]) == a)
    assert np.all(interior(prog, arrs["gy"]) == b)
    assert np.all(interior(prog, arrs["gz"]) == c)


def test_p2_laplacian_of_linear_field_is_zero():
    prog = P.c1(n=5)
    f = lambda i, j, k: 2 * i - 3 * j + 5 * k + 1 + 0.0 * i
    arrs = filled(prog, {"T": f})
    prog2 = dict(prog, kernels=prog["kernels"][1:])
    OracleProgram(prog2).run(arrs)
    assert np.all(interior(prog, arrs["B"]) == 0.0)


# ------------------------------------------------------------- P3 C1 closed form
def test_p3_c1_quadratic_dyadic_exact():
    """A = i^2+j^2+k^2: dyadic Jacobi gives T = A + 3/4, Laplacian(T) = 6, exactly."""
    prog = P.c1(n=8, dyadic=True)
    A = lambda i, j, k: (i * i + j * j + k * k) + 0.0 * i
    arrs = filled(prog, {"A": A, "T": lambda i, j, k: A(i, j, k) + 0.75})
    poison(prog, arrs, ["T", "B"])
    OracleProgram(prog).run(arrs)
    i, j, k = coords(prog)
    assert np.array_equal(interior(prog, arrs["T"]), interior(prog, np.broadcast_to(
        A(i, j, k) + 0.75, arrs["T"].shape)))
    assert np.all(interior(prog, arrs["B"]) == 6.0)


def test_p3_c1_quadratic_one_seventh():
    """Jacobi 1/7: T = A + 6/7 and Laplacian(T) = 6 up to rounding (rel 1e-12)."""
    prog = P.c1(n=16)
    A = lambda i, j, k: (i * i + j * j + k * k) + 0.0 * i
    arrs = filled(prog, {"A": A, "T": lambda i, j, k: A(i, j, k) + 6.0 / 7.0})
    poison(prog, arrs, ["T", "B"])
    OracleProgram(prog).run(arrs)
    B = interior(prog, arrs["B"])
    assert np.max(np.abs(B - 6.0)) / 6.0 < 1e-12


# ------------------------------------------------------------- P4 hand values
def test_p4_chain3_golden():
    gold = json.load(open(os.path.join(GOLDEN, "chain3.json")))
    prog = P.chain3()
    arrs = filled(prog, {
        "A": lambda i, j, k: i + 2 * j + 4 * k + 0.0 * i,
        "B": lambda i, j, k: 1.0 + 0 * i,
        "T1": lambda i, j, k: 2 * i + 4 * j + 8 * k + 1.0 + 0 * i,
        "T2": lambda i, j, k: 2 * i + 4 * j + 8 * k + 5.0 + 0 * i,
    })
    poison(prog, arrs, ["T1", "T2", "O"])
    OracleProgram(prog).run(arrs)
    O = interior(prog, arrs["O"])
    for p in gold["points"]:
        assert O[p["k"], p["j"], p["i"]] == p["O"], p
    ci, cj, ck, c0 = gold["closed_form"]["O"]
    i, j, k = np.meshgrid(np.arange(4), np.arange(4), np.arange(4), indexing="xy")
    # meshgrid(xy) gives [j][i][k]; build [k][j][i] explicitly instead
    kk, jj, ii = np.meshgrid(np.arange(4), np.arange(4), np.arange(4), indexing="ij")
    assert np.array_equal(O, ci * ii + cj * jj + ck * kk + c0)
    for name in ("T1", "T2"):
        ci, cj, ck, c0 = gold["closed_form"][name]
        assert np.array_equal(interior(prog, arrs[name]), ci * ii + cj * jj + ck * kk + c0)


# ------------------------------------------------------------- P12 C2 linear field
def test_p12_c2_linear_field_exact():
    """phi = i + 2j + 3k, (u,v,w) = (0.5, 0.25, -0.125), kappa = 1/16, dt = 1/64:
    D = u*1 + v*2 + w*3 = 0.625 and phin = phi - 0.009765625, exactly.
    TEMP ghosts carry their analytic values (g = (1,2,3), F = -kappa g + (u,v,w) phi)."""
    prog = P.c2(n=6)
    kap = 1.0 / 16
    phi = lambda i, j, k: i + 2 * j + 3 * k + 0.0 * i
    arrs = filled(prog, {
        "phi": phi, "u": lambda i, j, k: 0.5 + 0 * i, "v": lambda i, j, k: 0.25 + 0 * i,
        "w": lambda i, j, k: -0.125 + 0 * i,
        "gx": lambda i, j, k: 1.0 + 0 * i, "gy": lambda i, j, k: 2.0 + 0 * i,
        "gz": lambda i, j, k: 3.0 + 0 * i,
        "Fx": lambda i, j, k: -kap * 1 + 0.5 * phi(i, j, k),
        "Fy": lambda i, j, k: -kap * 2 + 0.25 * phi(i, j, k),
        "Fz": lambda i, j, k: -kap * 3 - 0.125 * phi(i, j, k),
    })
    poison(prog, arrs, ["gx", "gy", "gz", "Fx", "Fy", "Fz", "D", "phin"])
    OracleProgram(prog).run(arrs)
    assert np.all(interior(prog, arrs["D"]) == 0.625)
    assert np.array_equal(interior(prog, arrs["phin"]),
                          interior(prog, arrs["phi"]) - 0.009765625)


# ------------------------------------------------------------- P13 C3 constant field
@pytest.mark.parametrize("plan_order", ["program"])
def test_p13_c3_constant_field_fp32_exact(plan_order):
    """All arrays 0.75, dyadic normalised 7/13-pt stencils: OUT = O1 + O2 = 3.0 exactly (fp32)."""
    prog = P.c3(n=7)
    arrs = filled(prog, {a["name"]: (lambda i, j, k: 0.75 + 0 * i) for a in prog["arrays"]})
    poison(prog, arrs, ["P", "Q", "P1", "P2", "Q1", "Q2", "O1", "O2", "OUT"])
    # ghosts of the temps keep 0.75 (filled above before poisoning interiors)
    OracleProgram(prog).run(arrs)
    out = interior(prog, arrs["OUT"])
    assert out.dtype == np.float32
    assert np.all(out == np.float32(3.0))


# ------------------------------------------------------------- order of summation (R4)
def test_r4_left_to_right_summation_order():
    """Terms 2^53, 1, -2^53 summed left to right give 0 in binary64 (2^53+1 rounds to 2^53);
    any other order gives 1.  Pins the fixed term order the GPU path must also use."""
    prog = {
        "name": "order", "dtype": "f64", "grid": {"nx": 3, "ny": 2, "nz": 2, "ghost": [1, 1, 1]},
        "arrays": [{"name": "X", "role": "in"}, {"name": "Y", "role": "out"}],
        "kernels": [P.kernel("K", P.stmt("Y", [{"c": 2.0 ** 53, "a": ["X", 0, 0, 0]},
                                               {"c": 1.0, "a": ["X", 1, 0, 0]},
                                               {"c": -(2.0 ** 53), "a": ["X", -1, 0, 0]}]))],
    }
    arrs = filled(prog, {"X": lambda i, j, k: 1.0 + 0 * i})
    OracleProgram(prog).run(arrs)
    assert np.all(interior(prog, arrs["Y"]) == 0.0)


def test_product_term_is_coef_times_a_times_b():
    """(c*a)*b with c = 3, a = x, b = y: pins that both factors and the coefficient are used."""
    prog = {
        "name": "prod", "dtype": "f64", "grid": {"nx": 4, "ny": 3, "nz": 2, "ghost": [1, 1, 1]},
        "arrays": [{"name": "X", "role": "in"}, {"name": "Z", "role": "in"},
                   {"name": "Y", "role": "out"}],
        "kernels": [P.kernel("K", P.stmt("Y", [{"c": 3.0, "a": ["X", 1, 0, 0], "b": ["Z", 0, -1, 0]},
                                               {"c": -1.0, "a": ["Z", 0, 0, 1]}]))],
    }
    arrs = filled(prog, {"X": lambda i, j, k: i + 0.0 * i, "Z": lambda i, j, k: j + 10.0 * k})
    OracleProgram(prog).run(arrs)
    kk, jj, ii = np.meshgrid(np.arange(2), np.arange(3), np.arange(4), indexing="ij")
    expect = 3.0 * (ii + 1) * ((jj - 1) + 10.0 * kk) - (jj + 10.0 * (kk + 1))
    assert np.array_equal(interior(prog, arrs["Y"]), expect)


# ------------------------------------------------------------- P5 independent evaluator
def random_box(rng, n):
    """Random loop bounds inside an interior of size n (possibly empty, possibly whole)."""
    box = []
    for d in range(3):
        lo = int(rng.integers(0, n[d] + 1))
        hi = int(rng.integers(lo, n[d] + 1))
        box += [lo, hi]
    return box


def random_program(rng, dtype="f64", boxes=False):
    nx, ny, nz = (int(v) for v in rng.integers(1, 8, size=3))
    h = [2, 2, 2]
    n_arr = int(rng.integers(3, 7))
    names = [f"a{i}" for i in range(n_arr)]
    roles = ["in"] + [str(rng.choice(["in", "temp", "out", "inout"])) for _ in range(n_arr - 1)]
    kernels = []
    for kk in range(int(rng.integers(1, 6))):
        stmts = []
        written = set()
        for _ in range(int(rng.integers(1, 4))):
            out = names[int(rng.integers(1, n_arr))]
            terms = []
            for _ in range(int(rng.integers(1, 6))):
                def rtap():
                    arr = names[int(rng.integers(0, n_arr))]
                    if arr in written or arr == out:
                        return [arr, 0, 0, 0]
                    return [arr] + [int(v) for v in rng.integers(-2, 3, size=3)]
                t = {"c": float(rng.uniform(-1, 1)), "a": rtap()}
                if rng.random() < 0.3:
                    t["b"] = rtap()
                terms.append(t)
            # R3: reads of an array written later in the same kernel must be at 0 too
            stmts.append({"out": out, "terms": terms})
            written.add(out)
        wr = {s["out"] for s in stmts}
        for s in stmts:
            for t in s["terms"]:
                for key in ("a", "b"):
                    if key in t and t[key][0] in wr:
                        t[key] = [t[key][0], 0, 0, 0]
        kernels.append({"name": f"K{kk}", "stmts": stmts})
        if boxes and rng.random() < 0.6:
            kernels[-1]["box"] = random_box(rng, (nx, ny, nz))
    return {"name": "rand", "dtype": dtype, "grid": {"nx": nx, "ny": ny, "nz": nz, "ghost": h},
            "arrays": [{"name": a, "role": r} for a, r in zip(names, roles)], "kernels": kernels}


@pytest.mark.parametrize("seed", range(40))
def test_p5_oracle_matches_slicing_evaluator_bitexact(seed):
    rng = np.random.default_rng(seed)
    prog = random_program(rng, dtype="f64" if seed % 3 else "f32")
    a1 = dense_arrays(prog, seed=seed)
    a2 = {k: v.copy() for k, v in a1.items()}
    OracleProgram(prog).run(a1)
    _numpy_eval.run(prog, a2)
    for name in a1:
        assert a1[name].tobytes() == a2[name].tobytes(), name


# ------------------------------------------------------------- window (box) evaluation
def test_box_window_centre_is_exact():
    """Evaluating a window wider than the accumulated reach reproduces the full-grid value
    at the window centre (used for sampled parity at full size)."""
    prog = P.c3(n=24)
    full = dense_arrays(prog, seed=5)
    OracleProgram(prog).run(full)
    from synth.fields import field
    # window of half-width R around (i0, j0, k0); C3's group reach is 1+1+2+1 = 5 per axis
    R, h = 6, 2
    i0, j0, k0 = 3, 20, 11
    lo = (i0 - R, j0 - R, k0 - R)
    n = (2 * R + 1,) * 3
    win = {}
    for aid, a in enumerate(prog["arrays"]):
        # window arrays: generated values at global coordinates of the window
        f = field(5, aid, (prog["grid"]["nx"], prog["grid"]["ny"], prog["grid"]["nz"]), (h, h, h), "f32")
        g0 = [l for l in lo]
        sl = f[max(0, g0[2]):, max(0, g0[1]):, max(0, g0[0]):]
        w = np.zeros((n[2] + 2 * h, n[1] + 2 * h, n[0] + 2 * h), dtype=np.float32)
        # fill from the full generated array (global coords -> padded index +h)
        for kk in range(n[2] + 2 * h):
            for jj in range(n[1] + 2 * h):
                gk, gj = lo[2] - h + kk, lo[1] - h + jj
                if not (-h <= gk < 24 + h and -h <= gj < 24 + h):
                    continue
                for ii in range(n[0] + 2 * h):
                    gi = lo[0] - h + ii
                    if -h <= gi < 24 + h:
                        w[kk, jj, ii] = f[gk + h, gj + h, gi + h]
        win[a["name"]] = w
    # global interior in window coordinates
    box = (0 - lo[0], 24 - lo[0], 0 - lo[1], 24 - lo[1], 0 - lo[2], 24 - lo[2])
    OracleProgram(prog).run(win, box=box, n=n)
    got = win["OUT"][h + R, h + R, h + R]
    want = full["OUT"][h + k0, h + j0, h + i0]
    assert got == want


# ------------------------------------------------------------- fp32 rounding bound
def test_fp32_program_within_bound_of_binary64_evaluation():
    prog = P.c3(n=12)
    a32 = dense_arrays(prog, seed=9)
    w = {k: v.copy() for k, v in a32.items()}
    OracleProgram(prog).run(a32)
    OracleProgram(prog).run(w, wide=True)
    ref = interior(prog, w["OUT"]).astype(np.float64)
    got = interior(prog, a32["OUT"]).astype(np.float64)
    assert np.max(np.abs(got - ref)) / np.max(np.abs(ref)) < 1e-5


# ------------------------------------------------------------- validation
def test_rejects_in_kernel_race_R3():
    prog = P.c1(n=4)
    bad = dict(prog)
    bad["kernels"] = [P.kernel("K", P.stmt("T", [{"c": 1.0, "a": ["A", 0, 0, 0]}]),
                               P.stmt("B", [{"c": 1.0, "a": ["T", 1, 0, 0]}]))]
    with pytest.raises(ValueError):
        OracleProgram(bad)


def test_rejects_tap_beyond_ghost():
    prog = P.c1(n=4)
    bad = dict(prog)
    bad["kernels"] = [P.kernel("K", P.stmt("T", [{"c": 1.0, "a": ["A", 2, 0, 0]}]))]
    with pytest.raises(ValueError):
        OracleProgram(bad)


def test_ghosts_never_written():
    prog = P.c2(n=5)
    arrs = dense_arrays(prog, seed=3)
    before = {k: v.copy() for k, v in arrs.items()}
    OracleProgram(prog).run(arrs)
    h = 1
    for name, v in arrs.items():
        m = np.ones(v.shape, bool)
        m[h:-h, h:-h, h:-h] = False
        assert np.array_equal(v[m], before[name][m]), name


@pytest.mark.parametrize("seed", range(30))
def test_p5_boxed_kernels_match_slicing_evaluator_bitexact(seed):
    """Kernels with loop bounds (reading R2'): the oracle writes exactly the box."""
    rng = np.random.default_rng(1000 + seed)
    prog = random_program(rng, dtype="f64" if seed % 3 else "f32", boxes=True)
    a1 = dense_arrays(prog, seed=seed)
    a2 = {k: v.copy() for k, v in a1.items()}
    OracleProgram(prog).run(a1)
    _numpy_eval.run(prog, a2)
    for name in a1:
        assert a1[name].tobytes() == a2[name].tobytes(), name


def _box_prog(box, terms, n=(6, 5, 4)):
    return {"name": "box", "dtype": "f64",
            "grid": {"nx": n[0], "ny": n[1], "nz": n[2], "ghost": [1, 1, 1]},
            "arrays": [{"name": "A", "role": "in"}, {"name": "O", "role": "out"}],
            "kernels": [{"name": "K", "box": box, "stmts": [{"out": "O", "terms": terms}]}]}


def test_box_writes_exactly_the_box():
    """O = 1*A over box [1,4)x[2,5)x[0,2) with A = 3 everywhere and O = -1: O is 3
    exactly on the 3x3x2 box and keeps -1 everywhere else (ghosts included)."""
    prog = _box_prog([1, 4, 2, 5, 0, 2], [{"c": 1.0, "a": ["A", 0, 0, 0]}])
    arrs = {"A": np.full((6, 7, 8), 3.0), "O": np.full((6, 7, 8), -1.0)}
    OracleProgram(prog).run(arrs)
    O = arrs["O"]
    inside = np.zeros_like(O, dtype=bool)
    inside[1:3, 1 + 2:1 + 5, 1 + 1:1 + 4] = True
    assert np.all(O[inside] == 3.0) and np.all(O[~inside] == -1.0)
    assert inside.sum() == 18


def test_box_boundary_plane_kernel_linear_field():
    """A boundary kernel on the bottom plane only (k = 0): centred
    difference in z of A = 2k + j gives 0.5*A[k+1] - 0.5*A[k-1] = 2 exactly there;
    the other planes keep O = 0."""
    n = (5, 4, 6)
    prog = _box_prog([0, n[0], 0, n[1], 0, 1],
                     [{"c": 0.5, "a": ["A", 0, 0, 1]}, {"c": -0.5, "a": ["A", 0, 0, -1]}], n)
    k, j, i = np.meshgrid(np.arange(-1, n[2] + 1), np.arange(-1, n[1] + 1), np.arange(-1, n[0] + 1),
                          indexing="ij")
    arrs = {"A": np.ascontiguousarray(2.0 * k + j), "O": np.zeros(k.shape)}
    OracleProgram(prog).run(arrs)
    O = arrs["O"][1:-1, 1:-1, 1:-1]
    assert np.all(O[0] == 2.0) and np.all(O[1:] == 0.0)


def test_box_window_origin_translation():
    """Evaluating a window of the grid with the window's global origin gives the
    same points as the whole grid (statement boxes move with the window)."""
    rng = np.random.default_rng(5)
    prog = _box_prog([2, 5, 1, 4, 1, 3], [{"c": 0.25, "a": ["A", 1, 0, 0]},
                                           {"c": 0.75, "a": ["A", 0, -1, 1]}])
    full = dense_arrays(prog, seed=3)
    ref = {k: v.copy() for k, v in full.items()}
    OracleProgram(prog).run(ref)
    # window: global interior x in [1,6), y in [0,5), z in [1,4) (with its ghosts)
    win = {k: np.ascontiguousarray(v[1:6, 0:7, 1:8]) for k, v in full.items()}
    OracleProgram(prog).run(win, n=(5, 5, 3), origin=(1, 0, 1))
    assert np.array_equal(win["O"][1:-1, 1:-1, 1:-1], ref["O"][2:5, 1:6, 2:7])


@pytest.mark.parametrize("cfg", ["C5", "C3"])
def test_window_evaluation_matches_full_grid(cfg):
    """The sampled full-size GPU checks evaluate the oracle on w^3 windows with generated
    ghosts; pinned here against the whole-grid oracle: exact inside the accumulated-reach
    margin (and up to the global boundary on boundary sides)."""
    import sys
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    from _harness import accumulated_reach, window_field
    prog = {"C5": lambda: P.c5(nx=40, ny=36, nz=30), "C3": lambda: P.c3(nx=40, ny=36, nz=30)}[cfg]()
    g = prog["grid"]
    N, h = (g["nx"], g["ny"], g["nz"]), tuple(g["ghost"])
    full = dense_arrays(prog, 4)
    OracleProgram(prog).run(full)
    m, w = accumulated_reach(prog), 24
    for origin in [(0, 0, 0), tuple((N[d] - w) // 2 for d in range(3)), tuple(N[d] - w for d in range(3))]:
        win = {a["name"]: window_field(4, aid, origin, (w, w, w), h, prog["dtype"])
               for aid, a in enumerate(prog["arrays"])}
        OracleProgram(prog).run(win, n=(w, w, w), origin=origin)
        lo = [origin[d] + (m[d] if origin[d] > 0 else 0) for d in range(3)]
        hi = [origin[d] + w - (m[d] if origin[d] + w < N[d] else 0) for d in range(3)]
        for nm in [a["name"] for a in prog["arrays"] if a["role"] in ("out", "inout")]:
            sl = lambda o: (slice(h[2] + lo[2] - o[2], h[2] + hi[2] - o[2]),  # noqa: E731
                            slice(h[1] + lo[1] - o[1], h[1] + hi[1] - o[1]),
                            slice(h[0] + lo[0] - o[0], h[0] + hi[0] - o[0]))
            assert np.array_equal(win[nm][sl(origin)], full[nm][sl((0, 0, 0))]), (cfg, origin, nm)


@pytest.mark.parametrize("cfg", ["C2", "C3", "C5"])
def test_openmp_build_identical(cfg):
    """The OpenMP build of the oracle (parallel CPU baseline) splits the
    planes of one statement across threads; results are bit-identical to the serial one."""
    prog = {"C2": lambda: P.c2(nx=24, ny=20, nz=18), "C3": lambda: P.c3(nx=24, ny=20, nz=18),
            "C5": lambda: P.c5(nx=24, ny=20, nz=18)}[cfg]()
    a = dense_arrays(prog, 6)
    b = {k: v.copy() for k, v in a.items()}
    OracleProgram(prog).run(a)
    OracleProgram(prog, parallel=True).run(b)
    for k in a:
        assert a[k].tobytes() == b[k].tobytes(), k


def test_wide_variant_pinned_to_independent_binary64_evaluator():
    """oracle_run_f32_in_f64 (binary64 arithmetic on binary32 storage, used as the fp32
    error-bound reference) equals the independent NumPy slicing evaluator run in binary64
    (double coefficients, fp32 arrays promoted, each statement's result rounded to fp32
    when stored) bit for bit, on random fp32 programs with products and loop bounds."""
    import _numpy_eval
    from _fuzz import random_lib_program
    for seed in range(10):
        rng = np.random.default_rng(700 + seed)
        prog = random_lib_program(rng, n=(7, 5, 4), dtype="f32", boxes=seed % 2 == 1)
        a = dense_arrays(prog, seed=seed)
        w = {k: v.copy() for k, v in a.items()}
        OracleProgram(prog).run(w, wide=True)
        ref = _numpy_eval.run(dict(prog, dtype="f64"), {k: v.copy() for k, v in a.items()})
        for name in w:
            assert w[name].dtype == np.float32
            assert w[name].tobytes() == ref[name].astype(np.float32).tobytes(), (seed, name)
