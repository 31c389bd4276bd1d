"""ctypes front end of the C oracle (oracle.c) — TEST INFRASTRUCTURE ONLY.

The loader below turns the program dict (synth/programs.py schema) into the
oracle's own C structs.  It shares no code with the product binding.

Validation here follows the same readings the product enforces, written
independently:
  * R3: inside one kernel, an array written by the kernel may only
    be read at offset (0,0,0) — otherwise the original CUDA kernel would race
    and the program has no defined result.
  * every tap lies within the ghost width (R1: reads outside the interior hit
    ghost storage, never beyond it).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_LIB_OMP_PATH = os.path.join(_HERE, "liboracle_omp.so")  # same source, -fopenmp
_lib = None
_lib_omp = None


class OrTap(ctypes.Structure):
    _fields_ = [("arr", ctypes.c_int), ("dx", ctypes.c_int), ("dy", ctypes.c_int),
                ("dz", ctypes.c_int)]


class OrTerm(ctypes.Structure):
    _fields_ = [("coef", ctypes.c_double), ("a", OrTap), ("has_b", ctypes.c_int), ("b", OrTap)]


class OrStmt(ctypes.Structure):
    _fields_ = [("out", ctypes.c_int), ("n_terms", ctypes.c_int),
                ("terms", ctypes.POINTER(OrTerm)), ("has_box", ctypes.c_int),
                ("box", ctypes.c_long * 6)]


class OrGrid(ctypes.Structure):
    _fields_ = [("nx", ctypes.c_long), ("ny", ctypes.c_long), ("nz", ctypes.c_long),
                ("hx", ctypes.c_int), ("hy", ctypes.c_int), ("hz", ctypes.c_int)]


def build_oracle(force: bool = False) -> str:
    """Compile oracle.c with the flags reading R4 requires (no FMA contraction); also
    the OpenMP build of the same source (parallel CPU baseline)."""
    src = os.path.join(_HERE, "oracle.c")
    for path, extra in ((_LIB_PATH, []), (_LIB_OMP_PATH, ["-fopenmp"])):
        if force or not os.path.exists(path) or \
                os.path.getmtime(path) < max(os.path.getmtime(src),
                                             os.path.getmtime(os.path.join(_HERE, "oracle.h"))):
            subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c11",
                                   "-fPIC", "-shared"] + extra + ["-o", path, src])
    return _LIB_PATH


def load_library(parallel: bool = False):
    global _lib, _lib_omp
    if (_lib_omp if parallel else _lib) is None:
        build_oracle()
        lib = ctypes.CDLL(_LIB_OMP_PATH if parallel else _LIB_PATH)
        for name, real in (("f64", ctypes.c_double), ("f32", ctypes.c_float)):
            f = getattr(lib, f"oracle_run_{name}")
            f.argtypes = [ctypes.POINTER(OrGrid), ctypes.c_int, ctypes.POINTER(ctypes.POINTER(real)),
                          ctypes.c_int, ctypes.POINTER(OrStmt)]
            f.restype = ctypes.c_int
            f = getattr(lib, f"oracle_run_box_{name}")
            f.argtypes = [ctypes.POINTER(OrGrid), ctypes.POINTER(ctypes.c_long), ctypes.c_int,
                          ctypes.POINTER(ctypes.POINTER(real)), ctypes.c_int,
                          ctypes.POINTER(OrStmt)]
            f.restype = ctypes.c_int
        lib.oracle_run_f32_in_f64.argtypes = [
            ctypes.POINTER(OrGrid), ctypes.c_int, ctypes.POINTER(ctypes.POINTER(ctypes.c_float)),
            ctypes.c_int, ctypes.POINTER(OrStmt)]
        lib.oracle_run_f32_in_f64.restype = ctypes.c_int
        if parallel:
            _lib_omp = lib
        else:
            _lib = lib
    return _lib_omp if parallel else _lib


class OracleProgram:
    """The original program, flattened to statements in program order."""

    def __init__(self, prog: dict, parallel: bool = False):
        self.parallel = parallel  # OpenMP build over z (identical results, reading R3)
        self.prog = prog
        self.dtype = prog["dtype"]
        g = prog["grid"]
        self.n = (int(g["nx"]), int(g["ny"]), int(g["nz"]))
        self.h = tuple(int(v) for v in g["ghost"])
        self.names = [a["name"] for a in prog["arrays"]]
        self.index = {a: i for i, a in enumerate(self.names)}
        self.roles = {a["name"]: a["role"] for a in prog["arrays"]}
        self._validate()
        stmts = [s for k in prog["kernels"] for s in k["stmts"]]
        # loop bounds (reading R2'): the kernel's box, in global interior coordinates
        self.boxes = [k.get("box") for k in prog["kernels"] for _ in k["stmts"]]
        self._keep = []
        self.c_stmts = (OrStmt * len(stmts))()
        for si, s in enumerate(stmts):
            terms = (OrTerm * len(s["terms"]))()
            for ti, t in enumerate(s["terms"]):
                terms[ti].coef = float(t["c"])
                terms[ti].a = self._tap(t["a"])
                if "b" in t:
                    terms[ti].has_b = 1
                    terms[ti].b = self._tap(t["b"])
            self._keep.append(terms)
            self.c_stmts[si].out = self.index[s["out"]]
            self.c_stmts[si].n_terms = len(s["terms"])
            self.c_stmts[si].terms = terms
        self.n_stmts = len(stmts)
        self._set_origin((0, 0, 0))

    def _set_origin(self, origin):
        """Statement boxes in the coordinates of a window whose interior point
        (0,0,0) is the global point `origin`."""
        for si, b in enumerate(self.boxes):
            self.c_stmts[si].has_box = int(b is not None)
            if b is not None:
                for d in range(6):
                    self.c_stmts[si].box[d] = int(b[d]) - int(origin[d // 2])

    def _tap(self, t):
        return OrTap(self.index[t[0]], int(t[1]), int(t[2]), int(t[3]))

    def _validate(self):
        hx, hy, hz = self.h
        for k in self.prog["kernels"]:
            written = {s["out"] for s in k["stmts"]}
            for s in k["stmts"]:
                if s["out"] not in self.index:
                    raise ValueError(f"unknown array {s['out']}")
                for t in s["terms"]:
                    for key in ("a", "b"):
                        if key not in t:
                            continue
                        arr, dx, dy, dz = t[key]
                        if arr not in self.index:
                            raise ValueError(f"unknown array {arr}")
                        if abs(dx) > hx or abs(dy) > hy or abs(dz) > hz:
                            raise ValueError(f"tap {t[key]} beyond ghost width {self.h}")
                        if arr in written and (dx, dy, dz) != (0, 0, 0):
                            raise ValueError(f"kernel {k['name']}: {arr} written and read at "
                                             f"offset {(dx, dy, dz)} (reading R3)")

    def _grid(self, n=None, h=None):
        n = n or self.n
        h = h or self.h
        return OrGrid(n[0], n[1], n[2], h[0], h[1], h[2])

    def _ptrs(self, arrays: dict, real):
        ptrs = (ctypes.POINTER(real) * len(self.names))()
        want = np.float64 if real is ctypes.c_double else np.float32
        for i, name in enumerate(self.names):
            a = arrays[name]
            if a.dtype != want or not a.flags["C_CONTIGUOUS"]:
                raise TypeError(f"{name}: need C-contiguous {want}")
            ptrs[i] = a.ctypes.data_as(ctypes.POINTER(real))
        return ptrs

    def run(self, arrays: dict, box=None, wide=False, n=None, origin=(0, 0, 0)):
        """Evaluate in place on dense padded arrays {name: ndarray}.

        box: optional (i0,i1,j0,j1,k0,k1) restricting the evaluated points;
        wide: fp32 programs only — evaluate in binary64 (error bound check);
        n: interior size of the arrays if they are a window, not the program grid;
        origin: global coordinates of the window's interior point (0,0,0).
        """
        lib = load_library(self.parallel)
        self._set_origin(origin)
        grid = self._grid(n)
        real = ctypes.c_double if self.dtype == "f64" else ctypes.c_float
        ptrs = self._ptrs(arrays, real)
        if wide:
            assert self.dtype == "f32"
            rc = lib.oracle_run_f32_in_f64(ctypes.byref(grid), len(self.names), ptrs,
                                           self.n_stmts, self.c_stmts)
        elif box is None:
            f = lib.oracle_run_f64 if self.dtype == "f64" else lib.oracle_run_f32
            rc = f(ctypes.byref(grid), len(self.names), ptrs, self.n_stmts, self.c_stmts)
        else:
            b = (ctypes.c_long * 6)(*[int(v) for v in box])
            f = lib.oracle_run_box_f64 if self.dtype == "f64" else lib.oracle_run_box_f32
            rc = f(ctypes.byref(grid), b, len(self.names), ptrs, self.n_stmts, self.c_stmts)
        if rc != 0:
            raise RuntimeError("oracle rejected the program")
        return arrays


def dense_arrays(prog: dict, seed: int, poison_temp: bool = False, z_offset: int = 0,
                 n=None) -> dict:
    """Seeded dense padded arrays for every program array (synth/fields.py generator).

    Array ids are the positions in prog["arrays"].  poison_temp fills TEMP
    interiors with NaN (their ghosts keep generated values)."""
    from synth.fields import field
    g = prog["grid"]
    n = n or (g["nx"], g["ny"], g["nz"])
    h = tuple(g["ghost"])
    out = {}
    for aid, a in enumerate(prog["arrays"]):
        arr = field(seed, aid, n, h, prog["dtype"], z_offset=z_offset)
        if poison_temp and a["role"] == "temp":
            arr[h[2]:h[2] + n[2], h[1]:h[1] + n[1], h[0]:h[0] + n[0]] = np.nan
        out[a["name"]] = np.ascontiguousarray(arr)
    return out
