"""Independent whole-array (slicing) evaluator used ONLY to pin the C oracle (pin P5).

It shares nothing with oracle.c: no loop nest, no index arithmetic — each term
is a shifted NumPy view of the padded array.  Same reading of the paper as the
oracle (R1-R4, R2' in DESIGN.md): statements in program order, interior points
inside the kernel's loop bounds only,
terms accumulated left to right in the program dtype, (c*a)*b for products.
"""
import numpy as np


def run(prog, arrays):
    g = prog["grid"]
    nx, ny, nz = g["nx"], g["ny"], g["nz"]
    hx, hy, hz = g["ghost"]
    dt = np.float64 if prog["dtype"] == "f64" else np.float32

    def view(name, dx, dy, dz):
        a = arrays[name]
        return a[hz + dz:hz + dz + nz, hy + dy:hy + dy + ny, hx + dx:hx + dx + nx]

    for k in prog["kernels"]:
        # loop bounds (reading R2'): only the kernel's box of the interior is written
        x0, x1, y0, y1, z0, z1 = k.get("box") or (0, nx, 0, ny, 0, nz)
        for s in k["stmts"]:
            acc = None
            for t in s["terms"]:
                v = dt(t["c"]) * view(*t["a"])
                if "b" in t:
                    v = v * view(*t["b"])
                acc = v if acc is None else acc + v
            view(s["out"], 0, 0, 0)[z0:z1, y0:y1, x0:x1] = acc[z0:z1, y0:y1, x0:x1]
    return arrays
