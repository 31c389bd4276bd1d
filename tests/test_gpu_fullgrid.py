"""Full-grid parity at the BASELINE sizes, in the launch configuration bench.py times.

P:L319 §6.1.2: "Output of the automated method was verified against the output of the
original code base for every single run."  Here every interior point of every OUT
array is compared with the oracle, for
  * C3 (BASELINE configs[2], 512^3 fp32): plans measured, fission_fused, fused, single
    and the (tuned) unfused baseline;
  * C5's per-GPU grid (BASELINE configs[4], 1024x1024x128 fp64): plans fused, single
    and unfused.
Perf build (FMA contraction on), tolerance R17 (1e-5 fp32, 1e-12 fp64).  The GPU side
NaN-poisons TEMP interiors, so a fused kernel that consumes a value it did not compute
fails.  The checker is the oracle's OpenMP build (the same C loop nest, pinned
bit-identical to the serial build by tests/test_oracle_pins.py), run once per workload
on the host; inputs come from synth/fields.py (torch on the CPU), never from the GPU.
"""
import os
import sys

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SEED = 4  # bench.fill_inputs' seed


def _host_inputs(prog):
    import torch
    from synth.fields import field_torch
    g = prog["grid"]
    n = (g["nx"], g["ny"], g["nz"])
    out = {}
    for aid, a in enumerate(prog["arrays"]):
        out[a["name"]] = field_torch(SEED, aid, n, tuple(g["ghost"]), prog["dtype"], "cpu").numpy()
    return out


_REF = {}


def _reference(workload):
    """OUT interiors of the oracle on the full grid (OpenMP build), cached per workload."""
    if workload not in _REF:
        sys.path.insert(0, ROOT)
        import bench
        from _harness import compared_arrays, interior
        from oracle import OracleProgram
        prog = bench.load_workload(workload)
        arrs = _host_inputs(prog)
        OracleProgram(prog, parallel=True).run(arrs)
        _REF.clear()  # one workload's arrays at a time (C5: 17.5 GB)
        _REF[workload] = {n: interior(prog, arrs[n]).copy() for n in compared_arrays(prog)}
        del arrs
    return _REF[workload]


def _gpu_outputs(workload, plan):
    import torch
    sys.path.insert(0, ROOT)
    import bench
    from _harness import compared_arrays, gpu_program
    prog = bench.load_workload(workload)
    unfused = plan == "unfused"
    p = gpu_program(prog, plan=bench.plan_of(prog, "fused" if unfused else plan))
    bench.apply_tuning(p, prog, "fused" if unfused else plan)
    dev = torch.device("cuda:0")
    p.allocate(dev, fill=0.0)
    bench.fill_inputs(p, prog, dev, 0, prog["grid"]["ghost"][2])
    for a in prog["arrays"]:
        if a["role"] == "temp":
            p.interior_view(p.tensors[a["name"]]).fill_(float("nan"))
    p.run_unfused() if unfused else p.run_fused()
    torch.cuda.synchronize()
    out = {n: p.interior_view(p.tensors[n]).cpu().numpy() for n in compared_arrays(prog)}
    del p
    torch.cuda.empty_cache()
    return prog, out


def _check(workload, plan):
    from _harness import rel_err, tolerance
    prog, got = _gpu_outputs(workload, plan)
    ref = _reference(workload)
    for n, r in ref.items():
        g = got[n]
        assert g.shape == r.shape
        assert np.isfinite(g).all(), f"{workload}/{plan} {n}: non-finite output"
        e = rel_err(g, r)
        assert e <= tolerance(prog["dtype"]), f"{workload}/{plan} {n}: rel err {e}"
        print(f"{workload}/{plan} {n}: {g.size} points, inf-norm rel err {e:.3e}")


# fission_fused / fused run in the region-vector (frame) form at their bench pins; the
# *_block plans keep the register-block form at its round-1 pins
@pytest.mark.parametrize("plan", ["measured", "fission_fused", "fused", "single", "unfused",
                                  "fission_fused_block"])
def test_c3_full_grid(cuda_device, plan):
    _check("C3", plan)


@pytest.mark.parametrize("plan", ["fused", "single", "unfused"])
def test_c5_full_grid_per_gpu(cuda_device, plan):
    _check("C5", plan)
