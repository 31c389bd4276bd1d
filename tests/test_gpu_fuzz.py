"""GPU fuzz parity: random legal programs — random taps within the
ghost width, products, multi-output kernels, INOUT/TEMP reuse, optionally kernels
with loop bounds (reading R2') — under the unfused plan, the single-group plan and
random contiguous cuts (fission where a cut splits a kernel), in the parity build
(fmad=0): every plan the library accepts must reproduce the oracle bit-exactly
(P6, R13).  Plans it rejects must be rejected with a plan error, never computed."""
import numpy as np
import pytest

from _fuzz import random_lib_program, random_plans
from _harness import assert_close, gpu_run, oracle_outputs
from paper_conf_hpdc_wahibm15_b200 import StencilError

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("boxes", [False, True], ids=["full", "boxed"])
@pytest.mark.parametrize("seed", range(12))
def test_fuzz_parity_bitexact(cuda_device, seed, boxes):
    rng = np.random.default_rng(100 * seed + boxes)
    prog = random_lib_program(rng, dtype="f32" if seed % 4 == 3 else "f64", boxes=boxes)
    ref = oracle_outputs(prog, seed=seed, poison=False)
    got = gpu_run(prog, "unfused", seed, options={"fmad": 0}, poison=False)
    assert_close(prog, got, ref, exact=True)
    for plan in random_plans(rng, prog, count=3):
        try:
            got = gpu_run(prog, "fused", seed, options={"fmad": 0}, plan=plan, poison=False)
        except StencilError as e:
            assert e.code in (4, 5, 6), e
            continue
        assert_close(prog, got, ref, exact=True)
