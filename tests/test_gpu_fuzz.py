"""GPU fuzz parity: random legal programs — random taps within the
ghost width, products, multi-output kernels, INOUT/TEMP reuse, optionally kernels
with loop bounds (reading R2') — under the unfused plan and up to four fusion plans the
library accepts (tests/_fuzz.legal_plans: the single group, the model's greedy plan,
random contiguous cuts; fission where a cut splits a kernel; plans that fuse a boxed
kernel first), in the parity build (fmad=0): every accepted plan must reproduce the
oracle bit-exactly (P6, R13), in the register-block and the region-vector (frame) form.  Each seed must actually run fused plans (at least two,
and for boxed programs at least one fusing a boxed kernel with another statement);
rejected candidates must carry a plan error code (tests/test_host.py checks the
acceptance counts on the CPU)."""
import pytest

from _fuzz import _fuses_boxed, fuzz_case
from _harness import assert_close, gpu_run, oracle_outputs

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("frame", [0, 1, 2], ids=["block", "frame", "frame2"])
@pytest.mark.parametrize("boxes", [False, True], ids=["full", "boxed"])
@pytest.mark.parametrize("seed", range(12))
def test_fuzz_parity_bitexact(cuda_device, seed, boxes, frame):
    prog, plans, rejected, _ = fuzz_case(seed, boxes)
    ref = oracle_outputs(prog, seed=seed, poison=False)
    got = gpu_run(prog, "unfused", seed, options={"fmad": 0}, poison=False)
    assert_close(prog, got, ref, exact=True)
    assert all(code in (4, 5, 6) for _, code in rejected), rejected
    assert len(plans) >= 2, f"only {len(plans)} fused plans accepted"
    if boxes and any(k.get("box") is not None for k in prog["kernels"]):
        assert _fuses_boxed(prog, plans[0]), "no accepted plan fuses a boxed kernel"
    for plan in plans:
        got = gpu_run(prog, "fused", seed, options={"fmad": 0, "frame": frame}, plan=plan, poison=False)
        assert_close(prog, got, ref, exact=True)
