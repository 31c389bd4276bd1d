"""Dynamic race / sync / memory checking of the generated kernels (SURVEY.md §4 T3, §5:
the paper's complex fusion needs barriers "to prevent data races", §5.5.3).

compute-sanitizer runs small C1, C2, chain3, C3 (fission+fusion) and C4 programs,
unfused and fused, through the C ABI (tests/_sanitize_case.py, each result also
bit-exact with the oracle):
  * racecheck: shared-memory hazards between the compute warps (halo stages, plane
    rings, named barriers) and with the TMA producer warp's ring refills;
  * synccheck: illegal barrier use (named barriers over the compute warps only,
    mbarrier phases);
  * memcheck: out-of-bounds / misaligned global and shared accesses (ghost loads,
    128-bit stores, TMA boxes).
Each must report 0 errors."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _sanitizer():
    for c in ("/usr/local/cuda/bin/compute-sanitizer", "compute-sanitizer"):
        if os.path.exists(c) or c == "compute-sanitizer":
            return c


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer(cuda_device, tool):
    cmd = [_sanitizer(), "--tool", tool, "--error-exitcode", "99", "--print-limit", "20"]
    if tool == "racecheck":
        cmd += ["--racecheck-report", "all"]
    cmd += [sys.executable, os.path.join(ROOT, "tests", "_sanitize_case.py")]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=1500, cwd=ROOT)
    out = r.stdout + r.stderr
    print(out[-3000:])
    if r.returncode == 86 and "closed on this pool" in out:
        # the GPU pool's operators closed compute-sanitizer (it wraps the binary and exits 86
        # without running anything); the last runs are kept in profiles/r2_sanitizer.log
        pytest.skip("compute-sanitizer closed on this GPU pool: " + out.strip().splitlines()[-1][:200])
    assert r.returncode == 0, out[-6000:]
    assert ("ERROR SUMMARY: 0 errors" in out or "(0 errors, 0 warnings)" in out), out[-6000:]
    for name in ("C1", "C2", "chain3", "C3", "C4"):
        assert f"{name}: ok" in out
