"""compute-sanitizer over small JIT and interpreter runs (SURVEY §4
"Sanitizers"): no memory errors, no shared-memory races, no barrier misuse."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CS = "/usr/local/cuda/bin/compute-sanitizer"


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer(tool):
    if not os.path.exists(CS):
        pytest.skip("compute-sanitizer not installed")
    env = dict(os.environ, RTLSIM_JIT_CACHE="")   # compile under the tool, no cache
    r = subprocess.run([CS, "--tool", tool, "--error-exitcode", "97", sys.executable,
                        os.path.join(ROOT, "tools", "sanitize_run.py")],
                       capture_output=True, text=True, timeout=1500, env=env, cwd=ROOT)
    out = r.stdout + r.stderr
    if r.returncode == 86 and "closed on this pool" in out:
        # the GPU pool's compute-sanitizer wrapper refuses to run (runs under
        # it left GPUs needing a reset); parity tests and the JIT's own
        # bounds checks remain
        pytest.skip("compute-sanitizer is closed on this GPU pool")
    assert r.returncode == 0, out[-4000:]
    assert "sanitize_run ok" in out
    assert "ERROR SUMMARY: 0 errors" in out or "RACECHECK SUMMARY: 0 hazards" in out, out[-2000:]
