"""compute-sanitizer racecheck (shared-memory hazards inside each kernel: the TMA / mbarrier
rings, the epilogue staging) and synccheck (barrier misuse) over a small 2-stage bf16
pipeline run through the product library."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

HERE = os.path.dirname(os.path.abspath(__file__))
SAN = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"


@pytest.mark.parametrize("tool", ["racecheck", "synccheck"])
def test_sanitizer_two_stage_bf16(tool):
    if not os.path.exists(SAN):
        pytest.skip("compute-sanitizer not installed")
    p = subprocess.run([SAN, "--tool", tool, "--error-exitcode", "97", sys.executable,
                        os.path.join(HERE, "sanitizer_run.py")], capture_output=True, text=True, timeout=1200)
    out = p.stdout + p.stderr
    print(out[-3000:])
    if p.returncode != 0 and "is closed on this pool" in out:
        # the GPU pool's compute-sanitizer wrapper refuses to run (operator decision); the last
        # runs it allowed earlier in round 2 reported 0 hazards / 0 errors (profiles/SUMMARY_r02.md)
        pytest.skip("compute-sanitizer closed on this GPU pool")
    assert p.returncode == 0, out[-3000:]
    assert "ERROR SUMMARY: 0 errors" in out or "RACECHECK SUMMARY: 0 hazards" in out, out[-3000:]
