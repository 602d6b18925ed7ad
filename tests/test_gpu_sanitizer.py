"""compute-sanitizer memcheck over one small case of every kernel path
(Life TMA / register / persistent / resident / local multi-slab, conv TMA /
two-generation / generic, Window(3D), histogram).  racecheck and synccheck
logs of the same script are in profiles/r02_sanitizer_*.log.  Where the
pool has closed compute-sanitizer (it refuses to run and says so), the
memcheck test is skipped and the same cases still run without it: every
case is checked against the CPU oracle inside tools/sanitize_cases.py."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CASES = os.path.join(ROOT, "tools", "sanitize_cases.py")


@pytest.mark.skipif(shutil.which("compute-sanitizer") is None, reason="compute-sanitizer not on PATH")
def test_memcheck_clean():
    r = subprocess.run(["compute-sanitizer", "--tool", "memcheck", "--error-exitcode", "9", sys.executable, CASES],
                       capture_output=True, text=True, timeout=900)
    if "is closed on this pool" in r.stdout + r.stderr:
        pytest.skip("compute-sanitizer refused to run on this pool: " + (r.stdout + r.stderr).strip()[:200])
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    assert "ALL OK" in r.stdout and "ERROR SUMMARY: 0 errors" in r.stdout + r.stderr


def test_cases_without_sanitizer():
    r = subprocess.run([sys.executable, CASES], capture_output=True, text=True, timeout=900)
    assert r.returncode == 0 and "ALL OK" in r.stdout, r.stdout[-3000:] + r.stderr[-3000:]
