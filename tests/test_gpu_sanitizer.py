"""compute-sanitizer memcheck over one small case of every kernel path
(Life TMA / register / persistent / local multi-slab, conv TMA / generic,
histogram).  racecheck and synccheck logs of the same script are in
profiles/r01_sanitizer_*.log."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.skipif(shutil.which("compute-sanitizer") is None, reason="compute-sanitizer not on PATH")
def test_memcheck_clean():
    r = subprocess.run(["compute-sanitizer", "--tool", "memcheck", "--error-exitcode", "9", sys.executable,
                        os.path.join(ROOT, "tools", "sanitize_cases.py")], capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    assert "ALL OK" in r.stdout and "ERROR SUMMARY: 0 errors" in r.stdout + r.stderr
