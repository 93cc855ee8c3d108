"""compute-sanitizer over every kernel family: memcheck on all of
them (out-of-bounds / misaligned accesses, API errors), racecheck and synccheck on the
deterministic wavefront kernels, which must be race-free (Hogwild races on P/Q by design and is
excluded).  The workload is tools/sanitize_case.py: tiny seeded sets, 2 epochs, RMSE and
factor read-back per case."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SAN = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"


def _run(tool, which, timeout=900):
    if not os.path.exists(SAN):
        pytest.skip("compute-sanitizer not installed")
    cmd = [SAN, "--tool", tool, "--error-exitcode", "9", "--print-limit", "20"]
    if tool == "memcheck":
        cmd += ["--leak-check", "no"]
    cmd += [sys.executable, os.path.join(ROOT, "tools", "sanitize_case.py"), which]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=timeout, cwd=ROOT)
    out = r.stdout + r.stderr
    if "closed on this pool" in out:
        # the GPU pool's compute-sanitizer wrapper refuses to run (operator policy); the clean
        # runs of this suite are recorded in DESIGN.md section 6 (commit 3891f99)
        pytest.skip("compute-sanitizer closed on this GPU pool: " + out.strip()[:200])
    assert r.returncode == 0, out[-4000:]
    assert ("ERROR SUMMARY: 0 errors" in out                      # memcheck, synccheck
            or "0 hazards displayed (0 errors, 0 warnings)" in out), out[-4000:]   # racecheck
    return out


def test_memcheck_all_kernels():
    out = _run("memcheck", "all")
    assert out.count("ok {") == 18


@pytest.mark.parametrize("tool", ["racecheck", "synccheck"])
def test_deterministic_kernels_race_and_sync_clean(tool):
    out = _run(tool, "det")
    assert out.count("ok {") == 8


def test_tma_rating_ring_race_clean():
    """The TMA rating stream's shared-memory ring (bulk copies, mbarriers, generic reads) under
    racecheck, at 1 worker (no by-design races on P/Q)."""
    out = _run("racecheck", "smem")
    assert out.count("ok {") == 2
