"""compute-sanitizer over the whole kernel set (SURVEY 4 "GPU parity", 5 "Race detection"):
memcheck (out-of-bounds / misaligned accesses), racecheck (shared-memory hazards) and synccheck
(illegal barriers / warp syncs) on small graphs through every path (scripts/sanitize_target.py:
graph build, root modes, warp / thread / register tiers, forced splits and donation, streaming,
GMBE-WARP / GMBE-BLOCK), each result also checked against the oracle.  Logs go to
$GMBE_SANITIZER_LOG_DIR when set (profiles/r02_sanitizer_*.log)."""
import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _sanitizer():
    # The GPU pool this build is tested on closed compute-sanitizer after runs under it left GPUs
    # needing a reset; the round-2 logs in profiles/ were taken before that.  Opt-in only.
    if os.environ.get("GMBE_SANITIZER") != "1":
        pytest.skip("compute-sanitizer runs are opt-in (GMBE_SANITIZER=1); logs: profiles/r02_sanitizer_*.log")
    for c in (shutil.which("compute-sanitizer"), "/usr/local/cuda/bin/compute-sanitizer"):
        if c and os.path.exists(c):
            return c
    pytest.skip("compute-sanitizer not found")


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_compute_sanitizer(tool):
    cmd = [_sanitizer(), "--tool", tool, "--error-exitcode", "99", "--print-limit", "50"]
    if tool == "racecheck":
        cmd += ["--racecheck-report", "all"]
    cmd += [sys.executable, os.path.join(ROOT, "scripts", "sanitize_target.py")]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=3000, cwd=ROOT)
    log = r.stdout + r.stderr
    d = os.environ.get("GMBE_SANITIZER_LOG_DIR")
    if d:
        os.makedirs(d, exist_ok=True)
        with open(os.path.join(d, "r02_sanitizer_%s.log" % tool), "w") as f:
            f.write(" ".join(cmd) + "\n" + log)
    if "is closed on this pool" in log:
        pytest.skip(log.strip().splitlines()[0])
    assert "SANITIZE TARGET PASSED" in log, log[-4000:]
    assert r.returncode == 0, log[-4000:]
    # memcheck / synccheck end with "ERROR SUMMARY", racecheck with its own hazard summary
    assert ("ERROR SUMMARY: 0 errors" in log or
            "RACECHECK SUMMARY: 0 hazards displayed (0 errors, 0 warnings)" in log), log[-4000:]
