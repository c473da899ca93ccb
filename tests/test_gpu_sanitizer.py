"""compute-sanitizer over a tiny end-to-end run of every path (tools/sanitize_run.py, SURVEY §5
"race detection / failure detection"): memcheck (out-of-bounds and misaligned device accesses,
also the arena bounds), racecheck (shared-memory hazards: the look-back scan, the partition
passes, the mbarrier / TMEM pipelines' staging buffers), synccheck (barrier misuse) and initcheck
(reads of uninitialised device memory; on the paths without TMA stores — initcheck does not see
global writes made by the tensor-memory-access unit, so every read of a TMA-stored activation
would be reported).  Each must report 0 errors."""
import os
import shutil
import subprocess
import sys

import pytest
import torch

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SAN = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck", "initcheck"])
def test_sanitizer_clean(tool):
    assert torch.cuda.is_available()
    cmd = [SAN, "--tool", tool, "--error-exitcode", "99", "--target-processes", "all"]
    if tool == "memcheck":
        cmd += ["--leak-check", "no"]
    which = "mean_ffma,pool,lstm,gat,clustering" if tool == "initcheck" else "all"
    cmd += [sys.executable, os.path.join(ROOT, "tools", "sanitize_run.py"), which]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=1500, cwd=ROOT)
    out = r.stdout + r.stderr
    if "ERROR SUMMARY" not in out and "RACECHECK SUMMARY" not in out and "closed" in out:
        # the pool's compute-sanitizer wrapper refused to run (it is disabled on these boxes)
        pytest.skip("compute-sanitizer unavailable here: " + out.strip().splitlines()[-1][:200])
    clean = "ERROR SUMMARY: 0 errors" in out or "RACECHECK SUMMARY: 0 hazards displayed (0 errors, 0 warnings)" in out
    assert r.returncode == 0 and clean, out[-4000:]
