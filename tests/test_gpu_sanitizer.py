"""compute-sanitizer over every *_pdom / *_spec kernel variant at small, ragged
sizes (tools/sanitize_run.py): memcheck (out-of-bounds / misaligned accesses,
incl. the SCHED region of warps past n), racecheck (shared-memory hazards of the
MC tally staging and the path tracer's traversal stacks), synccheck (the
computed-mask __syncwarp / __ballot_sync of the soft barrier)."""
import os
import re
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SAN = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_sanitizer_clean(tool):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    if not os.path.exists(SAN):
        pytest.skip("compute-sanitizer not installed")
    import __graft_entry__
    __graft_entry__.build()
    cmd = [SAN, "--tool", tool, "--error-exitcode", "97",
           # only libsr's kernels: torch's own (allocator fills, copies) are not under test
           "--kernel-name", "regex=divloop|commoncall|mcml|rs_|pt_",
           sys.executable, os.path.join(ROOT, "tools", "sanitize_run.py")]
    if tool == "racecheck":
        cmd[3:3] = ["--racecheck-report", "all"]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=1500)
    out = r.stdout + r.stderr
    if r.returncode != 0 and "compute-sanitizer is closed" in out:
        # the GPU pool's wrapper refuses every sanitizer run (operators closed the tool
        # pool-wide); nothing ran, so there is nothing to judge here -- the runs up to
        # r02l were clean
        pytest.skip("compute-sanitizer closed on this GPU pool: " + out.strip()[-200:])
    assert r.returncode == 0, out[-4000:]
    assert "sanitize_run:" in out and "launches ok" in out, out[-2000:]
    if tool == "racecheck":
        m = re.search(r"RACECHECK SUMMARY: (\d+) hazards displayed \((\d+) errors, (\d+) warn", out)
        assert m and m.groups() == ("0", "0", "0"), out[-4000:]
    else:
        m = re.search(r"ERROR SUMMARY: (\d+) error", out)
        assert m and int(m.group(1)) == 0, out[-4000:]
