"""The checking build (SR_BOUNDS_CHECK: every kernel traps on an out-of-range index of its
tally grid, traversal stack, scene records or prolog window) over every *_pdom / *_spec
kernel variant at small, ragged sizes (tools/sanitize_run.py).  It stands in for
compute-sanitizer memcheck where the GPU pool refuses that tool (tests/test_gpu_sanitizer.py);
the default build compiles the checks away (tests/test_simt_prediction.py ties its SASS to
the profiled kernels)."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _sass(lib):
    return subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout


def test_bounds_checked_build_runs_clean():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    sys.path.insert(0, ROOT)
    from paper_conf_cgo_damanijskymg20_b200 import build as B
    lib = B.build(defines=["SR_BOUNDS_CHECK"], lib=os.path.join(B.HERE, "libsr_bounds.so"))
    # the checks are really in the kernels (and only in the checking build)
    assert _sass(lib).count("BPT.TRAP") > 10
    env = dict(os.environ, SR_LIB=lib)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "sanitize_run.py")],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=1500)
    out = r.stdout + r.stderr
    assert r.returncode == 0, out[-4000:]
    assert "sanitize_run:" in out and "launches ok" in out, out[-2000:]
