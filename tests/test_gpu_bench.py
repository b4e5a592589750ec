"""bench.py keeps the driver contract (one JSON line, required keys) at N=1
and on the N>1 code path (two ranks sharing the one GPU over gloo; the driver's
SCALE run uses NCCL, one GPU per rank)."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
REQUIRED = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
            "higher_is_better", "scaling", "vs_baseline", "dtype", "data", "config", "clocks",
            "e2e", "gpu_launches", "roofline"}


def _last_json(out):
    lines = [l for l in out.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out[-2000:]
    return json.loads(lines[0])


def test_bench_single_gpu_contract():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    r = subprocess.run([sys.executable, "bench.py", "--steps", "3", "--warmup", "3",
                        "--photons-per-gpu", "2000000", "--no-configs", "--no-cpu"],
                       cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    d = _last_json(r.stdout)
    assert REQUIRED <= set(d)
    assert d["n_gpus"] == 1 and d["value"] > 0 and d["speedup_vs_pdom"] > 1.0
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert d["gpu_launches"] == 3
    assert d["collective"] is None   # no collective at N = 1


def _two_rank(extra, port):
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
                        "--nproc-per-node", "2", "--master-addr", "127.0.0.1", "--master-port",
                        str(port), "bench.py", "--gpus", "2", "--steps", "3", "--warmup", "3",
                        "--dist-backend", "gloo", *extra],
                       cwd=ROOT, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-2000:]
    return _last_json(r.stdout)


def test_bench_two_rank_strong_gloo():
    """configs[4] as specified: a fixed total sharded over the ranks (strong), the
    whole job on one GPU alone gives t_1 and the bit-exact reference tallies."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    d = _two_rank(["--total-photons", "1024000", "--no-configs"], 29541)
    assert d["n_gpus"] == 2 and d["scaling"] == "strong"
    assert d["config"]["total_photons"] == 1024000
    assert d["config"]["photons_per_gpu"] == 512000
    assert "cpu_baseline" not in d and "configs" not in d   # rank 0 at N=1 only
    c = d["collective"]   # the tally all-reduce timed alone
    assert c["ms"] > 0 and c["bytes"] > 0 and c["share_of_step"] > 0
    assert d["tallies_equal_single_gpu_run"] is True   # sharded + all-reduced == one launch
    s = d["scaling_detail"]
    assert s["kind"] == "strong" and s["t1_ms"] > 0
    assert abs(s["efficiency"] - s["t1_ms"] / (2 * d["ms_per_step"])) < 1e-9
    assert s["weak"]["photons_per_gpu"] == 10**7 and s["weak"]["value"] > 0


def test_bench_two_rank_weak_gloo():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    d = _two_rank(["--scaling", "weak", "--photons-per-gpu", "512000"], 29542)
    assert d["n_gpus"] == 2 and d["scaling"] == "weak"
    assert d["config"]["photons_per_gpu"] == 512000   # a multiple of photons_per_lane
    assert d["config"]["total_photons"] == 1024000
    assert d["tallies_equal_single_gpu_run"] is True


def test_bench_reference_arm():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--steps", "2",
                        "--warmup", "1"], cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    d = _last_json(r.stdout)
    assert d["impl"] == "reference" and d["cpu_baseline"]["kind"] == "oracle"
    assert d["e2e"]["h2d_bytes_per_step"] == 0
