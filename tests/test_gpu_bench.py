"""bench.py end to end on one GPU: the N = 1 line and the N = 2 code path
(torchrun, 2 ranks time-sliced on cuda:0 through the test hooks
DDT_BENCH_BACKEND=gloo / DDT_BENCH_SHARE_GPU=1 -- timings meaningless, the
point is that every arm of the multi-rank path runs and rank 0 prints one
contract line)."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _line(out: str) -> dict:
    lines = [ln for ln in out.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, out[-3000:]
    return json.loads(lines[0])


def _check(d, n):
    assert d["n_gpus"] == n and d["unit"] == "us/iter" and d["higher_is_better"] is False
    assert d["value"] > 0 and d["gpu_launches"] >= d["steps"]
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert "failed" not in d["e2e"]["flow"], d["e2e"]["flow"]
    assert d["roofline"]["bound"] == "hbm" and 0 < d["roofline"]["frac"]


def test_bench_n1():
    r = subprocess.run([sys.executable, "bench.py", "--steps", "30", "--warmup", "3", "--no-extras"], cwd=ROOT,
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    d = _line(r.stdout)
    _check(d, 1)
    # the reference arm (CPU oracle) prints the same metric / unit / direction / config
    r2 = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--steps", "3", "--warmup", "1"],
                        cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r2.returncode == 0, r2.stderr[-3000:]
    ref = _line(r2.stdout)
    assert ref["impl"] == "reference"
    for k in ("metric", "unit", "higher_is_better", "data"):
        assert ref[k] == d[k], k
    assert ref["config"] == dict(d["config"], distinct_replicas_timed=min(3, d["config"]["replicas"])), \
        (ref["config"], d["config"])


@pytest.mark.parametrize("mode,port", [("p2p", 29533), ("p2p_direct", 29534)])
def test_bench_n2_shared_gpu(mode, port):
    """N = 2: the K steps of the flagged P2P exchange are one captured CUDA graph
    (device-resident epoch), as at N = 1."""
    env = dict(os.environ, DDT_BENCH_BACKEND="gloo", DDT_BENCH_SHARE_GPU="1", DDT_BENCH_REPLICAS="4")
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                        "--master-addr", "127.0.0.1", "--master-port", str(port), "bench.py", "--gpus", "2",
                        "--steps", "10", "--warmup", "3", "--no-extras", "--mode", mode],
                       cwd=ROOT, capture_output=True, text=True, timeout=900, env=env)
    assert r.returncode == 0, (r.stdout[-2000:], r.stderr[-3000:])
    d = _line(r.stdout)
    _check(d, 2)
    assert d["run"]["mode"] == mode
    assert d["run"]["launch"].startswith("K-step CUDA graph"), d["run"]["launch"]
