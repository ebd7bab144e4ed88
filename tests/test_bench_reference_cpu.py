"""bench.py's reference arm (this tier: the CPU oracle) runs without a GPU and
prints the contract line: one JSON line with impl = "reference", the headline
metric / unit / direction, the workload config, cpu_baseline and e2e with zero
copies (test infrastructure: runs oracle/ through bench.py)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_line():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--steps", "3", "--warmup", "3"],
                       cwd=ROOT, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["unit"] == "us/iter" and d["higher_is_better"] is False
    assert d["metric"].startswith("bulk halo-exchange latency") and d["value"] > 0 and d["n_gpus"] == 1
    assert d["config"]["workload"].startswith("configs[1]") and d["config"]["distinct_replicas_timed"] == 3
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"] == {"value": d["value"], "unit": "us/iter", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}
