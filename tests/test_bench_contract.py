"""The bench.py JSON contract, checked on CPU through the reference arm (the oracle) on the
tiny workload, plus the bench's own algorithmic-bytes arithmetic."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--workload", "tiny",
                        "--steps", "2", "--warmup", "1"], capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["steps"] == 2
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["config"]["workload"] == "tiny"


def test_algorithmic_bytes():
    sys.path.insert(0, ROOT)
    import bench
    from xs_workloads import WORKLOADS
    # E[n_nuc] x 96 B (nuclide), + 4 B (unionized), + 8 ceil(log2(W+1)) B (hash) per pair
    assert abs(bench.algorithmic_bytes_per_lookup(WORKLOADS["small"]) - 15.490 * 96) < 1e-9
    assert abs(bench.algorithmic_bytes_per_lookup(WORKLOADS["large"]) - 55.383 * 96) < 1e-9
    assert abs(bench.algorithmic_bytes_per_lookup(WORKLOADS["large-U"]) - 55.383 * 100) < 1e-9
    assert abs(bench.algorithmic_bytes_per_lookup(WORKLOADS["XL"]) - 55.383 * (96 + 8 * 5)) < 1e-9
