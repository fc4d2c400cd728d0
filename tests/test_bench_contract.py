"""The bench.py JSON contract, checked on CPU through the reference arm (the oracle) on the
tiny workload, plus the bench's own arithmetic: rank ranges, golden-hash
lookup, the roofline model and the random-gather bytes."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def _reference(*args):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", *args],
                       capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) <= 1
    return json.loads(lines[0]) if lines else None


def test_reference_arm_json_line():
    d = _reference("--workload", "tiny", "--steps", "2", "--warmup", "1")
    for k in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["steps"] == 2
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["config"]["workload"] == "tiny"
    import bench
    a = bench.parse(["--workload", "tiny"])
    assert d["config"] == bench.config_of(a, bench.WORKLOADS["tiny"], 1)  # the same config as our arm


def test_reference_arm_other_ranks_silent(monkeypatch):
    """under torchrun only rank 0 runs the oracle and prints; the others exit 0 at once"""
    env = dict(os.environ, RANK="1", WORLD_SIZE="2")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--workload", "tiny",
                        "--gpus", "2"], capture_output=True, text=True, timeout=120, cwd=ROOT, env=env)
    assert r.returncode == 0 and not r.stdout.strip()


def test_default_workload_and_scaling():
    import bench
    a = bench.parse([])
    assert a.workload == "large-U" and a.gpus == 1
    W = bench.WORKLOADS
    assert bench.scaling_of(a, W["large-U"]) == "strong" and bench.scaling_of(a, W["XL"]) == "weak"
    # XL at N = 8 is BASELINE.json configs[4]: 1B lookups
    assert bench.job_lookups(W["XL"], "weak", 0, 8) == 1_000_000_000
    assert bench.job_lookups(W["large-U"], "strong", 0, 8) == 100_000_000


@pytest.mark.parametrize("name", ["tiny", "small", "large", "large-U", "XL"])
@pytest.mark.parametrize("world", [1, 2, 4, 8])
def test_rank_ranges_hit_golden_boundaries(name, world):
    """every rank's range at N in {1, 2, 4, 8} is a union of golden eighths, so bench.py can
    check every rank's hash against the oracle at any of these N"""
    import bench
    w = bench.WORKLOADS[name]
    sc = w.scaling
    gd = json.load(open(bench.GOLDEN)).get(name)
    if gd is None:
        pytest.skip("golden hashes not written yet")
    parts = [bench.rank_range(w, sc, 0, r, world) for r in range(world)]
    if sc == "weak" and world * w.lookups > gd["total"]:
        pytest.skip("weak ranges beyond the golden total")
    assert sum(c for _, c in parts) == bench.job_lookups(w, sc, 0, world)
    for first, count in parts:
        exp = bench.golden_expect(name, first, count)
        assert exp is not None
    assert sum(bench.golden_expect(name, f, c)[0] for f, c in parts) == (
        gd["hash_total"] if bench.job_lookups(w, sc, 0, world) == gd["total"] else
        sum(gd["hash"][: world * 8 * w.lookups // gd["total"]]))


def test_golden_expect_rejects_unaligned():
    import bench
    assert bench.golden_expect("tiny", 0, 100_000) is not None
    assert bench.golden_expect("tiny", 1, 99_999) is None
    assert bench.golden_expect("nope", 0, 1) is None


def test_roofline_model_is_a_bound():
    """the reported fraction is achieved / peak for the binding resource; with any kernel time
    at least the FP64 / HBM minimum time it stays <= 1"""
    import bench
    w = bench.WORKLOADS["small"]
    pairs = 263_301_940
    lookups = 17_000_000
    peak_tf, _ = bench.fp64_peak_tflops(148)
    hbm_peak, _ = bench.measured_hbm_peak()
    t_alu = bench.FLOPS_PER_PAIR * pairs / (peak_tf * 1e12) * 1e3
    t_hbm = bench.hbm_min_bytes(w, lookups) / (hbm_peak * 1e9) * 1e3
    for ms in (max(t_alu, t_hbm), 0.66, 5.0):
        r = bench.roofline(w, "S", "material_energy", lookups, pairs, ms, 148, with_ncu=False)
        assert r["frac"] <= 1.0 + 1e-9
        assert r["frac"] == max(r["alu_fp64"]["frac"], r["hbm_min"]["frac"])
        assert r["bound"] == ("alu" if r["alu_fp64"]["frac"] >= r["hbm_min"]["frac"] else "hbm")
    r = bench.roofline(w, "S", "material_energy", lookups, pairs, max(t_alu, t_hbm), 148, with_ncu=False)
    assert abs(r["frac"] - 1.0) < 1e-9
    # the FP64 peak: 148 SMs x 64 lanes x 2 flops x ~1.965 GHz ~ 37 TFLOP/s (or the measured one)
    assert 20 < peak_tf < 60


def test_hbm_min_bytes():
    import bench
    w = bench.WORKLOADS["XL"]
    assert bench.hbm_min_bytes(w, 125_000_000) == 355 * 238847 * 48 + 12 * 125_000_000


def test_algorithmic_bytes():
    import bench
    from xs_workloads import WORKLOADS
    # E[n_nuc] x 96 B (nuclide), + 4 B (unionized), + 8 ceil(log2(W+1)) B (hash) per pair
    assert abs(bench.algorithmic_bytes_per_lookup(WORKLOADS["small"]) - 15.490 * 96) < 1e-9
    assert abs(bench.algorithmic_bytes_per_lookup(WORKLOADS["large"]) - 55.383 * 96) < 1e-9
    assert abs(bench.algorithmic_bytes_per_lookup(WORKLOADS["large-U"]) - 55.383 * 100) < 1e-9
    assert abs(bench.algorithmic_bytes_per_lookup(WORKLOADS["XL"]) - 55.383 * (96 + 8 * 5)) < 1e-9
