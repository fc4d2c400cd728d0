"""The N > 1 path through libxs on a GPU: world_size-2 process groups over gloo, both ranks on
the visible GPU(s) (a gpurun box has one), each running the CUDA path on its shard.

SURVEY.md §8e: rank r of R owns lookups [floor(rN/R), floor((r+1)N/R)); the grid is
replicated (one checksum MIN/MAX proves it); the verification reduction sums the hashes.
The same driver code runs over NCCL on an 8-GPU node."""
import json
import os
import socket
import subprocess
import sys

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = json.load(open(os.path.join(ROOT, "tests", "golden", "hashes.json")))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, total, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world), LOCAL_RANK=str(rank))
    sys.path.insert(0, ROOT)
    import paper_conf_cgo_murtovigplls24_b200 as xs
    from paper_conf_cgo_murtovigplls24_b200 import driver
    from xs_workloads import GRID_SEED, LOOKUP_SEED
    R = driver.init(backend="gloo")
    first, count = driver.shard(total, R.rank, R.world)
    with xs.Grid(68, 1000, xs.XS_NUCLIDE, GRID_SEED) as g:
        ok = driver.replicas_identical(g.checksum())
        st = g.lookup_range(first, count, LOOKUP_SEED)
        h, n, pairs, ms = driver.reduce_stats(st.hash, st.lookups, st.pairs, st.device_ms)
    driver.barrier()
    if rank == 0:
        q.put((ok, h, n, pairs, ms > 0))
    driver.finalize()


def test_two_ranks_libxs_gloo():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    total = 100_000
    procs = [ctx.Process(target=_worker, args=(r, 2, port, total, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(300)
        assert p.exitcode == 0
    ok, h, n, pairs, timed = q.get(timeout=10)
    gd = GOLDEN["tiny"]
    assert ok and timed
    assert (h, n, pairs) == (gd["hash_total"], total, gd["pairs_total"])


def _bench(*args, timeout=900):
    env = dict(os.environ, XS_DIST_BACKEND="gloo")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       timeout=timeout, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


@pytest.mark.parametrize("scaling,lookups", [("strong", 0), ("strong-index", 0), ("weak", 50_000)])
def test_bench_two_ranks(scaling, lookups):
    """`bench.py --gpus 2` launches two ranks itself (torch.distributed.run) and reports the
    job: n_gpus 2, the oracle's hash over the union of the ranks' lookups (strong: key-range
    shards of the whole range; strong-index: index ranges; weak: 50k per rank)"""
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    d = _bench("--gpus", "2", "--workload", "tiny", "--scaling", scaling, "--lookups", str(lookups),
               "--steps", "3", "--warmup", "3", "--ab", "", "--workloads", "", "--no-e2e", "--no-cpu-baseline")
    gd = GOLDEN["tiny"]
    assert d["n_gpus"] == 2 and d["scaling"] == ("weak" if scaling == "weak" else "strong")
    assert d["path"]["backend"] == "gloo"
    assert ("key-range" in d["config"]["parallelism"]) == (scaling == "strong")
    assert d["config"]["lookups_total"] == 100_000
    assert d["verification"]["hash"] == gd["hash_total"] and d["verification"]["pairs"] == gd["pairs_total"]
    assert d["verification"]["golden_match"] is True
    assert d["value"] > 0 and d["roofline"]["frac"] <= 1.0
    for label, v in d["north_star"].items():
        assert v["hash_ok"] and v["golden_match"] is True, label


def test_bench_one_rank_golden_and_contract():
    """N = 1 line of the default protocol on tiny: keys of the contract, golden hash, a
    roofline fraction that cannot exceed 1, algorithmic bytes per step below the peak"""
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    d = _bench("--workload", "tiny", "--steps", "3", "--warmup", "3", "--ab", "M,U2,S", "--workloads", "small",
               "--cpu-seconds", "1")
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "gpu_launches", "clocks"):
        assert k in d, k
    assert d["n_gpus"] == 1 and d["verification"]["golden_match"] is True
    assert d["verification"]["oracle_sample_hash_match"] is True
    rf = d["roofline"]
    assert rf["bound"] in ("alu", "hbm") and 0 < rf["frac"] <= 1.0
    assert rf["hbm_min"]["bytes_per_launch"] / (d["ms_per_step"] / 1e3) / 1e9 <= rf["hbm_min"]["peak"]
    assert d["workloads"]["small"]["golden_match"] is True
    assert d["workloads"]["small"]["roofline"]["frac"] <= 1.0
    assert d["gpu_launches"] > 0


def test_bench_nccl_all_gpus():
    """The production path: one rank per GPU over NCCL (NVLink / NVSwitch), launched by
    bench.py itself -- runs only where more than one GPU is visible (an 8-GPU node)."""
    if not torch.cuda.is_available() or torch.cuda.device_count() < 2:
        pytest.skip("needs >= 2 GPUs")
    n = min(torch.cuda.device_count(), 8)
    env = {k: v for k, v in os.environ.items() if k != "XS_DIST_BACKEND"}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", str(n), "--workload", "tiny",
                        "--steps", "3", "--warmup", "3", "--ab", "", "--workloads", "", "--no-e2e",
                        "--no-cpu-baseline"], capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    d = json.loads([l for l in r.stdout.splitlines() if l.startswith("{")][-1])
    gd = GOLDEN["tiny"]
    assert d["n_gpus"] == n and d["path"]["backend"] == "nccl"
    assert d["verification"]["hash"] == gd["hash_total"] and d["verification"]["golden_match"] is True
