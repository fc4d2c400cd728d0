"""Key-range sharding (xs_opts.shard_index / shard_count): every shard draws all
lookups of the range and orders / looks up only those whose (material, energy) bucket lies in
its share of the buckets.  The shards must partition the lookups exactly: every lookup's
macroscopic XS is written by exactly one shard and equals the oracle's bit for bit, and the
shards' hashes, pairs and lookup counts sum to the oracle's totals -- at the tiny size for
every grid type and several shard counts (including more shards than some materials have
buckets), and at full size against the golden hashes."""
import json
import os

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SENT = np.int64(0x7FF4DEADBEEF1234)


@pytest.fixture(scope="module")
def torch_gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    return torch


@pytest.mark.parametrize("gt", [0, 1, 2])
@pytest.mark.parametrize("nshards", [2, 3, 8, 61])
def test_shards_partition_the_lookups(torch_gpu, gt, nshards):
    torch = torch_gpu
    import oracle
    import paper_conf_cgo_murtovigplls24_b200 as xs
    first, count = 777, 100_003
    ref = oracle.Problem(68, 1000, gt, 42).run_range(1070, first, count)
    owner = np.zeros(count, dtype=np.int64)
    got = np.zeros((count, 5))
    h = p = n = 0
    with xs.Grid(68, 1000, gt, 42) as g:
        for s in range(nshards):
            buf = torch.full((count * 5,), int(SENT), dtype=torch.int64, device="cuda")
            out = buf.view(torch.float64).view(count, 5)
            st = g.lookup_range(first, count, 1070, out, search="S", shard=(s, nshards))
            bits = buf.view(count, 5).cpu().numpy()
            mine = ~(bits == SENT).all(axis=1)
            assert not (bits[mine] == SENT).any(), "a shard wrote part of a row"
            assert int(mine.sum()) == st.lookups, (s, int(mine.sum()), st.lookups)
            owner += mine
            got[mine] = out.cpu().numpy()[mine]
            h, p, n = h + st.hash, p + st.pairs, n + st.lookups
    assert (owner == 1).all(), "every lookup in exactly one shard"
    assert (h, p, n) == (ref["hash"], ref["pairs"], count)
    assert np.array_equal(got, ref["macro"])


def test_shard_argument_checks(torch_gpu):
    import paper_conf_cgo_murtovigplls24_b200 as xs
    with xs.Grid(68, 200, xs.XS_NUCLIDE, 42) as g:
        for bad in (dict(search="U2", shard=(0, 2)), dict(search="S", sort="material", shard=(0, 2)),
                    dict(search="S", split=True, shard=(0, 2)), dict(search="S", coarse=True, shard=(1, 2)),
                    dict(search="S", shard=(2, 2)), dict(search="S", shard=(-1, 2)), dict(search="S", shard=(1, 1))):
            with pytest.raises(xs.XSError):
                g.lookup_range(0, 1000, 1070, None, **bad)
        st = g.lookup_range(0, 1000, 1070, None, search="S", shard=(0, 1))
        assert st.lookups == 1000


@pytest.mark.slow
@pytest.mark.parametrize("nshards", [2, 8])
def test_shards_sum_to_golden_large_u(torch_gpu, nshards):
    """the metric's configuration at full size: 100M lookups over 2 or 8 key-range shards
    sum to the oracle's golden hash and pairs"""
    import paper_conf_cgo_murtovigplls24_b200 as xs
    from xs_workloads import GRID_SEED, LOOKUP_SEED, WORKLOADS
    w = WORKLOADS["large-U"]
    gold = json.load(open(os.path.join(ROOT, "tests", "golden", "hashes.json")))["large-U"]
    h = p = n = 0
    with xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED) as g:
        for s in range(nshards):
            st = g.lookup_range(0, w.lookups, LOOKUP_SEED, None, search="S", shard=(s, nshards))
            assert st.lookups > 0
            h, p, n = h + st.hash, p + st.pairs, n + st.lookups
    assert (h, p, n) == (sum(gold["hash"]), sum(gold["pairs"]), w.lookups)


CHUNK_SCRIPT = r"""
import sys; sys.path.insert(0, %r)
import numpy as np, torch
import oracle
import paper_conf_cgo_murtovigplls24_b200 as xs
first, count, n = 5, 100_003, 3
ref = oracle.Problem(68, 1000, 0, 42).run_range(1070, first, count)
SENT = np.int64(0x7FF4DEADBEEF1234)
got = np.zeros((count, 5)); owner = np.zeros(count, dtype=np.int64); h = p = nl = 0
with xs.Grid(68, 1000, 0, 42) as g:
    for s in range(n):
        buf = torch.full((count * 5,), int(SENT), dtype=torch.int64, device="cuda")
        out = buf.view(torch.float64).view(count, 5)
        st = g.lookup_range(first, count, 1070, out, search="S", shard=(s, n))
        mine = ~(buf.view(count, 5).cpu().numpy() == SENT).all(axis=1)
        owner += mine; got[mine] = out.cpu().numpy()[mine]
        h, p, nl = h + st.hash, p + st.pairs, nl + st.lookups
assert (owner == 1).all() and np.array_equal(got, ref["macro"])
assert (h, p, nl) == (ref["hash"], ref["pairs"], count), (h, p, nl)
print("SHARD CHUNKS OK")
""" % ROOT


def test_shards_across_chunks(torch_gpu):
    """XS_TEST_MAX_CHUNK forces many internal chunks: every chunk is sharded on its own and the
    shard's lookups accumulate across chunks (stats.lookups, the published hash / pairs)"""
    import subprocess
    import sys
    env = dict(os.environ, XS_TEST_MAX_CHUNK="30011")
    r = subprocess.run([sys.executable, "-c", CHUNK_SCRIPT], capture_output=True, text=True, env=env, timeout=600)
    assert r.returncode == 0 and "SHARD CHUNKS OK" in r.stdout, (r.stdout[-2000:], r.stderr[-3000:])
