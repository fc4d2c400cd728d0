"""Full-size parity: the CUDA path at BASELINE.json's full sizes, in the launch configuration
bench.py times, against the CPU oracle's golden hashes (tests/golden/hashes.json, written by
tools/oracle_golden.py from oracle/ only), plus the q = 1.0 edge through every pipeline.

north_star: "the hash must match bit-exactly" -- here over every lookup of small (17M),
large (17M), large-U (100M) and XL (1B = 8 ranks x 125M), range by range exactly as the
ranks of bench.py split them."""
import json
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from xs_workloads import GRID_SEED, LOOKUP_SEED, WORKLOADS  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = json.load(open(os.path.join(ROOT, "tests", "golden", "hashes.json")))


@pytest.fixture(scope="module")
def xs():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_cgo_murtovigplls24_b200 as pkg
    return pkg


def _golden(name):
    if name not in GOLDEN:
        pytest.skip(f"no golden hashes for {name} (run tools/oracle_golden.py)")
    return GOLDEN[name]


@pytest.mark.slow
@pytest.mark.parametrize("name", ["small", "large", "large-U", "XL"])
def test_full_size_hash_golden(xs, name):
    """Every eighth of the workload (= rank r's range at N = 8; XL: rank r's 125M weak block)
    with the bench's default path, then N = 1 / 2 / 4 ranges (strong) as one launch each."""
    gd = _golden(name)
    w = WORKLOADS[name]
    b = gd["bounds"]
    with xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED) as g:
        for r in range(8):
            st = g.lookup_range(b[r], b[r + 1] - b[r], LOOKUP_SEED)
            assert (st.hash, st.pairs) == (gd["hash"][r], gd["pairs"][r]), (name, r)
        if name != "XL":  # strong-scaling ranges of N = 1, 2, 4 (XL runs weak at 125M per rank)
            for parts in (1, 2, 4):
                step = 8 // parts
                for r in range(parts):
                    i, j = r * step, (r + 1) * step
                    st = g.lookup_range(b[i], b[j] - b[i], LOOKUP_SEED)
                    assert st.hash == sum(gd["hash"][i:j]) and st.pairs == sum(gd["pairs"][i:j]), (name, parts, r)


@pytest.mark.slow
@pytest.mark.parametrize("name", ["small", "large", "large-U", "XL"])
@pytest.mark.parametrize("search,sort", [("U2", "material_energy"), ("M", "material_energy"), ("H", "material_energy"),
                                         ("U2", "none")])
def test_full_size_hash_golden_variants(xs, name, search, sort):
    """The paper's A/B variants (merged M, unmerged U2, unsorted XSBench order) and H on one
    full-size eighth (XL: one rank's 125M block) -- the same golden hash."""
    gd = _golden(name)
    w = WORKLOADS[name]
    b = gd["bounds"]
    r = 5
    with xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED) as g:
        st = g.lookup_range(b[r], b[r + 1] - b[r], LOOKUP_SEED, search=search, sort=sort)
        assert (st.hash, st.pairs) == (gd["hash"][r], gd["pairs"][r])


# ------------------------------------------------------------------ q = 1.0 exactly (R7)
Q_ONE_SEED = 5527465283667400870  # lookup 0 draws q = 1.0 exactly (one inverted LCG step)
PIPES = [("none", {}), ("material", {}), ("material_energy", {}), ("material", {"split": True}),
         ("material_energy", {"split": True}), ("history", {}), ("material_energy", {"coarse": True})]


@pytest.fixture(scope="module")
def q_one(xs, oracle_mod):
    out = {}
    for gt in (0, 1, 2):
        g = xs.Grid(68, 1000, gt, GRID_SEED)
        P = oracle_mod.Problem(68, 1000, gt, GRID_SEED)
        assert P.run_range(Q_ONE_SEED, 0, 1, mat=True, q=True)["q"][0] == 1.0
        ref = P.run_range(Q_ONE_SEED, 0, 4099, idx=True)
        out[gt] = (g, ref)
    yield out
    for g, _ in out.values():
        g.close()


@pytest.mark.parametrize("gt", [0, 1, 2])
@pytest.mark.parametrize("search", ["M", "U1", "U2", "U8", "B", "W", "H", "S"])
@pytest.mark.parametrize("sort,extra", PIPES)
def test_q_equal_one_every_pipeline(q_one, gt, search, sort, extra):
    """q = 1.0 exercises the clamps of bucket_key / refine_bin (sort), the bin tables (H, S)
    and the hash-grid bin (R7) -- every output and index against the oracle"""
    g, ref = q_one[gt]
    out, st = g.macro_xs(0, 4099, Q_ONE_SEED, search=search, sort=sort, **extra)
    assert st.hash == ref["hash"] and st.pairs == ref["pairs"]
    assert np.array_equal(out.cpu().numpy(), ref["macro"])
    idx = g.indices(0, 4099, Q_ONE_SEED, search=search, sort=sort, **extra)
    assert np.array_equal(idx.cpu().numpy(), ref["idx"])


def test_q_equal_one_full_size_grids(xs, oracle_mod):
    """the same edge on the full-size small nuclide grid and the XL hash grid (the bench's
    launch configuration), first lookup plus a ragged tail"""
    for name in ("small", "XL"):
        w = WORKLOADS[name]
        P = oracle_mod.Problem(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED)
        ref = P.run_range(Q_ONE_SEED, 0, 3001)
        with xs.Grid(w.n_nuclides, w.n_gridpoints, w.grid_type, GRID_SEED) as g:
            for search in ("S", "H", "U2"):
                out, st = g.macro_xs(0, 3001, Q_ONE_SEED, search=search)
                assert st.hash == ref["hash"], (name, search)
                assert np.array_equal(out.cpu().numpy(), ref["macro"]), (name, search)
