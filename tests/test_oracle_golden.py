"""Pins for what the full-size parity rests on (CPU only):

* the oracle's on-demand unionized path (IDX = NULL: IDX[e][i] computed by its definition,
  L_i(U[e]), oracle/xs_oracle.c or_lower) equals the table path (IDX built once) -- every
  large-U comparison and golden hash uses the on-demand path (5.7 GB of IDX is not built);
* tests/golden/hashes.json is what oracle/ computes: the tiny workload in full, the small
  workload's eighths re-run, and the structure (bounds = floor(r T / 8), sums) of every
  entry; the values come from tools/oracle_golden.py, which calls only oracle/."""
import json
import os

import numpy as np
import pytest

from xs_workloads import GRID_SEED, LOOKUP_SEED

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden", "hashes.json")


@pytest.mark.parametrize("n_nuc,n", [(68, 1000), (355, 300), (68, 2)])
def test_unionized_on_demand_equals_table(oracle_mod, n_nuc, n):
    P_tab = oracle_mod.Problem(n_nuc, n, oracle_mod.UNIONIZED, GRID_SEED, build_idx=True)
    P_dem = oracle_mod.Problem(n_nuc, n, oracle_mod.UNIONIZED, GRID_SEED, build_idx=False)
    assert P_tab.IDX is not None and P_dem.IDX is None
    for first, count in ((0, 20_000), (2 ** 40, 3_001)):
        a = P_tab.run_range(LOOKUP_SEED, first, count, idx=True)
        b = P_dem.run_range(LOOKUP_SEED, first, count, idx=True)
        assert a["hash"] == b["hash"] and a["pairs"] == b["pairs"]
        assert np.array_equal(a["idx"], b["idx"])
        assert np.array_equal(a["macro"], b["macro"])
    # and both equal the nuclide grid's definition L_i(q) (proof 2 of SURVEY.md §8c)
    P_nuc = oracle_mod.Problem(n_nuc, n, oracle_mod.NUCLIDE, GRID_SEED)
    c = P_nuc.run_range(LOOKUP_SEED, 0, 20_000, idx=True)
    assert np.array_equal(c["idx"], P_dem.run_range(LOOKUP_SEED, 0, 20_000, idx=True)["idx"])


def test_unionized_on_demand_edges(oracle_mod):
    """energies exactly at unionized points, 0 and 1: table and definition agree"""
    P_tab = oracle_mod.Problem(68, 200, oracle_mod.UNIONIZED, GRID_SEED, build_idx=True)
    P_dem = oracle_mod.Problem(68, 200, oracle_mod.UNIONIZED, GRID_SEED, build_idx=False)
    qs = np.concatenate([P_tab.U[::37], np.nextafter(P_tab.U[::53], 2), [0.0, 1.0, P_tab.U[-1]]])
    for q in qs:
        for mat in (0, 1, 6, 11):
            a, La = P_tab.macro_xs(mat, float(q))
            b, Lb = P_dem.macro_xs(mat, float(q))
            assert np.array_equal(a, b) and np.array_equal(La, Lb)


def _golden():
    if not os.path.exists(GOLDEN):
        pytest.skip("tests/golden/hashes.json not written yet")
    return json.load(open(GOLDEN))


def test_golden_structure():
    g = _golden()
    for name, d in g.items():
        if name.startswith("_"):
            continue
        T = d["total"]
        assert d["bounds"] == [T * r // 8 for r in range(9)]
        assert len(d["hash"]) == len(d["pairs"]) == 8
        assert d["hash_total"] == sum(d["hash"]) and d["pairs_total"] == sum(d["pairs"])
        for r in range(8):  # v in [1, 5] per lookup
            n = d["bounds"][r + 1] - d["bounds"][r]
            assert n <= d["hash"][r] <= 5 * n


def test_golden_tiny_is_the_oracle(oracle_mod):
    g = _golden()["tiny"]
    P = oracle_mod.Problem(68, 1000, oracle_mod.NUCLIDE, GRID_SEED)
    b = g["bounds"]
    for r in range(8):
        res = P.run_range(LOOKUP_SEED, b[r], b[r + 1] - b[r], macro=False)
        assert (res["hash"], res["pairs"]) == (g["hash"][r], g["pairs"][r])


def test_golden_small_is_the_oracle(oracle_mod):
    """two of small's eighths re-run (~2 s): the committed values are the oracle's"""
    g = _golden()
    if "small" not in g:
        pytest.skip("no small entry")
    g = g["small"]
    P = oracle_mod.Problem(68, 11303, oracle_mod.NUCLIDE, GRID_SEED)
    b = g["bounds"]
    for r in (0, 7):
        res = P.run_range(LOOKUP_SEED, b[r], b[r + 1] - b[r], macro=False)
        assert (res["hash"], res["pairs"]) == (g["hash"][r], g["pairs"][r])
