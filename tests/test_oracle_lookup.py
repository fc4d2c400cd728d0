"""Pins for interpolation, accumulation, verification and the hash.

Closed forms use dyadic data so every intermediate is exact and the expected value
is known with no rounding (reading R8); argmax cases are hand-made
(reading R10); hash invariances are properties of a sum over independent lookups."""
from fractions import Fraction

import numpy as np
import pytest

from xs_workloads import GRID_SEED, LOOKUP_SEED


def _dyadic_problem(oracle_mod, n_nuc=68, n=64, grid_type=1, linear=True):
    E = np.tile(np.arange(n, dtype=np.float64) / 64.0, (n_nuc, 1))  # k/64
    alpha = np.array([1.0, 2.0, 0.5, 3.0, 0.25])
    beta = np.array([0.5, -1.0, 2.0, 0.0, 4.0])
    if linear:
        X = alpha[None, None, :] + beta[None, None, :] * E[:, :, None]
    else:
        X = np.broadcast_to(alpha, (n_nuc, n, 5)).copy()
    num, mats, mx = oracle_mod.materials(n_nuc)
    concs = np.zeros((12, mx))
    for m in range(12):
        concs[m, : num[m]] = (np.arange(num[m]) % 7 + 1) / 8.0  # dyadic
    P = oracle_mod.Problem(n_nuc, n, grid_type, E=E, X=X, concs=concs)
    return P, alpha, beta


@pytest.mark.parametrize("gt", [0, 1, 2])
def test_linear_channels_exact(oracle_mod, gt):
    P, alpha, beta = _dyadic_problem(oracle_mod, grid_type=gt)
    # queries: dyadic points inside, at gridpoints, and outside (extrapolation, R6)
    qs = [k / 1024.0 for k in range(0, 1024, 7)] + [-0.25, 1.5, 63 / 64.0, 0.0]
    for q in qs:
        for nuc in (0, 5, 67):
            Lx = min(max(int(np.floor(q * 64)), 0), 62)
            micro = P.micro_xs(nuc, q, Lx)
            expect = alpha + beta * q
            assert np.array_equal(micro, expect), (q, micro, expect)


def test_linear_channels_random_grid(oracle_mod):
    # non-dyadic grid: the interpolant of linear data equals it to a few ulp
    rng = np.random.default_rng(0)
    n_nuc, n = 68, 100
    E = np.sort(rng.random((n_nuc, n)), axis=1)
    alpha = rng.random(5)
    beta = rng.random(5)
    X = alpha + beta * E[:, :, None]
    P = oracle_mod.Problem(n_nuc, n, 1, E=E, X=X)
    for _ in range(2000):
        nuc = int(rng.integers(0, n_nuc))
        q = float(rng.random())
        L = oracle_mod.search_def(E[nuc], q)
        micro = P.micro_xs(nuc, q, L)
        np.testing.assert_allclose(micro, alpha + beta * q, rtol=1e-13, atol=1e-15)


def test_gridpoint_gives_f1(oracle_mod, tiny_problem):
    P = tiny_problem
    for nuc in (0, 33, 67):
        for k in (0, 1, 500, 998):
            q = P.E[nuc, k]
            micro = P.micro_xs(nuc, q, k)
            # f = 1 exactly at the lower gridpoint: micro = X_hi - (X_hi - X_lo) = X_lo (to rounding of d)
            np.testing.assert_allclose(micro, P.X[nuc, k], rtol=0, atol=1e-15)


@pytest.mark.parametrize("gt", [0, 1, 2])
def test_constant_channels_macro_exact(oracle_mod, gt):
    P, alpha, _ = _dyadic_problem(oracle_mod, grid_type=gt, linear=False)
    for mat in range(12):
        macro, _ = P.macro_xs(mat, 0.3)
        S = sum(Fraction(float(c)) for c in P.concs[mat, : P.num_nucs[mat]])
        for c in range(5):
            assert Fraction(macro[c]) == Fraction(float(alpha[c])) * S


def test_verify_argmax_semantics(oracle_mod):
    assert oracle_mod.verify([1, 2, 3, 4, 5]) == 5
    assert oracle_mod.verify([5, 4, 3, 2, 1]) == 1
    assert oracle_mod.verify([1, 3, 3, 2, 0]) == 2  # first maximum wins
    assert oracle_mod.verify([0, 0, 0, 0, 0]) == 1
    nan = float("nan")
    assert oracle_mod.verify([nan] * 5) == 1
    assert oracle_mod.verify([nan, 0.5, nan, 0.7, 0.1]) == 4
    assert oracle_mod.verify([-2, -3, -1.5, -4, -5]) == 1  # nothing beats -1.0


def test_lookup_values_in_range(tiny_problem):
    r = tiny_problem.run_range(LOOKUP_SEED, 0, 20_000, macro=True, mat=True, q=True, idx=True)
    assert r["hash"] >= 20_000 and r["hash"] <= 5 * 20_000
    assert np.all((r["q"] >= 0) & (r["q"] <= 1))
    num = tiny_problem.num_nucs
    assert r["pairs"] == int(num[r["mat"]].sum())
    for row, m in zip(r["idx"][:500], r["mat"][:500]):
        assert np.all(row[: num[m]] >= 0) and np.all(row[: num[m]] <= 998)
        assert np.all(row[num[m]:] == -1)


def test_hash_shard_and_permutation_invariance(tiny_problem):
    P = tiny_problem
    full = P.run_range(LOOKUP_SEED, 0, 30_000)
    parts = [P.run_range(LOOKUP_SEED, a, b - a) for a, b in [(0, 7_001), (7_001, 20_000), (20_000, 30_000)]]
    assert sum(p["hash"] for p in parts) == full["hash"]
    assert sum(p["pairs"] for p in parts) == full["pairs"]
    assert np.array_equal(np.concatenate([p["macro"] for p in parts]), full["macro"])
    perm = np.random.default_rng(1).permutation(30_000)
    h, macro = P.run_indices(LOOKUP_SEED, perm)
    assert h == full["hash"]
    assert np.array_equal(macro, full["macro"][perm])
    # thread count does not matter
    assert P.run_range(LOOKUP_SEED, 0, 30_000, threads=1)["hash"] == full["hash"]


def test_definition_mode_equals_listing1_tiny(oracle_mod):
    """Full tiny config: Listing-1 oracle == plain-definition oracle (linear scans)."""
    P = oracle_mod.Problem(68, 1000, oracle_mod.NUCLIDE, GRID_SEED)
    a = P.run_range(LOOKUP_SEED, 0, 100_000, idx=True)
    P.with_search_mode(1)
    b = P.run_range(LOOKUP_SEED, 0, 100_000, idx=True)
    assert a["hash"] == b["hash"]
    assert np.array_equal(a["idx"], b["idx"])
    assert np.array_equal(a["macro"], b["macro"])


def test_three_grid_types_agree(oracle_mod):
    """SURVEY.md §8c proofs 2-3: unionized, nuclide and hash paths give identical L."""
    res = {}
    for gt in (0, 1, 2):
        P = oracle_mod.Problem(68, 1000, gt, GRID_SEED)
        res[gt] = P.run_range(LOOKUP_SEED, 0, 30_000, idx=True)
    for gt in (0, 2):
        assert np.array_equal(res[gt]["idx"], res[1]["idx"])
        assert np.array_equal(res[gt]["macro"], res[1]["macro"])
        assert res[gt]["hash"] == res[1]["hash"]


def test_hash_grid_bin_edges(oracle_mod):
    """Queries at and next to every hash-bin edge hit the window guards (R7)."""
    P1 = oracle_mod.Problem(68, 300, oracle_mod.NUCLIDE, 7)
    P2 = oracle_mod.Problem(68, 300, oracle_mod.HASH, 7)
    Pu = oracle_mod.Problem(68, 300, oracle_mod.UNIONIZED, 7)
    du = 1.0 / 10000
    qs = []
    for b in list(range(0, 10000, 97)) + [9999]:
        e = b * du
        qs += [e, np.nextafter(e, 0), np.nextafter(e, 1)]
    qs += [1.0, 0.0, np.nextafter(1.0, 0)] + list(P1.E[3, :5]) + list(P1.E[3, -5:])
    for q in qs:
        a = P1.macro_xs(0, float(q))
        b = P2.macro_xs(0, float(q))
        c = Pu.macro_xs(0, float(q))
        assert np.array_equal(a[1], b[1]) and np.array_equal(a[1], c[1]), q
        assert np.array_equal(a[0], b[0]) and np.array_equal(a[0], c[0])
        # the indices are the plain definition
        for j, nuc in enumerate(P1.mats[0, : P1.num_nucs[0]]):
            assert a[1][j] == oracle_mod.search_def(P1.E[nuc], float(q))
