"""Pins for the oracle's search: Listing 3 against hand-traced
golden runs, a brute-force linear scan, numpy.searchsorted, and the invariants
A[L] <= q < A[L+1] with endpoint clamps (SURVEY.md §8c proof 1)."""
import os

import numpy as np
import pytest

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "listing3_traces.txt")


def _golden():
    rows = []
    for line in open(GOLDEN):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        A, lo, hi, q, res, probes = [x.strip() for x in line.split("|")]
        rows.append((np.array([float(v) for v in A.split(",")]), int(lo), int(hi), float(q), int(res),
                     [int(p) for p in probes.split(",")] if probes else []))
    return rows


def test_golden_traces(oracle_mod):
    rows = _golden()
    assert len(rows) >= 10
    for A, lo, hi, q, res, probes in rows:
        r, p = oracle_mod.search_listing1_trace(A, lo, hi, q)
        assert r == res and p == probes, (A, q, r, p)
        assert oracle_mod.search_listing1(A, lo, hi, q) == res


def _L_numpy(A, q):
    n = len(A)
    return int(min(max(np.searchsorted(A, q, side="right") - 1, 0), n - 2))


@pytest.mark.parametrize("n", [2, 3, 4, 5, 17, 1000])
def test_listing1_vs_bruteforce_and_library(oracle_mod, n):
    rng = np.random.default_rng(n)
    for trial in range(20):
        A = np.sort(rng.random(n))
        A = np.unique(A)
        if len(A) < 2:
            continue
        m = len(A)
        mids = (A[:-1] + A[1:]) / 2
        qs = np.concatenate([A, mids, [A[0] - 1.0, A[-1] + 1.0, np.nextafter(A[0], -1), 0.0, 1.0],
                             np.nextafter(A, 2.0), np.nextafter(A, -2.0)])
        for q in qs:
            L = oracle_mod.search_listing1(A, 0, m - 1, q)
            assert L == oracle_mod.search_def(A, q) == _L_numpy(A, q)
            # invariant for interior q; clamps outside
            if A[0] <= q < A[-1]:
                assert A[L] <= q < A[L + 1]
            elif q < A[0]:
                assert L == 0
            else:
                assert L == m - 2


def test_listing1_duplicates_unique_result(oracle_mod):
    rng = np.random.default_rng(11)
    for _ in range(200):
        A = np.sort(rng.integers(0, 6, size=rng.integers(2, 12)).astype(float))
        for q in np.arange(-1, 7, 0.5):
            assert oracle_mod.search_listing1(A, 0, len(A) - 1, q) == _L_numpy(A, q)


def test_listing1_subrange_window(oracle_mod):
    # On a window [lo, hi] with A[lo] <= q < A[hi], the search returns L(q)
    rng = np.random.default_rng(5)
    A = np.sort(rng.random(500))
    for _ in range(2000):
        q = rng.random() * (A[-1] - A[0]) + A[0]
        L = _L_numpy(A, q)
        lo = rng.integers(0, L + 1)
        hi = rng.integers(L + 1, len(A))
        assert oracle_mod.search_listing1(A, lo, hi, q) == L


def test_iteration_count_bound(oracle_mod):
    # probes = floor or ceil of log2(n-1)
    A = np.arange(11303, dtype=float)
    rng = np.random.default_rng(1)
    for q in rng.random(500) * 11303:
        _, p = oracle_mod.search_listing1_trace(A, 0, 11302, q)
        assert 13 <= len(p) <= 14
