"""Pins for the bezier-surface oracle (oracle/bezier_oracle.c; Listing 2,
readings BZ1-BZ5): closed forms (binomial coefficients, Bernstein polynomials), exact
special cases (k = 0, k = n, the four corners), linear precision, and an independent
algorithm (de Casteljau) -- none of them re-types the oracle's formulas."""
import math

import numpy as np
import pytest

import oracle
from xs_workloads import bezier_control_net


@pytest.mark.parametrize("n", list(range(0, 41)))
def test_blend_loop_is_binomial(n):
    # Listing 2 computes n! / (k! (n-k)!) with interleaved divisions
    for k in range(n + 1):
        exact = math.comb(n, k)
        got = oracle.blend_loop(k, n)
        assert abs(got - exact) <= 4 * n * 2.3e-16 * exact, (n, k, got, exact)
        g32 = oracle.blend_loop(k, n, np.float32)
        assert abs(g32 - exact) <= 4 * n * 1.2e-7 * exact, (n, k, g32, exact)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_blend_loop_exact_ends(dtype):
    # k = 0 and k = n: every division undoes the preceding multiplication exactly
    for n in range(0, 200):
        assert oracle.blend_loop(0, n, dtype) == 1.0
        assert oracle.blend_loop(n, n, dtype) == 1.0


def test_blend_loop_small_exact():
    # the first few rows of Pascal's triangle come out exact (every intermediate is an
    # integer or a quotient that is immediately multiplied back to an integer)
    for n, row in [(1, [1, 1]), (2, [1, 2, 1]), (3, [1, 3, 3, 1]), (4, [1, 4, 6, 4, 1])]:
        assert [oracle.blend_loop(k, n) for k in range(n + 1)] == row


@pytest.mark.parametrize("n", [1, 2, 3, 5, 8, 16, 31])
def test_bernstein_closed_form_and_partition(n):
    for mu in [0.0, 1e-3, 0.1, 1 / 3, 0.5, 0.77, 0.999, 1.0]:
        vals = [oracle.bezier_blend(k, mu, n) for k in range(n + 1)]
        for k, v in enumerate(vals):
            ref = math.comb(n, k) * mu ** k * (1 - mu) ** (n - k)
            assert v >= 0.0 and abs(v - ref) <= 1e-14 * max(1.0, ref) * n, (n, k, mu, v, ref)
        assert abs(math.fsum(vals) - 1.0) <= 1e-14 * n


def _de_casteljau_curve(pts, t):
    pts = [np.array(p, dtype=np.float64) for p in pts]
    while len(pts) > 1:
        pts = [(1 - t) * a + t * b for a, b in zip(pts[:-1], pts[1:])]
    return pts[0]


def _de_casteljau_surface(P, u, v):
    # evaluate every row curve at v, then the column of results at u (independent of
    # the blend formula: repeated linear interpolation)
    rows = [_de_casteljau_curve(P[ki], v) for ki in range(P.shape[0])]
    return _de_casteljau_curve(rows, u)


@pytest.mark.parametrize("ni,nj", [(5, 4), (1, 1), (0, 3), (3, 0), (7, 2)])
def test_surface_matches_de_casteljau(ni, nj):
    P = bezier_control_net(ni, nj, seed=3)
    res_i, res_j = 9, 6
    S = oracle.bezier_surface(P, res_i, res_j)
    for i in range(res_i):
        for j in range(res_j):
            ref = _de_casteljau_surface(P, i / (res_i - 1), j / (res_j - 1))
            assert np.allclose(S[i, j], ref, rtol=1e-13, atol=1e-13), (i, j, S[i, j], ref)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_surface_corners_exact(dtype):
    P = bezier_control_net(5, 4, seed=11, dtype=dtype)
    S = oracle.bezier_surface(P, 13, 7)
    assert S.dtype == dtype
    assert np.array_equal(S[0, 0], P[0, 0]) and np.array_equal(S[-1, -1], P[-1, -1])
    assert np.array_equal(S[0, -1], P[0, -1]) and np.array_equal(S[-1, 0], P[-1, 0])


def test_surface_linear_precision():
    # Bernstein polynomials reproduce bilinear data: P = (ki/ni, kj/nj, ki kj/(ni nj))
    # gives S(u, v) = (u, v, u v); x depends on i only, y on j only (catches a transposed net)
    ni, nj, ri, rj = 6, 3, 11, 8
    ki, kj = np.meshgrid(np.arange(ni + 1), np.arange(nj + 1), indexing="ij")
    P = np.stack([ki / ni, kj / nj, ki * kj / (ni * nj)], axis=-1)
    S = oracle.bezier_surface(P, ri, rj)
    u = (np.arange(ri) / (ri - 1))[:, None]
    v = (np.arange(rj) / (rj - 1))[None, :]
    assert np.allclose(S[..., 0], u + 0 * v, atol=1e-14)
    assert np.allclose(S[..., 1], v + 0 * u, atol=1e-14)
    assert np.allclose(S[..., 2], u * v, atol=1e-14)


def test_surface_fp32_tracks_fp64():
    P = bezier_control_net(5, 4, seed=5)
    S64 = oracle.bezier_surface(P, 33, 17)
    S32 = oracle.bezier_surface(P.astype(np.float32), 33, 17)
    assert np.allclose(S32, S64, rtol=1e-5, atol=1e-5)
    assert not np.array_equal(S32.astype(np.float64), S64)   # really computed in fp32


def test_surface_points_match_surface():
    P = bezier_control_net(5, 4)
    S = oracle.bezier_surface(P, 21, 19)
    rng = np.random.default_rng(0)
    ii, jj = rng.integers(0, 21, 50), rng.integers(0, 19, 50)
    assert np.array_equal(oracle.bezier_surface_points(P, 21, 19, ii, jj), S[ii, jj])
