"""Pins for the oracle's grids: every point's draws recomputed with Python big-int
LCG stepping, sortedness, and IDX / H checked by numpy.searchsorted (a library
routine) against their definitions (readings R4, R7, R11)."""
import numpy as np

M = 2 ** 63
A = 2806196910506780709


def test_nuclide_grid_points_from_stream(oracle_mod):
    n_nuc, n, seed = 68, 12, 42
    P = oracle_mod.Problem(n_nuc, n, oracle_mod.NUCLIDE, seed)
    s = seed
    vals = []
    for _ in range(6 * n_nuc * n):
        s = (A * s + 1) % M
        vals.append(float(s) / 2.0 ** 63)
    vals = np.array(vals).reshape(n_nuc, n, 6)
    for i in range(n_nuc):
        order = np.argsort(vals[i, :, 0], kind="stable")
        row = vals[i, order]
        assert np.array_equal(P.E[i], row[:, 0])
        assert np.array_equal(P.X[i], row[:, 1:])
    # concentrations continue the stream at 6N, material-major
    t = 0
    for m in range(12):
        for j in range(P.max_nucs):
            if j < P.num_nucs[m]:
                s = (A * s + 1) % M
                assert P.concs[m, j] == float(s) / 2.0 ** 63
            else:
                assert P.concs[m, j] == 0.0
            t += 1


def test_grid_sorted_strictly(tiny_problem):
    E = tiny_problem.E
    assert np.all(np.diff(E, axis=1) > 0)
    assert np.all((E >= 0) & (E <= 1))
    assert np.all((tiny_problem.X >= 0) & (tiny_problem.X <= 1))


def test_unionized_grid_definition(oracle_mod):
    P = oracle_mod.Problem(68, 200, oracle_mod.UNIONIZED, 42)
    assert np.array_equal(P.U, np.sort(P.E.ravel()))
    for i in range(68):
        Li = np.clip(np.searchsorted(P.E[i], P.U, side="right") - 1, 0, 198)
        assert np.array_equal(P.IDX[:, i], Li)


def test_hash_grid_definition(oracle_mod):
    P = oracle_mod.Problem(68, 200, oracle_mod.HASH, 42, bins=10000)
    du = 1.0 / 10000
    energies = np.arange(10000, dtype=np.float64) * du
    for i in range(68):
        Li = np.clip(np.searchsorted(P.E[i], energies, side="right") - 1, 0, 198)
        assert np.array_equal(P.H[:, i], Li)


def test_large_table_grid_small_n(oracle_mod):
    P = oracle_mod.Problem(355, 50, oracle_mod.NUCLIDE, 42)
    assert P.E.shape == (355, 50)
    assert np.all(np.diff(P.E, axis=1) > 0)
