"""Pins for pick_mat (reading R9) and the material tables."""
import numpy as np
import pytest

# dist[] from XSBench [XSB]; the thresholds are dist[i] + ... + dist[1] (dist[0] never enters)
DIST = [0.140, 0.052, 0.275, 0.134, 0.154, 0.064, 0.066, 0.055, 0.008, 0.015, 0.025, 0.013]
DECIMAL_T = [0.0, 0.052, 0.327, 0.461, 0.615, 0.679, 0.745, 0.800, 0.808, 0.823, 0.848, 0.861]


def test_thresholds_decimal(oracle_mod):
    T = oracle_mod.pick_mat_thresholds()
    for i in range(12):
        assert abs(T[i] - DECIMAL_T[i]) < 1e-12
    assert np.all(np.diff(T) > 0)


def test_pick_mat_boundaries(oracle_mod):
    T = oracle_mod.pick_mat_thresholds()
    assert oracle_mod.pick_mat(0.0) == 1
    for m in range(1, 12):
        assert oracle_mod.pick_mat(np.nextafter(T[m], 0)) == m
        # exactly at T[m] the comparison `roll < running` fails
        expect = m + 1 if m < 11 else 0
        assert oracle_mod.pick_mat(T[m]) == expect
    assert oracle_mod.pick_mat(0.9999) == 0
    assert oracle_mod.pick_mat(1.0) == 0


def test_pick_mat_chi2(oracle_mod):
    from xs_workloads import LOOKUP_SEED
    P = oracle_mod.Problem(68, 16)
    res = P.run_range(LOOKUP_SEED, 0, 1_000_000, macro=False, mat=True)
    counts = np.bincount(res["mat"], minlength=12)
    p = np.array([1 - DECIMAL_T[11]] + [DECIMAL_T[m] - DECIMAL_T[m - 1] for m in range(1, 12)])
    exp = p * 1_000_000
    chi2 = float(((counts - exp) ** 2 / exp).sum())
    # 11 dof; P(chi2 > 31.3) ~ 0.001
    assert chi2 < 31.3, (chi2, counts)


@pytest.mark.parametrize("n_nuc,fuel", [(68, 34), (355, 321), (400, 321)])
def test_tables(oracle_mod, n_nuc, fuel):
    num, mats, mx = oracle_mod.materials(n_nuc)
    assert mx == fuel
    assert list(num) == [fuel, 5, 4, 4, 27, 21, 21, 21, 21, 21, 9, 9]
    for m in range(12):
        row = mats[m, : num[m]]
        assert np.all(row >= 0) and np.all(row < min(n_nuc, 355))
        assert len(set(row.tolist())) == num[m]  # no nuclide twice in a material
        assert np.all(mats[m, num[m]:] == -1)
    if fuel == 321:
        assert list(mats[0, 34:321]) == list(range(68, 355))


def test_invalid_nuclide_count(oracle_mod):
    with pytest.raises(ValueError):
        oracle_mod.materials(100)


def test_mean_nuclides_per_lookup(oracle_mod):
    from xs_workloads import MEAN_NUCS
    for n_nuc in (68, 355):
        num, _, _ = oracle_mod.materials(n_nuc)
        p = np.array([1 - DECIMAL_T[11]] + [DECIMAL_T[m] - DECIMAL_T[m - 1] for m in range(1, 12)])
        assert abs(float((p * num).sum()) - MEAN_NUCS[n_nuc]) < 1e-3
