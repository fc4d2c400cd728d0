"""CPU pin of the staged kernel's division (XS_SEARCH_S): Markstein's
quotient from a correctly rounded reciprocal equals IEEE division bit for bit on the inputs
the lookup meets (reading R8 keeps f = RN((E_hi - q) / (E_hi - E_lo)))."""
import os
import subprocess

import pytest

HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module")
def exe(tmp_path_factory):
    out = str(tmp_path_factory.mktemp("mk") / "markstein_check")
    subprocess.run(["gcc", "-O2", "-ffp-contract=off", "-o", out, os.path.join(HERE, "c", "markstein_check.c"),
                    "-lm"], check=True)
    return out


@pytest.mark.parametrize("seed", [1, 2, 3, 4])
def test_markstein_quotient_is_ieee_division(exe, seed):
    r = subprocess.run([exe, "5000000", str(seed)], capture_output=True, text=True, check=True)
    cases, bad = map(int, r.stdout.split())
    assert cases > 4_000_000
    assert bad == 0


def test_check_detects_a_wrong_quotient(exe, tmp_path):
    """the harness itself can fail: a plain product a * RN(1/d) is not correctly rounded"""
    src = open(os.path.join(HERE, "c", "markstein_check.c")).read()
    src = src.replace("const double f = fma(r, y, q0);", "const double f = q0; (void)r;")
    p = tmp_path / "wrong.c"
    p.write_text(src)
    out = str(tmp_path / "wrong")
    subprocess.run(["gcc", "-O2", "-ffp-contract=off", "-o", out, str(p), "-lm"], check=True)
    cases, bad = map(int, subprocess.run([out, "200000", "1"], capture_output=True, text=True,
                                         check=True).stdout.split())
    assert bad > 0
