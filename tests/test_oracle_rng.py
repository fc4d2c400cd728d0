"""Pins for the oracle's LCG, skip-ahead (Listing 7) and u63 -> double conversion.

Everything here is checked against Python big-integer arithmetic (brute force),
never against the oracle itself."""
import random

import pytest

M = 2 ** 63
A = 2806196910506780709
Cc = 1


def py_step(s):
    return (A * s + Cc) % M


def py_steps(s, n):
    for _ in range(n):
        s = py_step(s)
    return s


def test_lcg_full_period_conditions():
    # Hull-Dobell for m = 2^63: c odd, a = 1 mod 4 -> full period 2^63.
    assert Cc % 2 == 1 and A % 4 == 1


@pytest.mark.parametrize("seed", [0, 1, 42, 1070, M - 1, 0x123456789ABCDEF])
def test_step_matches_bigint(oracle_mod, seed):
    s = seed
    for _ in range(50):
        assert oracle_mod.lcg_step(s) == py_step(s)
        s = py_step(s)


@pytest.mark.parametrize("seed", [0, 42, 1070, M - 1])
def test_skip_equals_sequential_steps(oracle_mod, seed):
    # Listing 7 loop must equal n sequential steps.
    s = seed
    for n in range(0, 2000):
        assert oracle_mod.skip(seed, n) == s, n
        s = py_step(s)


def test_skip_large_n_and_additivity(oracle_mod):
    rng = random.Random(7)
    s0 = 42
    # brute force up to 1e5 steps
    seq = py_steps(s0, 100_000)
    assert oracle_mod.skip(s0, 100_000) == seq
    for _ in range(200):
        a = rng.randrange(0, 2 ** 40)
        b = rng.randrange(0, 2 ** 40)
        assert oracle_mod.skip(oracle_mod.skip(s0, a), b) == oracle_mod.skip(s0, a + b)
    assert oracle_mod.skip(12345, 0) == 12345
    # the period divides 2^63: skipping 2^63 is the identity
    assert oracle_mod.skip(987654321, 2 ** 63) == 987654321


def test_u63_to_double_correctly_rounded(oracle_mod):
    rng = random.Random(3)
    cases = [0, 1, 2 ** 52, 2 ** 53 + 1, 2 ** 62, M - 1, M - 512, M - 513, M - 511]
    cases += [rng.randrange(0, M) for _ in range(5000)]
    for s in cases:
        # Python's int -> float is correctly rounded (nearest, ties to even)
        assert oracle_mod.u63_to_double(s) == float(s) / 2.0 ** 63, s


def test_draw_can_round_to_one(oracle_mod):
    # reading R7: s >= 2^63 - 512 rounds to exactly 1.0
    assert oracle_mod.u63_to_double(M - 1) == 1.0
    assert oracle_mod.u63_to_double(M - 512) == 1.0
    assert oracle_mod.u63_to_double(M - 513) < 1.0


def test_draw_position_semantics(oracle_mod):
    # value at position t = step(skip(seed, t)) / 2^63
    for t in [0, 1, 5, 6, 1000]:
        s = py_steps(42, t + 1)
        assert oracle_mod.draw(42, t) == float(s) / 2.0 ** 63


def test_sample_definition(oracle_mod):
    # lookup i: q at position 2i, roll at 2i+1 of the lookup stream
    from xs_workloads import LOOKUP_SEED
    T = oracle_mod.pick_mat_thresholds()
    for i in [0, 1, 2, 17, 99_999]:
        s = py_steps(LOOKUP_SEED, 2 * i + 1)
        q = float(s) / 2.0 ** 63
        r = float(py_step(s)) / 2.0 ** 63
        mat = 0
        for m in range(1, 12):
            if r < T[m]:
                mat = m
                break
        assert oracle_mod.sample(LOOKUP_SEED, i) == (q, mat)
