"""Host transcription of search.cuh `search_K4` (the 4-ary window search of H and S, DESIGN.md
§6.5c), checked against the plain definition L(q) = clamp(#{k : A[k] <= q} - 1, lo, hi - 1)
on every window of small sorted rows (SURVEY.md §8c proof 1: Listing 1 returns exactly this
when A[lo] <= q < A[hi], or q >= A[hi] at the row's last index).  The device code is pinned
bit-exactly by the GPU parity tests; this pins the narrowing logic itself, including the
short windows where m1 == lower or m3 == m2."""
import numpy as np


def search_k4(A, lower, upper, q):
    while upper - lower > 1:
        m2 = lower + ((upper - lower) >> 1)
        m1 = lower + ((m2 - lower) >> 1)
        m3 = m2 + ((upper - m2) >> 1)
        e1, e2, e3 = A[m1], A[m2], A[m3]
        if e2 <= q:
            lower = m2
            if e3 <= q:
                lower = m3
            else:
                upper = m3
        else:
            upper = m2
            if e1 <= q:
                lower = m1
            else:
                upper = m1
    return lower


def test_k4_equals_definition_on_every_window():
    rng = np.random.default_rng(7)
    for n in (2, 3, 4, 5, 7, 16, 33):
        A = np.sort(rng.random(n))
        qs = np.concatenate([A, (A[:-1] + A[1:]) / 2, [A[0] - 1, A[-1] + 1]])
        for lo in range(n - 1):
            for hi in range(lo + 1, n):
                for q in qs:
                    inside = A[lo] <= q and (q < A[hi] or hi == n - 1)
                    if not inside:
                        continue  # the R7 guards send these to the full search
                    ub = int(np.searchsorted(A, q, side="right"))
                    want = min(max(ub - 1, lo), hi - 1)
                    assert search_k4(A, lo, hi, q) == want, (n, lo, hi, q)


def test_k4_terminates_outside_window():
    # q below A[lo]: the result is discarded by the caller, but the loop must end in range
    A = np.arange(10.0)
    for lo in range(9):
        for hi in range(lo + 1, 10):
            r = search_k4(A, lo, hi, -1.0)
            assert lo <= r <= hi
