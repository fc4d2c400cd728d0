"""Chunk boundaries: with XS_TEST_MAX_CHUNK forcing many internal passes, every pipeline and
output kind (device, pinned host, pageable host, indices) must match the oracle exactly."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r"""
import sys; sys.path.insert(0, %r)
import numpy as np, torch
import oracle
import paper_conf_cgo_murtovigplls24_b200 as xs
P = oracle.Problem(68, 1000, 1, 42)
first, count = 777, 23_456
ref = P.run_range(1070, first, count, idx=True)
with xs.Grid(68, 1000, 1, 42) as g:
    for sort, split in (("none", False), ("material_energy", False), ("material_energy", True), ("history", False)):
        for search in ("M", "U2", "W", "H", "S"):
            out, st = g.macro_xs(first, count, 1070, search=search, sort=sort, split=split, history_len=34)
            assert st.hash == ref["hash"] and st.pairs == ref["pairs"], (sort, split, search)
            assert np.array_equal(out.cpu().numpy(), ref["macro"]), (sort, split, search)
            idx = g.indices(first, count, 1070, search=search, sort=sort, split=split, history_len=34)
            assert np.array_equal(idx.cpu().numpy(), ref["idx"]), (sort, split, search)
        pinned = torch.empty((count, 5), dtype=torch.float64).pin_memory()
        g.lookup_range(first, count, 1070, pinned, sort=sort, split=split, history_len=34)
        assert np.array_equal(pinned.numpy(), ref["macro"]), sort
        pageable = np.zeros((count, 5))
        g.lookup_range(first, count, 1070, pageable, sort=sort, split=split, history_len=34)
        assert np.array_equal(pageable, ref["macro"]), sort
print("CHUNKS OK")
""" % ROOT


@pytest.mark.parametrize("chunk", [1000, 4099])
def test_many_chunks_match_oracle(chunk):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    env = dict(os.environ, XS_TEST_MAX_CHUNK=str(chunk))
    r = subprocess.run([sys.executable, "-c", SCRIPT], capture_output=True, text=True, env=env, timeout=900)
    assert r.returncode == 0 and "CHUNKS OK" in r.stdout, (r.stdout[-2000:], r.stderr[-3000:])


WINDOW_SCRIPT = r"""
import sys; sys.path.insert(0, %r)
import numpy as np
import oracle
import paper_conf_cgo_murtovigplls24_b200 as xs
for gt in (0, 1, 2):
    P = oracle.Problem(68, 1000, gt, 42)
    ref = P.run_range(1070, 5, 100_000, idx=True)
    with xs.Grid(68, 1000, gt, 42) as g:
        for search in ("H", "S"):
            for coarse in (False, True):
                out, st = g.macro_xs(5, 100_000, 1070, search=search, coarse=coarse)
                assert st.hash == ref["hash"] and st.pairs == ref["pairs"], (gt, search, coarse)
                assert np.array_equal(out.cpu().numpy(), ref["macro"]), (gt, search, coarse)
                idx = g.indices(5, 100_000, 1070, search=search, coarse=coarse)
                assert np.array_equal(idx.cpu().numpy(), ref["idx"]), (gt, search, coarse)
print("WINDOWS OK")
""" % ROOT


@pytest.mark.parametrize("zero", [False, True])
@pytest.mark.parametrize("windows", [1, 2, 7, 39])
def test_scatter_windows_match_oracle(windows, zero):
    """the windowed scatter (one launch per window of buckets) with the window count forced
    (XS_TEST_SCATTER_WINDOWS): every bucket is written by exactly one window; zero: each window
    pre-zeroed first (k_zero_window, on by size for large sort chunks; XS_TEST_SCATTER_ZERO
    forces it here, including windows whose slot range is not 16 B aligned)"""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    env = dict(os.environ, XS_TEST_SCATTER_WINDOWS=str(windows))
    if zero:
        env["XS_TEST_SCATTER_ZERO"] = "1"
    r = subprocess.run([sys.executable, "-c", WINDOW_SCRIPT], capture_output=True, text=True, env=env, timeout=900)
    assert r.returncode == 0 and "WINDOWS OK" in r.stdout, (r.stdout[-2000:], r.stderr[-3000:])
