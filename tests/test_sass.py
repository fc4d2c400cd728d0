"""The paper's A/B variants are control-flow shapes (Listings 4 and 5,
PAPER.md:354-452), and nvcc can undo them (round 1: the structured U1 came out of ptxas
if-converted to M's select form).  These tests read the SASS of the PRODUCTION lookup
kernels k_lookup<grid, search, sorted, outs=0, ilp2=0> in libxs.so (CPU only: cuobjdump) and
check, for every probe A[mid] of the search, what consumes its compare:

  M, M<k>, B   select form (Listing 4's selp): no branch on the probe result; M<k> has k
               probe copies per loop trip (unroll only)
  U1           unmerge only: a branch on the probe, 1 probe site, no select
  U<u>         unroll + unmerge: 2^u - 1 probe sites, every one a branch (each path its own
               back edge), the true-true guard `length >= 4` (as `len > 3` or `len >= 4`)
               and the `length >> 2` update of Listing 5
"""
import os

import pytest

from sass_shape import kernel_sass, mangled_k_lookup, shape

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_cgo_murtovigplls24_b200", "libxs.so")
SEARCH = {"M": 0, "U1": 1, "U2": 2, "U4": 3, "U8": 4, "B": 5, "M2": 6, "M4": 7, "M8": 8}
SITES = {"M": 1, "B": 1, "M2": 2, "M4": 4, "M8": 8, "U1": 1, "U2": 3, "U4": 15, "U8": 255}

pytestmark = pytest.mark.skipif(not os.path.exists(LIB), reason="libxs.so not built")


@pytest.mark.parametrize("sorted_", [True, False])
@pytest.mark.parametrize("grid", [1, 0])
@pytest.mark.parametrize("name", list(SEARCH))
def test_search_shape_in_k_lookup(name, grid, sorted_):
    sh = shape(kernel_sass(LIB, mangled_k_lookup(grid, SEARCH[name], sorted_)))
    assert sh["n_ins"] > 100, "kernel not found"
    assert sh["probes"] == SITES[name], sh
    if name.startswith("U"):
        assert sh["branch"] == sh["probes"] and sh["select"] == 0, sh
        assert sh["tt_guard"] >= 1, sh
        if name != "U1":
            assert sh["shr2"] >= SITES[name] // 4, sh
    else:
        assert sh["select"] == sh["probes"] and sh["branch"] == 0, sh
        assert sh["shr2"] == 0, sh


@pytest.mark.parametrize("name", list(SEARCH))
def test_search_shape_hash_grid(name):
    """hash grid: the window search and the R7 fallback search are two inlined copies, plus
    the two guard energies E[lo], E[hi] (consumed by the fallback branch)"""
    sh = shape(kernel_sass(LIB, mangled_k_lookup(2, SEARCH[name], True)))
    assert sh["probes"] == 2 * SITES[name] + 2, sh
    if name.startswith("U"):
        assert sh["branch"] == sh["probes"] and sh["select"] == 0, sh
    else:
        assert sh["select"] == 2 * SITES[name] and sh["branch"] == 2, sh


def test_u8_instruction_footprint():
    """u = 8: 255 probe copies -- the code-size cost the paper's heuristic bounds"""
    m = shape(kernel_sass(LIB, mangled_k_lookup(1, SEARCH["M"], True)))
    u8 = shape(kernel_sass(LIB, mangled_k_lookup(1, SEARCH["U8"], True)))
    assert u8["n_ins"] > 5 * m["n_ins"]
