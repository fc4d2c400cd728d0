"""Out-of-bounds writes into the caller's buffers, checked without compute-sanitizer (closed on
the GPU pool, see test_gpu_sanitizer.py): every output buffer is the middle of a larger
allocation whose guard regions hold a sentinel bit pattern.  After each call the guards must
be untouched and every output element written (no sentinel left), for every grid type,
pipeline and search variant, at ragged counts (1, a warp +- 1, a partial count tile, a
partial sort bucket group) and ranges that start mid-stream."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

GUARD = 4099                          # rows of guard on each side (not a multiple of any tile)
SENT = np.int64(0x7FF4DEADBEEF1234)   # a signalling-NaN payload no kernel produces


def _guarded(torch, rows, cols, dtype):
    n = (rows + 2 * GUARD) * cols
    if dtype == torch.float64:
        buf = torch.full((n,), 0, dtype=torch.int64, device="cuda")
        buf.fill_(int(SENT))
        full = buf.view(torch.float64).view(rows + 2 * GUARD, cols)
    else:
        full = torch.full((rows + 2 * GUARD, cols), -7, dtype=dtype, device="cuda")
    return full, full[GUARD:GUARD + rows]


def _check(torch, full, rows, dtype):
    if dtype == torch.float64:
        bits = full.view(torch.int64).cpu().numpy()
        head, body, tail = bits[:GUARD], bits[GUARD:GUARD + rows], bits[GUARD + rows:]
        assert (head == SENT).all() and (tail == SENT).all(), "write outside the output buffer"
        assert not (body == SENT).any(), "output element not written"
    else:
        a = full.cpu().numpy()
        head, tail = a[:GUARD], a[GUARD + rows:]
        assert (head == -7).all() and (tail == -7).all(), "write outside the index buffer"


@pytest.fixture(scope="module")
def grids():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_cgo_murtovigplls24_b200 as xs
    gs = {gt: xs.Grid(68, 200, gt, 42) for gt in (xs.XS_UNIONIZED, xs.XS_NUCLIDE, xs.XS_HASH)}
    yield gs
    for g in gs.values():
        g.close()


PIPES = [dict(sort="none"), dict(sort="material_energy"), dict(sort="material_energy", split=True),
         dict(sort="material_energy", coarse=True), dict(sort="history", history_len=7)]


@pytest.mark.parametrize("count", [1, 31, 33, 4097, 100_003])
@pytest.mark.parametrize("gt", [0, 1, 2])
def test_macro_xs_writes_stay_inside(grids, gt, count):
    import torch
    g = grids[gt]
    for pipe in PIPES:
        for search in ("M", "U2", "W", "H", "S"):
            full, out = _guarded(torch, count, 5, torch.float64)
            g.lookup_range(12345, count, 1070, out, search=search, **pipe)
            torch.cuda.synchronize()
            _check(torch, full, count, torch.float64)


@pytest.mark.parametrize("count", [1, 33, 4097])
@pytest.mark.parametrize("gt", [0, 1, 2])
def test_index_writes_stay_inside(grids, gt, count):
    import torch
    import paper_conf_cgo_murtovigplls24_b200 as xs
    g = grids[gt]
    for pipe in PIPES:
        for search in ("U2", "S"):
            full, out = _guarded(torch, count, g.max_nucs, torch.int32)
            xs.xs_lookup_indices(g.handle, 777, count, 1070, xs.make_opts(search=search, **pipe), out)
            torch.cuda.synchronize()
            _check(torch, full, count, torch.int32)


def test_host_outputs_stay_inside(grids):
    """pinned host output (the chunked D2H staging path) with guards"""
    import torch
    g = grids[1]
    count = 50_001
    buf = torch.empty(((count + 2 * GUARD) * 5,), dtype=torch.int64).pin_memory()
    buf.fill_(int(SENT))
    full = buf.view(torch.float64).view(count + 2 * GUARD, 5)
    g.lookup_range(3, count, 1070, full[GUARD:GUARD + count], search="S")
    bits = full.view(torch.int64).numpy()
    assert (bits[:GUARD] == SENT).all() and (bits[GUARD + count:] == SENT).all()
    assert not (bits[GUARD:GUARD + count] == SENT).any()
