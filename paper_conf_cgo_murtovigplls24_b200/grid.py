"""Grid: an owned xs_grid handle with torch-tensor conveniences (marshalling only)."""
from __future__ import annotations

import numpy as np
import torch

from . import _xs


def make_opts(search="S", sort="material_energy", stream=None, block=0, energy_bins=0, timing=False,
              split=False, history_len=0, coarse=False, shard=(0, 1)):
    o = _xs.xs_opts_default()
    o.search = _xs.SEARCH_NAMES[search] if isinstance(search, str) else int(search)
    o.sort = _xs.SORT_NAMES[sort] if isinstance(sort, str) else int(sort)
    if stream is None and torch.cuda.is_available():
        stream = torch.cuda.current_stream().cuda_stream
    o.stream = stream or None
    o.block = block
    o.energy_bins = energy_bins
    o.flags = ((_xs.XS_FLAG_TIMING if timing else 0) | (_xs.XS_FLAG_SPLIT if split else 0)
               | (_xs.XS_FLAG_COARSE if coarse else 0))
    o.history_len = history_len
    o.shard_index, o.shard_count = shard
    return o


class Grid:
    """A grid on the current CUDA device (xs_grid_create)."""

    def __init__(self, n_nuclides: int, n_gridpoints: int, grid_type: int = _xs.XS_NUCLIDE, seed: int = 42,
                 hash_bins: int = 10000):
        self.handle = _xs.xs_grid_create(n_nuclides, n_gridpoints, grid_type, seed, hash_bins)
        self.info = _xs.xs_grid_get_info(self.handle)
        self.n_nuclides, self.n_gridpoints, self.grid_type = n_nuclides, n_gridpoints, grid_type
        self.max_nucs = self.info.max_num_nucs
        self.device = torch.device("cuda", self.info.device)

    def close(self):
        if getattr(self, "handle", None):
            _xs.xs_grid_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # ---- hot path
    def lookup_range(self, first: int, count: int, seed: int, out=None, **opt) -> _xs.xs_stats:
        return _xs.xs_lookup_range(self.handle, first, count, seed, make_opts(**opt), out)

    def lookup_batch(self, n: int, seed: int, out=None) -> int:
        return _xs.xs_lookup_batch(self.handle, n, seed, out)

    def macro_xs(self, first: int, count: int, seed: int, **opt):
        out = torch.empty((count, 5), dtype=torch.float64, device=self.device)
        st = self.lookup_range(first, count, seed, out, **opt)
        return out, st

    # ---- parity / debug
    def indices(self, first: int, count: int, seed: int, **opt) -> torch.Tensor:
        out = torch.empty((count, self.max_nucs), dtype=torch.int32, device=self.device)
        _xs.xs_lookup_indices(self.handle, first, count, seed, make_opts(**opt), out)
        return out

    def sample(self, first: int, count: int, seed: int):
        q = torch.empty(count, dtype=torch.float64, device=self.device)
        m = torch.empty(count, dtype=torch.int32, device=self.device)
        _xs.xs_sample(self.handle, first, count, seed, q, m, torch.cuda.current_stream().cuda_stream)
        return q, m

    def search_points(self, q, nuc, search="U2") -> torch.Tensor:
        q = torch.as_tensor(q, dtype=torch.float64, device=self.device).contiguous()
        nuc = torch.as_tensor(nuc, dtype=torch.int32, device=self.device).contiguous()
        out = torch.empty(q.numel(), dtype=torch.int32, device=self.device)
        s = _xs.SEARCH_NAMES[search] if isinstance(search, str) else int(search)
        _xs.xs_search_points(self.handle, q.numel(), q, nuc, s, out, torch.cuda.current_stream().cuda_stream)
        return out

    def checksum(self) -> int:
        return _xs.xs_grid_checksum(self.handle)

    def export(self) -> dict:
        n, g, mx = self.n_nuclides, self.n_gridpoints, self.max_nucs
        E = np.empty((n, g), np.float64)
        X = np.empty((n, g, 5), np.float64)
        mats = np.empty((12, mx), np.int32)
        concs = np.empty((12, mx), np.float64)
        _xs.xs_grid_export(self.handle, E, X, mats, concs)
        d = {"E": E, "X": X, "mats": mats, "concs": concs,
             "num_nucs": np.array(list(self.info.num_nucs), np.int32)}
        if self.grid_type == _xs.XS_UNIONIZED:
            d["U"] = np.empty(n * g, np.float64)
            d["IDX"] = np.empty((n * g, n), np.int32)
            _xs.xs_grid_export_aux(self.handle, d["U"], d["IDX"], None)
        elif self.grid_type == _xs.XS_HASH:
            d["H"] = np.empty((self.info.hash_bins, n), np.int32)
            _xs.xs_grid_export_aux(self.handle, None, None, d["H"])
        return d
