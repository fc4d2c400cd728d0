"""CPU oracle for the XSBench-style macroscopic cross-section lookup.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` leg may import this package.
The product package never imports it and shares no code with it.

This module is argument marshalling around ``xs_oracle.c`` (plain C, built with
``gcc -O2 -ffp-contract=off -fopenmp``); every step of the arithmetic lives there,
each function citing the PAPER.md passage or DESIGN.md reading it follows.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "xs_oracle.c")
_SRCS = [_SRC, os.path.join(_HERE, "bezier_oracle.c")]
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

UNIONIZED, NUCLIDE, HASH = 0, 1, 2
HASH_BINS = 10000


def build(force: bool = False) -> str:
    """Compile oracle/liboracle.so (plain C, no CUDA)."""
    if force or not os.path.exists(_LIB) or any(os.path.getmtime(_LIB) < os.path.getmtime(s) for s in _SRCS):
        cmd = ["gcc", "-O2", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared",
               "-std=c99", "-Wall", "-o", _LIB + ".tmp", *_SRCS, "-lm"]
        subprocess.run(cmd, check=True)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


class _Problem(C.Structure):
    _fields_ = [
        ("n_nuc", C.c_int64), ("n", C.c_int64),
        ("E", C.c_void_p), ("X", C.c_void_p),
        ("grid_type", C.c_int32), ("search_mode", C.c_int32),
        ("U", C.c_void_p), ("IDX", C.c_void_p),
        ("bins", C.c_int64), ("H", C.c_void_p),
        ("num_nucs", C.c_void_p), ("mats", C.c_void_p), ("concs", C.c_void_p),
        ("max_nucs", C.c_int32), ("pad_", C.c_int32),
    ]


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = C.CDLL(_LIB)
            u64, i64, i32, dbl, vp = C.c_uint64, C.c_int64, C.c_int32, C.c_double, C.c_void_p
            sig = {
                "or_lcg_step": (u64, [u64]),
                "or_skip": (u64, [u64, u64]),
                "or_u63_to_double": (dbl, [u64]),
                "or_draw": (dbl, [u64, u64]),
                "or_mat_num_nucs": (i32, [i64, vp]),
                "or_mat_table": (C.c_int, [i64, vp]),
                "or_concs": (None, [u64, i64, vp, i32, vp]),
                "or_pick_mat": (i32, [dbl]),
                "or_pick_mat_thresholds": (None, [vp]),
                "or_search_listing1": (i64, [vp, i64, i64, dbl]),
                "or_search_listing1_trace": (i32, [vp, i64, i64, dbl, vp, i32, vp]),
                "or_search_def": (i64, [vp, i64, dbl]),
                "or_grid_nuclide": (C.c_int, [i64, i64, u64, vp, vp]),
                "or_grid_unionized": (None, [i64, i64, vp, vp, vp]),
                "or_grid_hash": (None, [i64, i64, vp, i64, vp]),
                "or_micro_xs": (None, [vp, i32, dbl, i64, vp]),
                "or_macro_xs": (None, [vp, i32, dbl, vp, vp]),
                "or_verify": (i32, [vp]),
                "or_sample": (None, [u64, i64, vp, vp]),
                "or_lookup": (i32, [vp, u64, i64, vp, vp, vp, vp]),
                "or_run_range": (C.c_int, [vp, u64, i64, i64, vp, vp, vp, vp, vp, vp, i32]),
                "or_run_indices": (C.c_int, [vp, u64, vp, i64, vp, vp, i32]),
                "or_max_threads": (i32, []),
                "ob_blend_loop_f64": (dbl, [C.c_int, C.c_int]),
                "ob_blend_loop_f32": (C.c_float, [C.c_int, C.c_int]),
                "ob_bezier_blend_f64": (dbl, [C.c_int, dbl, C.c_int]),
                "ob_bezier_blend_f32": (C.c_float, [C.c_int, C.c_float, C.c_int]),
                "ob_surface_f64": (None, [C.c_int, C.c_int, i64, i64, vp, vp]),
                "ob_surface_f32": (None, [C.c_int, C.c_int, i64, i64, vp, vp]),
                "ob_surface_points_f64": (None, [C.c_int, C.c_int, i64, i64, vp, i64, vp, vp, vp]),
                "ob_surface_points_f32": (None, [C.c_int, C.c_int, i64, i64, vp, i64, vp, vp, vp]),
            }
            for name, (res, args) in sig.items():
                f = getattr(L, name)
                f.restype = res
                f.argtypes = args
            _lib = L
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data


# ---------------------------------------------------------------- scalars
def lcg_step(s: int) -> int:
    return lib().or_lcg_step(s)


def skip(s: int, n: int) -> int:
    return lib().or_skip(s, n)


def u63_to_double(s: int) -> float:
    return lib().or_u63_to_double(s)


def draw(seed: int, t: int) -> float:
    return lib().or_draw(seed, t)


def pick_mat(roll: float) -> int:
    return lib().or_pick_mat(roll)


def pick_mat_thresholds() -> np.ndarray:
    T = np.zeros(12, np.float64)
    lib().or_pick_mat_thresholds(_p(T))
    return T


def sample(seed: int, i: int):
    q = C.c_double()
    m = C.c_int32()
    lib().or_sample(seed, i, C.byref(q), C.byref(m))
    return q.value, m.value


def verify(macro) -> int:
    m = np.ascontiguousarray(macro, np.float64)
    return lib().or_verify(_p(m))


def search_listing1(A: np.ndarray, lo: int, hi: int, q: float) -> int:
    A = np.ascontiguousarray(A, np.float64)
    return lib().or_search_listing1(_p(A), lo, hi, q)


def search_listing1_trace(A: np.ndarray, lo: int, hi: int, q: float):
    A = np.ascontiguousarray(A, np.float64)
    probes = np.zeros(128, np.int64)
    res = C.c_int64()
    n = lib().or_search_listing1_trace(_p(A), lo, hi, q, _p(probes), 128, C.byref(res))
    return res.value, probes[:n].tolist()


def search_def(A: np.ndarray, q: float) -> int:
    A = np.ascontiguousarray(A, np.float64)
    return lib().or_search_def(_p(A), len(A), q)


def materials(n_nuc: int):
    """(num_nucs[12] int32, mats[12][max] int32, max_nucs)"""
    num = np.zeros(12, np.int32)
    mx = lib().or_mat_num_nucs(n_nuc, _p(num))
    if mx < 0:
        raise ValueError(f"n_nuclides={n_nuc}: must be 68 or >= 355")
    mats = np.zeros((12, mx), np.int32)
    lib().or_mat_table(n_nuc, _p(mats))
    return num, mats, mx


# ---------------------------------------------------------------- problems
class Problem:
    """A complete lookup problem held in host numpy arrays.

    Build it from (n_nuc, n, grid_type, grid_seed) exactly as the method does, or
    pass explicit E / X / concs arrays (tests inject synthetic grids with closed-form
    channels)."""

    def __init__(self, n_nuc, n, grid_type=NUCLIDE, grid_seed=42, *, E=None, X=None,
                 concs=None, bins=HASH_BINS, build_idx=True, search_mode=0):
        L = lib()
        self.n_nuc, self.n, self.grid_type, self.grid_seed = int(n_nuc), int(n), int(grid_type), grid_seed
        self.num_nucs, self.mats, self.max_nucs = materials(n_nuc)
        N = self.n_nuc * self.n
        if E is None:
            self.E = np.empty((n_nuc, n), np.float64)
            self.X = np.empty((n_nuc, n, 5), np.float64)
            rc = L.or_grid_nuclide(n_nuc, n, grid_seed, _p(self.E), _p(self.X))
            if rc != 0:
                raise ValueError("duplicate energy within a nuclide (XS_EDUP)")
        else:
            self.E = np.ascontiguousarray(E, np.float64).reshape(n_nuc, n)
            self.X = np.ascontiguousarray(X, np.float64).reshape(n_nuc, n, 5)
        if concs is None:
            self.concs = np.zeros((12, self.max_nucs), np.float64)
            L.or_concs(grid_seed, N, _p(self.num_nucs), self.max_nucs, _p(self.concs))
        else:
            self.concs = np.ascontiguousarray(concs, np.float64).reshape(12, self.max_nucs)
        self.U = self.IDX = self.H = None
        self.bins = int(bins)
        if grid_type == UNIONIZED:
            self.U = np.empty(N, np.float64)
            if build_idx:
                self.IDX = np.empty((N, n_nuc), np.int32)
            L.or_grid_unionized(n_nuc, n, _p(self.E), _p(self.U), _p(self.IDX))
        elif grid_type == HASH:
            self.H = np.empty((self.bins, n_nuc), np.int32)
            L.or_grid_hash(n_nuc, n, _p(self.E), self.bins, _p(self.H))
        self.search_mode = search_mode
        self._mk()

    def _mk(self):
        self._s = _Problem(self.n_nuc, self.n, _p(self.E), _p(self.X), self.grid_type,
                           self.search_mode, _p(self.U), _p(self.IDX), self.bins, _p(self.H),
                           _p(self.num_nucs), _p(self.mats), _p(self.concs), self.max_nucs, 0)

    def with_search_mode(self, mode: int) -> "Problem":
        self.search_mode = mode
        self._mk()
        return self

    # --- per-lookup pieces
    def micro_xs(self, nuc: int, q: float, L: int) -> np.ndarray:
        out = np.zeros(5, np.float64)
        lib().or_micro_xs(C.byref(self._s), nuc, q, L, _p(out))
        return out

    def macro_xs(self, mat: int, q: float):
        out = np.zeros(5, np.float64)
        Ls = np.full(self.max_nucs, -1, np.int32)
        lib().or_macro_xs(C.byref(self._s), mat, q, _p(out), _p(Ls))
        return out, Ls[: self.num_nucs[mat]]

    def lookup(self, seed: int, i: int):
        out = np.zeros(5, np.float64)
        mat, q = C.c_int32(), C.c_double()
        Ls = np.full(self.max_nucs, -1, np.int32)
        v = lib().or_lookup(C.byref(self._s), seed, i, _p(out), C.byref(mat), C.byref(q), _p(Ls))
        return v, out, mat.value, q.value, Ls

    def run_range(self, seed: int, first: int, count: int, *, macro=True, mat=False, q=False,
                  idx=False, threads: int = 0):
        """Returns dict(hash, pairs, macro?, mat?, q?, idx?)."""
        res = {}
        om = np.empty((count, 5), np.float64) if macro else None
        omat = np.empty(count, np.int32) if mat else None
        oq = np.empty(count, np.float64) if q else None
        oL = np.empty((count, self.max_nucs), np.int32) if idx else None
        h, pr = C.c_uint64(), C.c_uint64()
        lib().or_run_range(C.byref(self._s), seed, first, count, _p(om), _p(omat), _p(oq), _p(oL),
                           C.byref(h), C.byref(pr), threads)
        res["hash"], res["pairs"] = h.value, pr.value
        for k, v in (("macro", om), ("mat", omat), ("q", oq), ("idx", oL)):
            if v is not None:
                res[k] = v
        return res

    def run_indices(self, seed: int, indices, threads: int = 0):
        idx = np.ascontiguousarray(indices, np.int64)
        om = np.empty((len(idx), 5), np.float64)
        h = C.c_uint64()
        lib().or_run_indices(C.byref(self._s), seed, _p(idx), len(idx), _p(om), C.byref(h), threads)
        return h.value, om


def max_threads() -> int:
    return lib().or_max_threads()


# ---------------------------------------------------------------- bezier-surface (Listing 2)
def blend_loop(k: int, n: int, dtype=np.float64) -> float:
    """Listing 2 from blend = 1 (reading BZ1)."""
    f = lib().ob_blend_loop_f64 if np.dtype(dtype) == np.float64 else lib().ob_blend_loop_f32
    return f(k, n)


def bezier_blend(k: int, mu: float, n: int, dtype=np.float64) -> float:
    """Listing 2 times mu^k (1-mu)^(n-k) (reading BZ2)."""
    f = lib().ob_bezier_blend_f64 if np.dtype(dtype) == np.float64 else lib().ob_bezier_blend_f32
    return f(k, mu, n)


def bezier_surface(P: np.ndarray, res_i: int, res_j: int) -> np.ndarray:
    """The surface (readings BZ3-BZ5) over the control net P[(ni+1), (nj+1), 3] in P's dtype."""
    P = np.ascontiguousarray(P)
    ni, nj = P.shape[0] - 1, P.shape[1] - 1
    out = np.zeros((res_i, res_j, 3), P.dtype)
    f = lib().ob_surface_f64 if P.dtype == np.float64 else lib().ob_surface_f32
    f(ni, nj, res_i, res_j, _p(P), _p(out))
    return out


def bezier_surface_points(P: np.ndarray, res_i: int, res_j: int, ii, jj) -> np.ndarray:
    """surface(ii[t], jj[t]) for sampled points of a res_i x res_j surface."""
    P = np.ascontiguousarray(P)
    ii = np.ascontiguousarray(ii, np.int64)
    jj = np.ascontiguousarray(jj, np.int64)
    ni, nj = P.shape[0] - 1, P.shape[1] - 1
    out = np.zeros((len(ii), 3), P.dtype)
    f = lib().ob_surface_points_f64 if P.dtype == np.float64 else lib().ob_surface_points_f32
    f(ni, nj, res_i, res_j, _p(P), len(ii), _p(ii), _p(jj), _p(out))
    return out
