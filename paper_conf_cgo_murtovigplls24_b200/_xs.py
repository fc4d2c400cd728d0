"""ctypes binding of libxs.so -- argument marshalling only.

Every function here has the name of the C entry point it wraps (include/xs.h) and
does nothing but convert arguments; every step of the lookup path runs in the CUDA
kernels of libxs.so.  There is no fallback: if the library is missing, importing this
module raises.
"""
from __future__ import annotations

import ctypes as C
import os
import re

_HERE = os.path.dirname(os.path.abspath(__file__))
# XS_LIB_VARIANT selects an experimental build (libxs_<variant>.so) for A/B probes only
LIB_PATH = os.path.join(_HERE, "libxs.so" if not os.environ.get("XS_LIB_VARIANT")
                        else f"libxs_{os.environ['XS_LIB_VARIANT']}.so")
HEADER_PATH = os.path.join(os.path.dirname(_HERE), "include", "xs.h")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
        "(there is no CPU fallback)")

_lib = C.CDLL(LIB_PATH)

XS_UNIONIZED, XS_NUCLIDE, XS_HASH = 0, 1, 2
XS_OK, XS_EINVAL, XS_ENOMEM, XS_ECUDA, XS_EDUP = 0, -1, -2, -3, -4
(XS_SEARCH_M, XS_SEARCH_U1, XS_SEARCH_U2, XS_SEARCH_U4, XS_SEARCH_U8, XS_SEARCH_B,
 XS_SEARCH_M2, XS_SEARCH_M4, XS_SEARCH_M8, XS_SEARCH_W, XS_SEARCH_H, XS_SEARCH_S) = range(12)
XS_SEARCH_COUNT = 12
XS_SORT_NONE, XS_SORT_MATERIAL, XS_SORT_MATERIAL_ENERGY, XS_SORT_HISTORY = 0, 1, 2, 3
XS_FLAG_TIMING = 1
XS_FLAG_SPLIT = 2
XS_FLAG_COARSE = 4

SEARCH_NAMES = {"M": 0, "U1": 1, "U2": 2, "U4": 3, "U8": 4, "B": 5, "M2": 6, "M4": 7, "M8": 8, "W": 9, "H": 10, "S": 11}
SORT_NAMES = {"none": 0, "material": 1, "material_energy": 2, "history": 3}
XS_BZ_M, XS_BZ_M2, XS_BZ_U1, XS_BZ_U2, XS_BZ_S, XS_BZ_T = range(6)
XS_BZ_COUNT = 6
XS_F64, XS_F32 = 0, 1
BZ_NAMES = {"M": 0, "M2": 1, "U1": 2, "U2": 3, "S": 4, "T": 5}


class xs_opts(C.Structure):
    _fields_ = [("search", C.c_int32), ("sort", C.c_int32), ("stream", C.c_void_p),
                ("block", C.c_int32), ("energy_bins", C.c_int32), ("flags", C.c_uint32),
                ("history_len", C.c_int32), ("shard_index", C.c_int32), ("shard_count", C.c_int32)]


class xs_stats(C.Structure):
    _fields_ = [("hash", C.c_uint64), ("lookups", C.c_uint64), ("pairs", C.c_uint64),
                ("device_ms", C.c_double), ("sample_ms", C.c_double), ("lookup_ms", C.c_double),
                ("search_ms", C.c_double), ("copy_ms", C.c_double), ("launches", C.c_int32),
                ("reserved", C.c_int32)]


class xs_grid_info(C.Structure):
    _fields_ = [("n_nuclides", C.c_int64), ("n_gridpoints", C.c_int64), ("n_points", C.c_int64),
                ("hash_bins", C.c_int64), ("seed", C.c_uint64), ("device_bytes", C.c_uint64),
                ("grid_type", C.c_int32), ("device", C.c_int32), ("max_num_nucs", C.c_int32),
                ("num_nucs", C.c_int32 * 12)]


_vp, _i64, _u64, _i32 = C.c_void_p, C.c_int64, C.c_uint64, C.c_int32
_SIGS = {
    "xs_opts_default": (None, [C.POINTER(xs_opts)]),
    "xs_grid_create": (_vp, [_i64, _i64, C.c_int, _u64]),
    "xs_grid_create_ex": (_vp, [_i64, _i64, C.c_int, _u64, _i64]),
    "xs_grid_destroy": (None, [_vp]),
    "xs_last_error": (C.c_char_p, []),
    "xs_lookup_batch": (C.c_int, [_vp, _i64, _u64, _vp, C.POINTER(_u64)]),
    "xs_lookup_range": (C.c_int, [_vp, _i64, _i64, _u64, C.POINTER(xs_opts), _vp, C.POINTER(xs_stats)]),
    "xs_lookup_indices": (C.c_int, [_vp, _i64, _i64, _u64, C.POINTER(xs_opts), _vp]),
    "xs_sample": (C.c_int, [_vp, _i64, _i64, _u64, _vp, _vp, _vp]),
    "xs_search_points": (C.c_int, [_vp, _i64, _vp, _vp, _i32, _vp, _vp]),
    "xs_grid_checksum": (C.c_int, [_vp, C.POINTER(_u64)]),
    "xs_grid_get_info": (C.c_int, [_vp, C.POINTER(xs_grid_info)]),
    "xs_grid_export": (C.c_int, [_vp, _vp, _vp, _vp, _vp]),
    "xs_grid_export_aux": (C.c_int, [_vp, _vp, _vp, _vp]),
    "xs_bezier_surface": (C.c_int, [_i32, _i32, _i64, _i64, _i32, _i32, _vp, _vp, _vp]),
    "xs_bezier_blend": (C.c_int, [_i64, _vp, _vp, _vp, _i32, _i32, _vp, _vp]),
}
for _name, (_res, _args) in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args


def header_functions() -> list[str]:
    """Every function the public header declares (for the export test)."""
    text = open(HEADER_PATH).read()
    return sorted(set(re.findall(r"\b(xs_[a-z_]+)\s*\(", text)) - {"xs_grid", "xs_opts", "xs_stats"})


class XSError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"libxs error {code}: {msg}")
        self.code = code


def _check(rc: int):
    if rc != XS_OK:
        raise XSError(rc, (_lib.xs_last_error() or b"").decode())


def _ptr(x):
    """A device/host address from a torch tensor, numpy array, int or None."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if hasattr(x, "ctypes"):
        return x.ctypes.data
    raise TypeError(type(x))


# ---------------------------------------------------------------- the C names
def xs_opts_default() -> xs_opts:
    o = xs_opts()
    _lib.xs_opts_default(C.byref(o))
    return o


def xs_grid_create(n_nuclides: int, n_gridpoints: int, grid_type: int, seed: int, hash_bins: int = 10000) -> int:
    h = _lib.xs_grid_create_ex(n_nuclides, n_gridpoints, grid_type, seed, hash_bins)
    if not h:
        raise XSError(-1, (_lib.xs_last_error() or b"").decode())
    return h


def xs_grid_destroy(grid: int) -> None:
    _lib.xs_grid_destroy(grid)


def xs_last_error() -> str:
    return (_lib.xs_last_error() or b"").decode()


def xs_lookup_batch(grid: int, n_lookups: int, seed: int, out_macro_xs=None) -> int:
    h = _u64()
    _check(_lib.xs_lookup_batch(grid, n_lookups, seed, _ptr(out_macro_xs), C.byref(h)))
    return h.value


def xs_lookup_range(grid: int, first: int, count: int, seed: int, opts: xs_opts | None = None,
                    out_macro_xs=None) -> xs_stats:
    st = xs_stats()
    _check(_lib.xs_lookup_range(grid, first, count, seed, C.byref(opts) if opts is not None else None,
                                _ptr(out_macro_xs), C.byref(st)))
    return st


def xs_lookup_indices(grid: int, first: int, count: int, seed: int, opts: xs_opts | None, out_idx) -> None:
    _check(_lib.xs_lookup_indices(grid, first, count, seed, C.byref(opts) if opts is not None else None,
                                  _ptr(out_idx)))


def xs_sample(grid: int, first: int, count: int, seed: int, out_q, out_mat, stream: int | None = None) -> None:
    _check(_lib.xs_sample(grid, first, count, seed, _ptr(out_q), _ptr(out_mat), stream))


def xs_search_points(grid: int, count: int, q, nuc, search: int, out_L, stream: int | None = None) -> None:
    _check(_lib.xs_search_points(grid, count, _ptr(q), _ptr(nuc), search, _ptr(out_L), stream))


def xs_grid_checksum(grid: int) -> int:
    h = _u64()
    _check(_lib.xs_grid_checksum(grid, C.byref(h)))
    return h.value


def xs_grid_get_info(grid: int) -> xs_grid_info:
    info = xs_grid_info()
    _check(_lib.xs_grid_get_info(grid, C.byref(info)))
    return info


def xs_grid_export(grid: int, E=None, X=None, mats=None, concs=None) -> None:
    _check(_lib.xs_grid_export(grid, _ptr(E), _ptr(X), _ptr(mats), _ptr(concs)))


def xs_grid_export_aux(grid: int, U=None, IDX=None, H=None) -> None:
    _check(_lib.xs_grid_export_aux(grid, _ptr(U), _ptr(IDX), _ptr(H)))


def xs_bezier_surface(ni: int, nj: int, res_i: int, res_j: int, dtype: int, variant: int, ctrl, out,
                      stream: int | None = None) -> None:
    _check(_lib.xs_bezier_surface(ni, nj, res_i, res_j, dtype, variant, _ptr(ctrl), _ptr(out), stream))


def xs_bezier_blend(count: int, k, n, mu, dtype: int, variant: int, out, stream: int | None = None) -> None:
    _check(_lib.xs_bezier_blend(count, _ptr(k), _ptr(n), _ptr(mu), dtype, variant, _ptr(out), stream))
