"""B200-native XSBench-style macroscopic cross-section lookup (CGO'24 u&u motivating kernel).

The product is libxs.so (CUDA for sm_100a behind the C ABI in include/xs.h).  This
package is its thin Python face: ``_xs`` binds the C entry points by name, ``Grid``
owns a grid handle, ``driver`` shards lookups over ranks.  PyTorch supplies device
memory, streams and process groups only.
"""
from __future__ import annotations

from ._xs import (  # noqa: F401  (the C names)
    SEARCH_NAMES, SORT_NAMES, XS_ECUDA, XS_EDUP, XS_EINVAL, XS_ENOMEM, XS_FLAG_SPLIT, XS_FLAG_TIMING, XS_HASH, XS_NUCLIDE, XS_OK,
    XS_SEARCH_B, XS_SEARCH_COUNT, XS_SEARCH_M, XS_SEARCH_M2, XS_SEARCH_M4, XS_SEARCH_M8, XS_SEARCH_U1,
    XS_SEARCH_U2, XS_SEARCH_U4, XS_SEARCH_U8, XS_SEARCH_W, XS_SEARCH_H, XS_SEARCH_S, XS_SORT_HISTORY, XS_SORT_MATERIAL, XS_SORT_MATERIAL_ENERGY, XS_SORT_NONE,
    XS_UNIONIZED, LIB_PATH, XSError, xs_grid_checksum, xs_grid_create, xs_grid_destroy, xs_grid_export,
    xs_grid_export_aux, xs_grid_get_info, xs_last_error, xs_lookup_batch, xs_lookup_indices, xs_lookup_range,
    xs_opts, xs_opts_default, xs_sample, xs_search_points, xs_stats,
    BZ_NAMES, XS_BZ_COUNT, XS_BZ_M, XS_BZ_M2, XS_BZ_S, XS_BZ_T, XS_BZ_U1, XS_BZ_U2, XS_F32, XS_F64,
    xs_bezier_blend, xs_bezier_surface)
from .grid import Grid, make_opts  # noqa: F401
from .bezier import bezier_blend, bezier_surface  # noqa: F401
