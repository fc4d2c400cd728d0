"""The C structs of include/xs.h and their ctypes mirrors in the Python binding agree field by
field (offset and size): a C program compiled against the header prints its layout, and the
binding's Structure classes must match it.  A drifted field (the xs_opts shard fields were
appended in round 2) would otherwise pass garbage options silently."""
import ctypes
import os
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

STRUCTS = {
    "xs_opts": ["search", "sort", "stream", "block", "energy_bins", "flags", "history_len", "shard_index",
                "shard_count"],
    "xs_stats": ["hash", "lookups", "pairs", "device_ms", "sample_ms", "lookup_ms", "search_ms", "copy_ms",
                 "launches", "reserved"],
}


def _c_layout(tmp_path):
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "xs.h"', "int main(void) {"]
    for s, fields in STRUCTS.items():
        lines.append(f'printf("{s} %zu\\n", sizeof({s}));')
        for f in fields:
            lines.append(f'printf("{s}.{f} %zu %zu\\n", offsetof({s}, {f}), sizeof((({s} *)0)->{f}));')
    lines.append("return 0; }")
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    r = subprocess.run(["gcc", "-std=c99", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)],
                       capture_output=True, text=True)
    if r.returncode != 0:
        pytest.skip("gcc cannot compile against xs.h here: " + r.stderr[-300:])
    out = subprocess.run([str(exe)], capture_output=True, text=True, check=True).stdout
    lay = {}
    for line in out.splitlines():
        k, *v = line.split()
        lay[k] = tuple(int(x) for x in v)
    return lay


def test_struct_layouts_match_the_header(tmp_path):
    from paper_conf_cgo_murtovigplls24_b200 import _xs
    lay = _c_layout(tmp_path)
    for s, fields in STRUCTS.items():
        cls = getattr(_xs, s)
        assert ctypes.sizeof(cls) == lay[s][0], s
        names = [f[0] for f in cls._fields_]
        assert names == fields, (s, names)
        for f in fields:
            d = getattr(cls, f)
            assert (d.offset, d.size) == lay[f"{s}.{f}"], (s, f, (d.offset, d.size), lay[f"{s}.{f}"])


def test_opts_default_matches_the_c_default():
    """xs_opts_default (C) and the binding agree: S, material_energy, no sharding"""
    from paper_conf_cgo_murtovigplls24_b200 import _xs
    o = _xs.xs_opts_default()
    assert (o.search, o.sort, o.block, o.energy_bins, o.flags, o.history_len) == (_xs.XS_SEARCH_S,
                                                                                 _xs.XS_SORT_MATERIAL_ENERGY,
                                                                                 0, 0, 0, 0)
    assert (o.shard_index, o.shard_count) == (0, 1)
