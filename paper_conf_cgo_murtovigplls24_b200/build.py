"""Build libxs.so in-tree: nvcc for sm_100a only (no JIT cache, no other arch)."""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
ROOT = os.path.dirname(HERE)
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(HERE, "libxs.so")
BUILD = os.path.join(HERE, "_build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

SOURCES = ["api.cu", "grid.cu", "sort.cu", "lookup_fused.cu", "lookup_staged.cu", "lookup_split.cu", "pipeline.cu", "bezier.cu"]
HEADERS = ["rng.cuh", "search.cuh", "search_uu.cuh", "xs_internal.cuh", "lookup_common.cuh"]
FLAGS = [
    "-O3", "-std=c++17",
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-lineinfo",
    "--fmad=false",           # no implicit contraction: every fma is explicit (R8)
    "-Xcompiler", "-fPIC",
    "-Xptxas", "-v",
    "-I", INCLUDE,
]


def source_digest() -> str:
    """sha256 (16 hex) over every source, header and flag that goes into libxs.so: the build
    identity profiles/ncu_traffic.json records are keyed by (deterministic, unlike the binary's
    own bytes across rebuilds)."""
    import hashlib
    h = hashlib.sha256()
    for f in sorted(SOURCES + HEADERS):
        with open(os.path.join(CSRC, f), "rb") as fh:
            h.update(f.encode() + b"\0" + fh.read())
    with open(os.path.join(INCLUDE, "xs.h"), "rb") as fh:
        h.update(fh.read())
    h.update(" ".join(f for f in FLAGS if not f.startswith("/")).encode())
    return h.hexdigest()[:16]


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [os.path.join(INCLUDE, "xs.h"), __file__]
    return any(os.path.getmtime(d) > t for d in deps)


def _compile(src: str, bdir: str = BUILD, defines=()) -> str:
    obj = os.path.join(bdir, src.replace(".cu", ".o"))
    log = os.path.join(bdir, src.replace(".cu", ".ptxas.log"))
    cmd = [NVCC, *FLAGS, *defines, "-c", os.path.join(CSRC, src), "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    with open(log, "w") as f:
        f.write(r.stdout + r.stderr)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr[-4000:]}")
    return obj


def build(force: bool = False, verbose: bool = False, defines=(), out: str | None = None) -> str:
    """defines/out: experimental variants (e.g. -DXS_LOOKUP_MIN_BLOCKS=4 into libxs_mb4.so);
    the product is always libxs.so built with no extra defines."""
    lib = out or LIB
    if not force and not defines and out is None and not _stale():
        return LIB
    bdir = BUILD if not defines else BUILD + "_" + "_".join(d.strip("-D").replace("=", "") for d in defines)
    os.makedirs(bdir, exist_ok=True)
    with cf.ThreadPoolExecutor(len(SOURCES)) as ex:
        objs = list(ex.map(lambda s: _compile(s, bdir, defines), SOURCES))
    tmp = lib + ".tmp"
    cmd = [NVCC, "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-o", tmp, *objs]
    subprocess.run(cmd, check=True)
    os.replace(tmp, lib)
    if verbose:
        print(f"built {LIB}", file=sys.stderr)
    return LIB


if __name__ == "__main__":
    defs = tuple(a for a in sys.argv[1:] if a.startswith("-D"))
    outs = [a.split("=", 1)[1] for a in sys.argv[1:] if a.startswith("--out=")]
    build(force="--force" in sys.argv, verbose=True, defines=defs, out=outs[0] if outs else None)
