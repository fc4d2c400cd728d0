"""SASS structure of the search variants inside a kernel of libxs.so (tests/test_sass.py; the
paper's A/B is about control flow, so it is checked where nvcc could undo it: in SASS).

A *probe* is a `LDG.E.64.CONSTANT` (the search's 8 B read-only load of A[mid]; the 96 B
gathers are LDG.E.128).  For each probe the compare that consumes its register is found
(`DSETP`), then what consumes that predicate: a predicated `BRA` (the paths are separate:
unmerged) or a `SEL`/predicated ALU op (if-converted: merged / select form)."""
from __future__ import annotations

import re
import subprocess

CUOBJDUMP = "/usr/local/cuda/bin/cuobjdump"
_INS = re.compile(r"/\*([0-9a-f]{4,})\*/\s+(.*?)\s*;")


def kernel_sass(lib: str, mangled: str) -> list[str]:
    out = subprocess.run([CUOBJDUMP, "-sass", "-fun", mangled, lib], capture_output=True, text=True).stdout
    return [m.group(2) for m in _INS.finditer(out)]


def _regs(op: str) -> list[str]:
    return re.findall(r"\bR\d+\b", op)


def shape(ins: list[str]) -> dict:
    probes = branch = select = 0
    sites = []
    for i, s in enumerate(ins):
        if not s.startswith("LDG.E.64.CONSTANT"):
            continue
        dst = _regs(s)[0]
        # the compare that reads the probed value
        k = next((j for j in range(i + 1, min(i + 40, len(ins)))
                  if ins[j].startswith("DSETP") and dst in _regs(ins[j].split(",", 1)[1])), None)
        if k is None:
            continue
        probes += 1
        pm = re.match(r"DSETP\.\S+ (P\d)", ins[k])
        p = pm.group(1) if pm else None
        used = None
        for j in range(k + 1, min(k + 8, len(ins))):
            t = ins[j]
            if p and re.match(rf"@!?{p} BRA", t):
                used = "branch"
                break
            if p and (re.search(rf"\bSEL .*!?{p}\b", t) or re.match(rf"@!?{p} (IADD3|IMAD|MOV|SEL)", t)):
                used = "select"
                break
        branch += used == "branch"
        select += used == "select"
        sites.append(used)
    return {"probes": probes, "branch": branch, "select": select, "n_ins": len(ins),
            "bra": sum(1 for s in ins if re.search(r"\bBRA\b", s)),
            "tt_guard": sum(1 for s in ins if re.search(r"ISETP\.(GE\.U32\.AND P\d, PT, R\d+, 0x4|GT\.U32\.AND P\d, PT, R\d+, 0x3)\b", s)),
            "shr2": sum(1 for s in ins if re.search(r"SHF\.R\.U32\.HI R\d+, RZ, 0x2, R\d+", s))}


def mangled_k_lookup(grid: int, search: int, sorted_: bool, outs: bool = False, ilp2: bool = False) -> str:
    b = lambda x: "1" if x else "0"
    return (f"_ZN2xs8k_lookupILi{grid}ELi{search}ELb{b(sorted_)}ELb{b(outs)}ELb{b(ilp2)}EEEvNS_8GridViewENS_10"
            "SampleViewENS_10SortedViewENS_6AffineEPdPiPy")
