"""Summarise ptxas -v logs: kernel, registers, spill bytes, stack (development aid)."""
import glob, os, re, sys
d = sys.argv[1] if len(sys.argv) > 1 and sys.argv[1] else os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "paper_conf_cgo_murtovigplls24_b200", "_build")
pat = sys.argv[2] if len(sys.argv) > 2 else ""
for log in sorted(glob.glob(os.path.join(d, "*.ptxas.log"))):
    txt = open(log).read()
    for m in re.finditer(r"Compiling entry function '([^']+)'[^\n]*\n[^\n]*\n\s*(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads\n[^\n]*Used (\d+) registers", txt):
        name, stack, ss, sl, regs = m.groups()
        short = re.sub(r"EEEvNS_.*|EvNS_.*", "", name.replace("_ZN2xs", ""))
        if pat in short:
            print(f"{os.path.basename(log)[:-10]:14s} {short:40s} regs={regs:>3s} stack={stack:>4s} spill={ss}/{sl}")
